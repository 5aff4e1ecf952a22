"""Pins of the oracle's paged-KV allocator (reading s12)."""
import json
import os

import numpy as np
import pytest

from oracle.kv import BlockAllocator, OracleOOM, OracleUnknownReq

GOLDEN = os.path.join(os.path.dirname(__file__), "golden", "kv_tables.json")


def test_block_counts_disjoint_conservation():
    a = BlockAllocator(200)
    rng = np.random.default_rng(0)
    live = {}
    for step in range(400):
        if live and rng.random() < 0.35:
            r = int(rng.choice(list(live)))
            a.free(r)
            del live[r]
        else:
            r = int(rng.integers(0, 40))
            n = int(rng.integers(0, 300))
            try:
                a.alloc(r, max(n, live.get(r, 0)))
                live[r] = max(n, live.get(r, 0))
            except OracleOOM:
                pass
        used = [b for t in a.tables.values() for b in t]
        assert len(used) == len(set(used))                       # disjoint
        assert len(used) + a.n_free == a.num_blocks              # conservation
        for r, n in live.items():
            assert len(a.tables[r]) == -(-n // 16)               # ceil(len/16)


def test_oom_leaves_state_unchanged():
    a = BlockAllocator(4)
    a.alloc(1, 40)            # 3 blocks
    before = (dict(a.tables), a.n_free)
    with pytest.raises(OracleOOM):
        a.alloc(2, 33)        # needs 3, only 1 free
    assert (dict(a.tables), a.n_free) == before


def test_unknown_free_raises():
    with pytest.raises(OracleUnknownReq):
        BlockAllocator(4).free(7)


def test_golden_table_sequence():
    """Hand-derived tables for a fixed alloc/free script (tests/golden/kv_tables.json): the
    expected lists follow from 'lowest free index first, ascending' by inspection."""
    g = json.load(open(GOLDEN))
    a = BlockAllocator(g["num_blocks"], 16)
    for op in g["script"]:
        if op[0] == "alloc":
            a.alloc(op[1], op[2])
        elif op[0] == "alloc_oom":
            with pytest.raises(OracleOOM):
                a.alloc(op[1], op[2])
        else:
            a.free(op[1])
    assert {int(k): v for k, v in g["expect"].items()} == a.tables
