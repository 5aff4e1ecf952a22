"""CPU checks of the C-ABI library: it loads, exports every symbol include/*.h declares, and its
pure-host calls behave (no compute call needs a GPU here)."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
LIB = os.path.join(ROOT, "paper_conf_asplos_goelmkar26_b200", "libqoserve.so")


def _declared():
    names = set()
    for h in ("qoserve.h", "qoserve_ops.h"):
        src = open(os.path.join(ROOT, "include", h)).read()
        src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
        for m in re.finditer(r"^\s*(?:const\s+)?\w+\**\s+\**(qos_\w+)\s*\(", src, flags=re.M):
            names.add(m.group(1))
    return names


@pytest.fixture(scope="module")
def q():
    if not os.path.exists(LIB):
        import __graft_entry__
        __graft_entry__.build()
    from paper_conf_asplos_goelmkar26_b200 import qoserve
    return qoserve


def test_library_exports_every_declared_symbol(q):
    declared = _declared()
    assert len(declared) >= 25, declared
    lib = ctypes.CDLL(LIB)
    missing = [n for n in sorted(declared) if not hasattr(lib, n)]
    assert not missing, missing
    assert set(q.EXPORTED) == declared, set(q.EXPORTED) ^ declared


def test_strerror_and_mem_sizes(q):
    assert q.lib.qos_strerror(0) == b"ok"
    assert b"kv_start" in q.lib.qos_strerror(-4)
    from paper_conf_asplos_goelmkar26_b200.presets import preset
    cfg = q.model_cfg(**preset("llama3-8b"), num_blocks=1000, max_seq_len=8192)
    s1 = q.qos_engine_mem_sizes(cfg, 1)
    # body + embed + head bf16 = 8.03 B params * 2 B (SURVEY.md §8 presets: 16.06 GB)
    assert abs(s1.weight_bytes / 1e9 - 16.06) < 0.05
    # KV: L x 2 x blocks x Hkv x 16 x hd x 2 B = 128 KiB per token
    assert s1.kv_bytes == 32 * 2 * 1000 * 8 * 16 * 128 * 2
    s8 = q.qos_engine_mem_sizes(cfg, 8)
    assert s8.kv_bytes * 8 == s1.kv_bytes
    assert s8.weight_bytes < s1.weight_bytes / 4


def test_invalid_configs_rejected(q):
    from paper_conf_asplos_goelmkar26_b200.presets import preset
    bad = q.model_cfg(**preset("tiny", head_dim=96))
    with pytest.raises(q.QosError) as ei:
        q.qos_engine_mem_sizes(bad, 1)
    assert ei.value.name == "UNSUPPORTED"
    with pytest.raises(q.QosError) as ei:
        q.qos_engine_mem_sizes(q.model_cfg(**preset("llama3-8b")), 3)   # 3 does not divide 8
    assert ei.value.name == "INVALID_ARG"


def test_engine_create_fails_loudly_without_gpu(q):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    from paper_conf_asplos_goelmkar26_b200.presets import preset
    cfg = q.model_cfg(**preset("tiny"), num_blocks=64)
    with pytest.raises(q.QosError) as ei:
        q.Engine(cfg, torch_arenas=False)
    assert ei.value.name in ("CUDA", "OOM")


def test_peer_group_host_calls(q):
    """qos_group_create / qos_group_destroy are pure host calls (the in-process TP peer group)."""
    with pytest.raises(q.QosError) as ei:
        q.Group(1)
    assert ei.value.name == "INVALID_ARG"
    with pytest.raises(q.QosError):
        q.Group(9)
    g = q.Group(4)
    g.close()
    g.close()  # idempotent in the binding


def test_cross_process_group_host_calls(q):
    """qos_group_unique_id / qos_group_open / qos_group_destroy are host calls (POSIX shm):
    rank 0 creates the segment; a second open of the same id as rank 0 fails (O_EXCL); a
    non-zero rank of a missing segment times out."""
    import os
    gid = q.qos_group_unique_id()
    assert gid.startswith(b"/qoserve_grp_") and len(gid) == 64
    g0 = q.Group(2, gid, 0)
    with pytest.raises(q.QosError) as ei:
        q.Group(2, gid, 0)
    assert ei.value.name == "COMM"
    with pytest.raises(q.QosError) as ei:   # size mismatch with rank 0's segment
        q.Group(4, gid, 1)
    assert ei.value.name == "INVALID_ARG"
    g1 = q.Group(2, gid, 1)
    name = gid.rstrip(b"\0").decode()
    assert os.path.exists("/dev/shm" + name)
    g1.close()
    g0.close()
    assert not os.path.exists("/dev/shm" + name)     # unlinked by the last rank
    os.environ["QOS_GROUP_TIMEOUT_MS"] = "200"
    try:
        with pytest.raises(q.QosError) as ei:
            q.Group(2, q.qos_group_unique_id(), 1)
        assert ei.value.name == "COMM"
    finally:
        del os.environ["QOS_GROUP_TIMEOUT_MS"]
