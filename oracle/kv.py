"""Paged KV block allocator of the oracle (test infrastructure only).

The paper keeps requests' KV resident in vLLM's paged cache (§3.6) and only
while needed (§3.4 "KV-cache ... remains in the GPU for the shortest
necessary duration").  Block size and placement policy are not stated; reading s12
(DESIGN.md §2): block size 16, lowest free block index first, all-or-nothing growth, no
prefix sharing.  The CUDA library's allocator must produce bit-identical tables for the same
sequence of alloc/free calls (tests/test_kv_tables.py).
"""
from __future__ import annotations

import heapq


class OracleOOM(Exception):
    pass


class OracleUnknownReq(Exception):
    pass


class BlockAllocator:
    def __init__(self, num_blocks: int, block_size: int = 16):
        self.num_blocks = int(num_blocks)
        self.block_size = int(block_size)
        self._free = list(range(self.num_blocks))   # already a valid min-heap
        self.tables: dict[int, list[int]] = {}

    @property
    def n_free(self) -> int:
        return len(self._free)

    def alloc(self, req: int, n_tokens_total: int) -> None:
        """Grow ``req``'s table to ceil(n_tokens_total / block_size) blocks, taking the lowest
        free indices in ascending order; OOM leaves the state unchanged."""
        if n_tokens_total < 0:
            raise ValueError("n_tokens_total < 0")
        need_total = -(-n_tokens_total // self.block_size)
        table = self.tables.get(req, [])
        need = need_total - len(table)
        if need > len(self._free):
            raise OracleOOM(f"need {need} blocks, {len(self._free)} free")
        new = [heapq.heappop(self._free) for _ in range(max(0, need))]
        self.tables[req] = table + new

    def free(self, req: int) -> None:
        if req not in self.tables:
            raise OracleUnknownReq(req)
        for b in self.tables.pop(req):
            heapq.heappush(self._free, b)

    def table(self, req: int) -> list[int]:
        if req not in self.tables:
            raise OracleUnknownReq(req)
        return list(self.tables[req])
