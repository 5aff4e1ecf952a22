"""bench.py contract under torchrun (the driver's N > 1 launch): two replica ranks on the one GPU
of the test box (gloo for the rank plumbing when ranks share a device), a 2-layer model so both
engines fit; rank 0 prints exactly one JSON line with the whole-job value.  Round 1 passed the
replica's global rank as its TP rank (tp_size 1), which every rank > 0 rejected."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_bench_two_replica_ranks_print_one_line():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", "29531", "bench.py", "--gpus", "2", "--steps", "2",
           "--warmup", "3", "--layers", "2", "--no-cpu-baseline"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["value"] > 0 and d["gpu_launches"] > 0
