"""HBM bandwidth ceilings on this box (context for the decode-attention roofline): device-timed
copy (read + write bytes) and read-only reductions over tensors far larger than L2.

  python tools/hbm_probe.py [--gib 4]
"""
import argparse
import json

import torch

ap = argparse.ArgumentParser()
ap.add_argument("--gib", type=float, default=4.0)
ap.add_argument("--iters", type=int, default=10)
a = ap.parse_args()
torch.cuda.set_device(0)
n = int(a.gib * (1 << 30)) // 2
x = torch.empty(n, dtype=torch.bfloat16, device="cuda").uniform_(-1, 1)
y = torch.empty_like(x)


def timed(fn, nbytes):
    for _ in range(3):
        fn()
    torch.cuda.synchronize()
    best = float("inf")
    for _ in range(a.iters):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        torch.cuda.synchronize()
        best = min(best, e0.elapsed_time(e1) * 1e-3)
    return round(nbytes / best / 1e9, 1)


xi = x.view(torch.int64)
print(json.dumps({"copy_gbs": timed(lambda: y.copy_(x), 4 * n),
                  "sum_bf16_gbs": timed(lambda: x.sum(dtype=torch.float32), 2 * n),
                  "max_i64_gbs": timed(lambda: xi.max(), 2 * n),
                  "gib": a.gib}), flush=True)
