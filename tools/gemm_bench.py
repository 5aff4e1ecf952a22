"""Microbenchmark of the tcgen05 GEMM (qos_op_gemm_ex) on the Llama-3-8B projection shapes across
M (= tokens in the step): achieved TFLOP/s and weight-streaming GB/s per launch.

  python tools/gemm_bench.py [--ms 16,64,128,256,512,2176] [--ksplit 0]
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402

SHAPES = {"qkv": (6144, 4096, "store_bf16"), "o": (4096, 4096, "add_f32"), "gateup": (28672, 4096, "silu_gate"),
          "down": (4096, 14336, "add_f32"), "head": (128256, 4096, "store_f32")}

ap = argparse.ArgumentParser()
ap.add_argument("--ms", default="16,64,128,256,384,512,1024,2176")
ap.add_argument("--ksplit", type=int, default=0)
ap.add_argument("--iters", type=int, default=20)
a = ap.parse_args()
torch.cuda.set_device(0)
flush = torch.empty(256 * 1024 * 1024, dtype=torch.uint8, device="cuda")   # > L2: weights come from HBM
for name, (N, K, epi) in SHAPES.items():
    B = (torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
    for M in [int(x) for x in a.ms.split(",")]:
        if name == "head" and M > 512:
            continue
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        Cn = N // 2 if epi == "silu_gate" else N
        Cout = torch.zeros(M, Cn, device="cuda", dtype=torch.float32 if "f32" in epi else torch.bfloat16)
        ts = []
        for it in range(a.iters + 3):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            q.qos_op_gemm_ex(A.data_ptr(), B.data_ptr(), Cout.data_ptr(), M, N, K, epi, None, a.ksplit)
            e1.record()
            torch.cuda.synchronize()
            if it >= 3:
                ts.append(e0.elapsed_time(e1))
        ts.sort()
        ms = ts[len(ts) // 2]
        print(json.dumps({"gemm": name, "M": M, "N": N, "K": K, "us": round(ms * 1e3, 1),
                          "tflops": round(2 * M * N * K / ms / 1e9, 1),
                          "weight_gbs": round(N * K * 2 / ms / 1e6, 1)}), flush=True)
