"""Per-clock efficiency of the projection GEMMs (ours vs cuBLAS) at one token count: run under
  ncu --metrics gpu__time_duration.sum,sm__cycles_elapsed.max --clock-control none --csv ...
and read FLOP / (cycles x 148 SMs) against the 8192 dense bf16 FLOP/clk/SM of sm_100.
  python tools/gemm_cycles.py [--m 2176] [--shapes qkv,o,gateup,down]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402

SHAPES = {"qkv": (6144, 4096, "store_bf16"), "o": (4096, 4096, "add_f32"), "gateup": (28672, 4096, "silu_gate"),
          "down": (4096, 14336, "add_f32")}
ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=2176)
ap.add_argument("--shapes", default="qkv,o,gateup,down")
a = ap.parse_args()
torch.cuda.set_device(0)
M = a.m
for name in a.shapes.split(","):
    N, K, epi = SHAPES[name]
    A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
    B = (torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16)
    Cn = N // 2 if epi == "silu_gate" else N
    C = torch.zeros(M, Cn, device="cuda", dtype=torch.float32 if "f32" in epi else torch.bfloat16)
    for _ in range(3):
        q.qos_op_gemm_ex(A.data_ptr(), B.data_ptr(), C.data_ptr(), M, N, K, epi, None, 0, None)
        torch.matmul(A, B.t())
    torch.cuda.synchronize()
    print(name, M, N, K, flush=True)
