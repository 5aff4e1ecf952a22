"""Microbenchmark of the tcgen05 GEMMs (qos_op_gemm_ex) on the Llama-3-8B projection shapes
across M (= tokens in the step): per-launch time, achieved TFLOP/s and weight-streaming GB/s.

Launches run back to back (as in a step, PDL on) over rotating copies of the weight matrix
whose total size exceeds L2, so every launch streams its weights from HBM and no launch pays
for write-backs of a dirty L2 (a zero-fill flush before each launch costs ~20 us of write-back
to the next kernel and hides the small-M behaviour).

  python tools/gemm_bench.py [--ms 1,16,64,128,256,512,2176] [--ksplit 0] [--shapes qkv,o]
  ksplit: 0 auto, >= 1 tile kernel with that split-K, -1 weight-streaming (swap-AB) kernel

Caveat (round 2): the op entry point maps A with exactly M rows, so at M not a multiple of 128
the tile kernels' 128-row A boxes read out of bounds (TMA zero fill), which is measurably slower
(gate/up: 62 us at M = 112 vs 48 us at M = 128).  Inside the engine the activation maps span the
whole workspace and never go out of bounds — confirm kernel choices with an in-step A/B
(tools/attn_bench.py --step-only --variants ...), as profiles/step_swab_r2a.jsonl did.
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
ap.add_argument("--ms", default="1,16,64,128,256,384,512,1024,2176")
ap.add_argument("--ksplit", type=int, default=0)
ap.add_argument("--iters", type=int, default=24)
ap.add_argument("--shapes", default=",".join(SHAPES))
ap.add_argument("--epi", default=None, help="override the epilogue of every shape")
a = ap.parse_args()
torch.cuda.set_device(0)
L2 = 126 * 1024 * 1024
for name in a.shapes.split(","):
    N, K, epi = SHAPES[name]
    epi = a.epi or epi
    wbytes = N * K * 2
    ncopy = max(2, -(-3 * L2 // wbytes))
    Bs = [(torch.randn(N, K, device="cuda") / K ** 0.5).to(torch.bfloat16) for _ in range(ncopy)]
    for M in [int(x) for x in a.ms.split(",")]:
        if name == "head" and M > 512:
            continue
        A = torch.randn(M, K, device="cuda").to(torch.bfloat16)
        Cn = N // 2 if epi == "silu_gate" else N
        Cout = torch.zeros(M, Cn, device="cuda", dtype=torch.float32 if "f32" in epi else torch.bfloat16)

        def launch(i, st=None):
            q.qos_op_gemm_ex(A.data_ptr(), Bs[i % ncopy].data_ptr(), Cout.data_ptr(), M, N, K, epi, None, a.ksplit,
                             st)

        for i in range(ncopy + 2):
            launch(i)
        torch.cuda.synchronize()
        # captured in a CUDA graph so host-side launch cost does not starve short kernels
        s = torch.cuda.Stream()
        g = torch.cuda.CUDAGraph()
        with torch.cuda.graph(g, stream=s):
            for i in range(a.iters):
                launch(i, s.cuda_stream)
        g.replay()
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        g.replay()
        e1.record()
        torch.cuda.synchronize()
        us = e0.elapsed_time(e1) * 1e3 / a.iters
        print(json.dumps({"gemm": name, "epi": epi, "M": M, "N": N, "K": K, "ksplit": a.ksplit, "us": round(us, 2),
                          "tflops": round(2 * M * N * K / us / 1e6, 1),
                          "weight_gbs": round(wbytes / us / 1e3, 1)}), flush=True)
        del A, Cout
    del Bs
    torch.cuda.empty_cache()
