"""Run the bench workload for a few steps with an NVTX range "step" around each, for ncu:

  ncu --metrics gpu__time_duration.sum --clock-control none --nvtx --nvtx-include "step/" \
      --csv --log-file gpurun_out/launches.csv python tools/profile_step.py --steps 1
  ncu --set full --clock-control none --import-source on --nvtx --nvtx-include "step/" \
      -k regex:gemm_tcgen05 -s 2 -c 1 -o gpurun_out/prof python tools/profile_step.py --steps 1
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import bench  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--steps", type=int, default=1)
ap.add_argument("--warmup", type=int, default=2)
ap.add_argument("--chunk", type=int, default=bench.CHUNK)
ap.add_argument("--n-dec", type=int, default=bench.N_DEC)
ap.add_argument("--ctx", type=int, default=bench.CTX)
ap.add_argument("--layers", type=int, default=None)
a = ap.parse_args()
torch.cuda.set_device(0)
wl = bench.Workload(0, a.warmup + a.steps + 2, chunk=a.chunk, n_dec=a.n_dec, ctx=a.ctx, n_layers=a.layers)
s = torch.cuda.current_stream().cuda_stream
out = torch.empty(a.n_dec + 1, dtype=torch.int32, device="cuda")
for _ in range(a.warmup):
    wl.step(wl.next_batch(), out.data_ptr(), False, s)
torch.cuda.synchronize()
for _ in range(a.steps):
    b = wl.next_batch()
    torch.cuda.nvtx.range_push("step")
    wl.step(b, out.data_ptr(), False, s)
    torch.cuda.nvtx.range_pop()
torch.cuda.synchronize()
print("done")
