"""Host cost of a step vs its device time (is the host enqueue hidden behind the GPU?).

  python tools/host_overhead.py [--chunk 2048 --n-dec 128 --ctx 4096 --layers 32]

Prints the medians of: building the descriptor, enqueueing qos_hybrid_step (device outputs), the
step's device time (CUDA events), the wall time of enqueue + synchronise, and the wall time of
the synchronous public call with host outputs (what a serving loop that feeds tokens back pays).
"""
import argparse
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402
import torch  # noqa: E402

import bench  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--chunk", type=int, default=bench.CHUNK)
ap.add_argument("--n-dec", type=int, default=bench.N_DEC)
ap.add_argument("--ctx", type=int, default=bench.CTX)
ap.add_argument("--layers", type=int, default=None)
ap.add_argument("--reps", type=int, default=10)
a = ap.parse_args()
torch.cuda.set_device(0)
wl = bench.Workload(0, 3 * a.reps + 8, chunk=a.chunk, n_dec=a.n_dec, ctx=a.ctx, n_layers=a.layers)
stream = torch.cuda.current_stream()
s = stream.cuda_stream
out = torch.empty(a.n_dec + 1, dtype=torch.int32, device="cuda")
host = np.empty(a.n_dec + 1, dtype=np.int32)
for _ in range(3):
    wl.step(wl.next_batch(), out.data_ptr(), False, s)
torch.cuda.synchronize()
tb, tl, ts, td = [], [], [], []
for _ in range(a.reps):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    t0 = time.perf_counter()
    b = wl.next_batch()
    t1 = time.perf_counter()
    e0.record(stream)
    wl.eng.qos_hybrid_step(b, None, wl.q.QOS_F32, out.data_ptr(), False, s)
    e1.record(stream)
    t2 = time.perf_counter()
    torch.cuda.synchronize()
    t3 = time.perf_counter()
    wl.retire()
    tb.append(t1 - t0)
    tl.append(t2 - t1)
    ts.append(t3 - t1)
    td.append(e0.elapsed_time(e1) * 1e-3)
# the synchronous public call with host outputs into pageable (numpy) and pinned memory,
# interleaved with enqueue + synchronise of the device-output call (same clock conditions)
pinned = torch.empty(a.n_dec + 1, dtype=torch.int32, pin_memory=True).numpy()
te, tp, ts2 = [], [], []
for _ in range(a.reps):
    for dst, acc in ((host, te), (pinned, tp), (None, ts2)):
        b = wl.next_batch()
        t0 = time.perf_counter()
        if dst is None:
            wl.eng.qos_hybrid_step(b, None, wl.q.QOS_F32, out.data_ptr(), False, s)
            torch.cuda.synchronize()
        else:
            wl.eng.qos_hybrid_step(b, None, wl.q.QOS_F32, dst.ctypes.data, True, s)
        acc.append(time.perf_counter() - t0)
        wl.retire()
med = lambda x: round(float(np.median(x)) * 1e3, 3)  # noqa: E731
print(json.dumps({"chunk": a.chunk, "n_decode": a.n_dec, "ctx": a.ctx, "descriptor_ms": med(tb), "enqueue_ms": med(tl),
                  "device_ms": med(td), "enqueue_plus_sync_ms": med(ts), "public_call_host_outputs_ms": med(te),
                  "public_call_pinned_outputs_ms": med(tp), "interleaved_enqueue_plus_sync_ms": med(ts2)}))
