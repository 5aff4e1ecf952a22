import os, sys, time
sys.path.insert(0, os.getcwd())
import numpy as np, torch
import bench
torch.cuda.set_device(0)
wl = bench.Workload(0, 40)
s = torch.cuda.current_stream().cuda_stream
out = torch.empty(bench.N_DEC + 1, dtype=torch.int32, device="cuda")
host = np.empty(bench.N_DEC + 1, dtype=np.int32)
for _ in range(3):
    wl.step(wl.next_batch(), out.data_ptr(), False, s)
torch.cuda.synchronize()
tb, tl, ts = [], [], []
for _ in range(10):
    t0 = time.perf_counter(); b = wl.next_batch(); t1 = time.perf_counter()
    wl.eng.qos_hybrid_step(b, None, wl.q.QOS_F32, out.data_ptr(), False, s); t2 = time.perf_counter()
    torch.cuda.synchronize(); t3 = time.perf_counter()
    wl.retire()
    tb.append(t1 - t0); tl.append(t2 - t1); ts.append(t3 - t1)
print("next_batch ms", np.median(tb) * 1e3, "enqueue ms", np.median(tl) * 1e3, "step wall ms", np.median(ts) * 1e3)
te = []
for _ in range(10):
    b = wl.next_batch()
    t0 = time.perf_counter()
    wl.eng.qos_hybrid_step(b, None, wl.q.QOS_F32, host.ctypes.data, True, s)
    te.append(time.perf_counter() - t0)
    wl.retire()
print("on_host step ms", np.median(te) * 1e3)
