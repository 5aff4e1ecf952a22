"""Quick device-timed sweep of hybrid-step latency (qos_profile_step) on Llama-3-8B shapes.
  python tools/sweep.py --points 256:0:0,256:128:1024,2048:128:4096  [--layers L] [--reps 5]
Each point is chunk:n_decode:ctx[:kv_start] (kv_start 0 by default: the chunk's cached prefix).
Prints one JSON line per point."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.presets import preset  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--points", default="256:0:0,512:0:0,256:128:1024,512:128:1024,2048:128:4096,8192:0:0")
ap.add_argument("--layers", type=int, default=None)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--breakdown", action="store_true", help="per-kernel-class ms per step (events)")
a = ap.parse_args()
import torch  # noqa: E402
torch.cuda.set_device(0)
pts = [tuple(int(x) for x in p.split(":")) for p in a.points.split(",")]
pts = [p if len(p) == 4 else p + (0,) for p in pts]
need = max(nd * (ctx + 1) + ks + c for c, nd, ctx, ks in pts) + 9000
over = {} if a.layers is None else {"n_layers": a.layers}
cfg = q.model_cfg(**preset("llama3-8b", **over), num_blocks=need // 16 + 600, max_seq_len=16384, max_requests=300,
                  max_batch_tokens=8192 + 256, max_batch_rows=257)
eng = q.Engine(cfg)
eng.qos_engine_load_synthetic(0)
for c, nd, ctx, ks in pts:
    if a.breakdown:
        eng.qos_engine_set_timing(True)
    ms, p95 = eng.qos_profile_step(c, [ctx] * nd, reps=a.reps, kv_start=ks)
    rec = {"chunk": c, "n_decode": nd, "ctx": ctx, "kv_start": ks, "ms": round(ms, 3), "p95": round(p95, 3),
           "tok_s": round((c + nd) / ms * 1e3)}
    if a.breakdown:
        tm = eng.qos_last_step_timing()
        rec["breakdown"] = {k: round(v[0] / (3 + a.reps), 3) for k, v in tm.items() if v[1]}
        eng.qos_engine_set_timing(False)
    print(json.dumps(rec), flush=True)
eng.close()
