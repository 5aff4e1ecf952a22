"""Refit the latency model (paper_conf_asplos_goelmkar26_b200.latency_model, current features)
on the MEASURED points of a latency-table JSON written by tools/latency_table.py — no new
measurements.

Protocol (--fit-random K): the model is fitted on the grid points PLUS the first K random
heterogeneous batches, and scored on the remaining random batches, which it never saw (a
held-out test set).  The paper's predictor is likewise trained on profiled batches
(§3.6.1); the grid alone (uniform contexts, three kv_start values) under-covers
the heterogeneous batches the scheduler forms.  The random batches' per-decode contexts are
replayed from the table's seeded generator (tools/latency_table.py: random_batches) when the
JSON does not store them.

  python tools/latency_refit.py gpurun_out/latency_table_r1e.json --fit-random 100 \
      --out profiles/latency_table_r1.json
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tools"))
from paper_conf_asplos_goelmkar26_b200.latency_model import LatencyModel, StepShape  # noqa: E402


def grid_shape(r):
    return StepShape([(r["kv_start"], r["chunk"])] if r["chunk"] else [], [r["ctx"]] * r["n_decode"])


def replay_ctx(d):
    """Per-decode contexts of the random batches, replayed from the seeded generator."""
    from latency_table import random_batches
    rng = np.random.default_rng(3)
    rng.permutation(len(d["table"]))      # the grid's profiling order draw comes first
    out = []
    for (chunk, ks, ctx), t in zip(random_batches(rng, len(d["tests"]), d["kv_capacity_tokens"]), d["tests"]):
        assert (chunk, ks, len(ctx), sum(ctx)) == (t["chunk"], t["kv_start"], t["n_decode"], t["sum_ctx"]), \
            "table was not written by this generator"
        out.append(ctx)
    return out


ap = argparse.ArgumentParser()
ap.add_argument("table")
ap.add_argument("--out", required=True)
ap.add_argument("--fit-random", type=int, default=0, help="random batches added to the fit set")
a = ap.parse_args()
d = json.load(open(a.table))
ctxs = [t["ctx"] for t in d["tests"]] if d["tests"] and "ctx" in d["tests"][0] else replay_ctx(d)
rshapes = [StepShape([(t["kv_start"], t["chunk"])], c) for t, c in zip(d["tests"], ctxs)]
k = a.fit_random
fit = [grid_shape(r) for r in d["table"]] + rshapes[:k]
fy = [r["ms"] for r in d["table"]] + [t["ms"] for t in d["tests"][:k]]
m = LatencyModel().fit(fit, fy)
fit_err = [abs(m.predict(s) - y) / y for s, y in zip(fit, fy)]
held = []
for i, (t, s) in enumerate(zip(d["tests"], rshapes)):
    t["ctx"] = ctxs[i]
    t["pred_ms"] = m.predict(s)
    t["rel_err"] = abs(t["pred_ms"] - t["ms"]) / t["ms"]
    t["in_fit"] = i < k
    if i >= k:
        held.append(t["rel_err"])
errs = np.array(held)
d.update(fit_points=len(fit), fit_rel_err_max=float(max(fit_err)), test_points=len(held),
         test_rel_err_max=float(errs.max()), test_rel_err_p95=float(np.percentile(errs, 95)),
         test_rel_err_mean=float(errs.mean()), within_5pct=float((errs <= 0.05).mean()),
         model_json=json.loads(m.to_json()),
         refit=(f"model refit offline by tools/latency_refit.py on the measured points of "
                f"{os.path.basename(a.table)}: fit = {len(d['table'])} grid points + the first {k} random "
                f"batches; test = the other {len(held)} random batches (held out)"))
json.dump(d, open(a.out, "w"), indent=1)
print(json.dumps({k2: v for k2, v in d.items() if k2 not in ("table", "tests", "model_json")}))
