"""Refit the latency model (paper_conf_asplos_goelmkar26_b200.latency_model, current features)
on the MEASURED points of a latency-table JSON written by tools/latency_table.py, and re-score
its random test batches — no new measurements.  Every feature is a function of (chunk,
kv_start, n_decode, sum of decode contexts), which the JSON records per point.

  python tools/latency_refit.py gpurun_out/latency_table_r1d.json --out profiles/latency_table_r1.json
"""
import argparse
import json
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_goelmkar26_b200.latency_model import LatencyModel, StepShape  # noqa: E402


def shape_of(r):
    nd = r["n_decode"]
    if "sum_ctx" in r:
        ctx = [r["sum_ctx"] // nd] * nd if nd else []
        if nd:
            ctx[0] += r["sum_ctx"] - sum(ctx)
    else:
        ctx = [r["ctx"]] * nd
    return StepShape([(r["kv_start"], r["chunk"])] if r["chunk"] else [], ctx)


ap = argparse.ArgumentParser()
ap.add_argument("table")
ap.add_argument("--out", required=True)
a = ap.parse_args()
d = json.load(open(a.table))
fit = [shape_of(r) for r in d["table"]]
fy = [r["ms"] for r in d["table"]]
m = LatencyModel().fit(fit, fy)
fit_err = [abs(m.predict(s) - y) / y for s, y in zip(fit, fy)]
for r in d["tests"]:
    r["pred_ms"] = m.predict(shape_of(r))
    r["rel_err"] = abs(r["pred_ms"] - r["ms"]) / r["ms"]
errs = np.array([r["rel_err"] for r in d["tests"]])
d.update(fit_rel_err_max=float(max(fit_err)), test_rel_err_max=float(errs.max()),
         test_rel_err_p95=float(np.percentile(errs, 95)), test_rel_err_mean=float(errs.mean()),
         within_5pct=float((errs <= 0.05).mean()), model_json=json.loads(m.to_json()),
         refit=f"model refit offline by tools/latency_refit.py on the measured points of {os.path.basename(a.table)}")
json.dump(d, open(a.out, "w"), indent=1)
print(json.dumps({k: v for k, v in d.items() if k not in ("table", "tests", "model_json")}))
