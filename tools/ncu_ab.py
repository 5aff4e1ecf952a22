"""Clock-independent A/B of one kernel class: runs tools/attn_bench.py once per variant under
ncu (metrics only: duration and SM cycles, --clock-control none) and reports per point the
median kernel cycles and time.  Cycles do not move with the power-capped SM clock, which
swings 1.3-1.97 GHz between and within runs on this pool.

  python tools/ncu_ab.py --kernel prefill_attn --points 2048:0:0:6144,8192:0:0:0 \
      --variants "fa_qtiles=1;fa_qtiles=2"
"""
import argparse
import csv
import json
import os
import statistics
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
ap = argparse.ArgumentParser()
ap.add_argument("--kernel", default="prefill_attn")
ap.add_argument("--points", default="2048:0:0:0,2048:0:0:6144,8192:0:0:0")
ap.add_argument("--variants", default="")
ap.add_argument("--layers", type=int, default=2)
ap.add_argument("--reps", type=int, default=2)
a = ap.parse_args()
os.makedirs(os.path.join(ROOT, "gpurun_out"), exist_ok=True)
for v in [x for x in a.variants.split(";")] or [""]:
    for pt in a.points.split(","):
        log = os.path.join(ROOT, "gpurun_out", "ncu_ab.csv")
        cmd = ["ncu", "--metrics", "gpu__time_duration.sum,sm__cycles_elapsed.max", "--clock-control", "none",
               "-k", "regex:" + a.kernel, "--csv", "--log-file", log, sys.executable,
               os.path.join(ROOT, "tools", "attn_bench.py"), "--points", pt, "--layers", str(a.layers), "--reps",
               str(a.reps)] + (["--variants", v] if v else [])
        subprocess.run(cmd, capture_output=True, text=True, timeout=600)
        rows = list(csv.reader(open(log)))
        i = [k for k, r in enumerate(rows) if "Metric Name" in r][0]
        h = rows[i]
        mn, mv = h.index("Metric Name"), h.index("Metric Value")
        us, cyc = [], []
        for r in rows[i + 1:]:
            if len(r) <= mv:
                continue
            val = float(r[mv].replace(",", ""))
            if r[mn] == "gpu__time_duration.sum":
                us.append(val / 1e3 if "ns" in r[h.index("Metric Unit")] else val)
            elif r[mn] == "sm__cycles_elapsed.max":
                cyc.append(val)
        c, nd, ctx, ks = (int(x) for x in pt.split(":"))
        rec = {"variant": v, "point": pt, "launches": len(cyc), "kcycles_median": round(statistics.median(cyc) / 1e3, 1),
               "us_median": round(statistics.median(us), 2),
               "kcycles_sum": round(sum(cyc) / 1e3, 1)}
        if c and a.kernel.startswith("prefill"):
            fl = 4 * 128 * 32 * (c * ks + c * (c + 1) // 2)  # Llama-3-8B: hd 128, 32 heads
            rec["flop_per_cycle_per_sm"] = round(fl / (statistics.median(cyc) * 148), 1)
        print(json.dumps(rec), flush=True)
