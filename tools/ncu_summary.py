"""Summarise ncu outputs into profiles/: per-kernel share of one step (launch list CSV) and the
key counters of `--set full` captures.  Usage:
  python tools/ncu_summary.py --tag r1 --launches gpurun_out/launches_r1.csv \
      --rep gemm_gateup=gpurun_out/prof_gateup_r1.ncu-rep --rep decode_attn=gpurun_out/prof_decode_r1.ncu-rep ...
Writes profiles/<tag>_ncu_summary.md and updates profiles/roofline_traffic.json."""
import argparse
import collections
import csv
import json
import os
import shutil
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
           "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
           "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__grid_size", "launch__block_size",
           "sm__cycles_elapsed.avg.per_second", "lts__t_bytes.sum"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "usecond": 1e-6,
         "ms": 1e-3, "msecond": 1e-3, "nsecond": 1e-9}


def launches(path):
    rows = list(csv.reader(open(path)))
    i = [k for k, r in enumerate(rows) if "Kernel Name" in r][0]
    h = rows[i]
    kn, mv, mu = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
    tot, cnt = collections.defaultdict(float), collections.Counter()
    for r in rows[i + 1:]:
        try:
            v = float(r[mv].replace(",", "")) * SCALE.get(r[mu], 1.0)
        except (ValueError, IndexError):
            continue
        name = r[kn].split("(")[0].replace("void ", "")
        tot[name] += v
        cnt[name] += 1
    return tot, cnt


def rep(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for m in METRICS:
            if m in hdr:
                j = hdr.index(m)
                d[m] = (r[j], units[j])
        res.append(d)
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--tag", required=True)
    ap.add_argument("--launches")
    ap.add_argument("--rep", action="append", default=[])
    ap.add_argument("--note", default="")
    a = ap.parse_args()
    lines = [f"# ncu summary {a.tag}", "", a.note, ""]
    if a.launches:
        dst = os.path.join(ROOT, "profiles", os.path.basename(a.launches))
        shutil.copy(a.launches, dst)
        tot, cnt = launches(a.launches)
        T = sum(tot.values())
        lines += [f"## launch list (`{os.path.basename(a.launches)}`): one step, serialised, cold-cache",
                  "", f"total {T*1e3:.2f} ms over {sum(cnt.values())} launches", "",
                  "| kernel | launches | total ms | share | avg us |", "|---|---|---|---|---|"]
        for k, v in sorted(tot.items(), key=lambda x: -x[1]):
            lines.append(f"| `{k}` | {cnt[k]} | {v*1e3:.3f} | {100*v/T:.1f}% | {v/cnt[k]*1e6:.1f} |")
        lines.append("")
    traffic_path = os.path.join(ROOT, "profiles", "roofline_traffic.json")
    traffic = json.load(open(traffic_path)) if os.path.exists(traffic_path) else {}
    for spec in a.rep:
        key, path = spec.split("=", 1)
        for d in rep(path):
            lines += [f"## `--set full` capture: {key}", "", f"kernel: `{d['kernel']}`", "",
                      "| metric | value | unit |", "|---|---|---|"]
            for m in METRICS:
                if m in d:
                    lines.append(f"| {m} | {d[m][0]} | {d[m][1]} |")
            lines.append("")
            rd = float(d["dram__bytes_read.sum"][0].replace(",", "")) * SCALE[d["dram__bytes_read.sum"][1]]
            wr = float(d["dram__bytes_write.sum"][0].replace(",", "")) * SCALE[d["dram__bytes_write.sum"][1]]
            traffic[key] = {"dram_bytes_per_launch": rd + wr, "tag": a.tag, "kernel": d["kernel"]}
    json.dump(traffic, open(traffic_path, "w"), indent=1)
    open(os.path.join(ROOT, "profiles", f"{a.tag}_ncu_summary.md"), "w").write("\n".join(lines) + "\n")


if __name__ == "__main__":
    main()
