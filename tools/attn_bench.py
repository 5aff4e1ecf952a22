"""Device-timed attention throughput on Llama-3-8B shapes (per-kernel-class CUDA events inside
qos_profile_step): prefill attention in TFLOP/s of algorithmic causal work
4*hd*H*L*sum_c[len*kv_start + len(len+1)/2] and decode attention in GB/s of 4*hd*Hkv*L*sum(ctx+1).

  python tools/attn_bench.py [--layers 4] [--reps 5] [--points 2048:0:0:0,2048:0:0:6144,...]
Each point is chunk:n_decode:ctx:kv_start.  Prints one JSON line per point."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.presets import preset  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--points", default="512:0:0:0,2048:0:0:0,2048:0:0:6144,8192:0:0:0,0:128:4096:0")
ap.add_argument("--layers", type=int, default=4)
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--variants", default="",
                help="A/B in one process: 'fa_poly=0;fa_poly=4' (engine options; they persist from one "
                     "variant to the next, so name every option a variant touches in every variant)")
ap.add_argument("--rounds", type=int, default=1, help="interleaved repetitions of all variants")
ap.add_argument("--step-only", action="store_true",
                help="whole-step device time only (no per-kernel events, attention overlap left on)")
a = ap.parse_args()
import threading  # noqa: E402
import time  # noqa: E402

import torch  # noqa: E402


class ClockSampler:
    """SM clock (MHz) sampled every 5 ms while active (nvml)."""

    def __init__(self):
        import pynvml
        pynvml.nvmlInit()
        self.nv, self.h = pynvml, pynvml.nvmlDeviceGetHandleByIndex(0)
        self.samples, self.on = [], False

    def __enter__(self):
        self.samples, self.on = [], True
        self.t = threading.Thread(target=self._run, daemon=True)
        self.t.start()
        return self

    def _run(self):
        while self.on:
            self.samples.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            time.sleep(0.005)

    def __exit__(self, *exc):
        self.on = False
        self.t.join()

    def median(self):
        s = sorted(self.samples)
        return s[len(s) // 2] if s else None



torch.cuda.set_device(0)
pts = [tuple(int(x) for x in p.split(":")) for p in a.points.split(",")]
need = max(nd * (ctx + 1) + ks + c for c, nd, ctx, ks in pts) + 9000
P = preset("llama3-8b", n_layers=a.layers)
cfg = q.model_cfg(**P, num_blocks=need // 16 + 600, max_seq_len=16384, max_requests=300,
                  max_batch_tokens=8192 + 256, max_batch_rows=257)
eng = q.Engine(cfg)
eng.qos_engine_load_synthetic(0)
L, H, Hkv, hd = P["n_layers"], P["n_heads"], P["n_kv_heads"], P["head_dim"]
if not a.step_only:
    eng.qos_engine_set_option("overlap_attn", 0)
variants = [v for v in a.variants.split(";") if v] or [""]


def run_point(c, nd, ctx, ks, tag):
    if a.step_only:
        with ClockSampler() as clk:
            ms, _ = eng.qos_profile_step(c, [ctx] * nd, reps=a.reps, kv_start=ks)
        print(json.dumps({"variant": tag, "chunk": c, "n_decode": nd, "ctx": ctx, "kv_start": ks, "layers": L,
                          "step_ms": round(ms, 3), "sm_mhz": clk.median()}), flush=True)
        return
    eng.qos_engine_set_timing(True)
    with ClockSampler() as clk:
        ms, _ = eng.qos_profile_step(c, [ctx] * nd, reps=a.reps, kv_start=ks)
    tm = eng.qos_last_step_timing()
    eng.qos_engine_set_timing(False)
    rec = {"variant": tag, "chunk": c, "n_decode": nd, "ctx": ctx, "kv_start": ks, "layers": L, "step_ms": round(ms, 3),
           "sm_mhz": clk.median()}
    if c:
        t, n = tm["prefill_attn"]
        per = t / n
        fl = 4 * hd * H * (c * ks + c * (c + 1) // 2)
        rec.update(prefill_us_per_layer=round(per * 1e3, 2), prefill_tflops=round(fl / (per * 1e-3) / 1e12, 1))
    if nd:
        t, n = tm["decode_attn"]
        per = t / n
        by = 4 * hd * Hkv * nd * (ctx + 1)
        rec.update(decode_us_per_layer=round(per * 1e3, 2), decode_gbs=round(by / (per * 1e-3) / 1e9, 1))
    rec["us_per_launch"] = {k: round(t / n * 1e3, 1) for k, (t, n) in tm.items() if n}
    print(json.dumps(rec), flush=True)


for _ in range(a.rounds):
    for v in variants:
        for kv in (x for x in v.split(",") if x):
            k, val = kv.split("=")
            eng.qos_engine_set_option(k, int(val))
        for c, nd, ctx, ks in pts:
            run_point(c, nd, ctx, ks, v)
eng.close()
