"""Overlap physics probe: can the HBM-bound decode work and the tensor-bound prefill work of a
hybrid step run concurrently on one B200 faster than back to back (under the 1 kW power cap)?

Two engines (Llama-3-8B shapes, same synthetic weights) on two streams:
  A: decode-only steps (n_dec decodes @ctx), B: prefill-only steps (one chunk @kv_start 0).
Reports device time of K steps of A alone, B alone, A||B interleaved on two streams, and the
fused hybrid step of the same rows (engine B, chunk + decodes), each with the median SM clock.

  python tools/overlap_probe.py [--layers 32] [--steps 6] [--gemm-sms 0,120] 
"""
import argparse
import json
import os
import sys
import threading
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_asplos_goelmkar26_b200 import qoserve as q  # noqa: E402
from paper_conf_asplos_goelmkar26_b200.presets import preset  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--layers", type=int, default=32)
ap.add_argument("--steps", type=int, default=6)
ap.add_argument("--chunk", type=int, default=2048)
ap.add_argument("--n-dec", type=int, default=128)
ap.add_argument("--ctx", type=int, default=4096)
ap.add_argument("--gemm-sms", default="0", help="SM budgets of engine B's GEMMs to try in A||B")
ap.add_argument("--a-gemm-sms", default="0")
a = ap.parse_args()
import torch  # noqa: E402


class Clk:
    def __init__(self):
        import pynvml
        pynvml.nvmlInit()
        self.nv, self.h = pynvml, pynvml.nvmlDeviceGetHandleByIndex(0)

    def __enter__(self):
        self.s, self.on = [], True
        self.t = threading.Thread(target=self.run, daemon=True)
        self.t.start()
        return self

    def run(self):
        while self.on:
            self.s.append(self.nv.nvmlDeviceGetClockInfo(self.h, self.nv.NVML_CLOCK_SM))
            time.sleep(0.005)

    def __exit__(self, *x):
        self.on = False
        self.t.join()

    def med(self):
        s = sorted(self.s)
        return s[len(s) // 2] if s else None


torch.cuda.set_device(0)
K = a.steps
P = preset("llama3-8b", n_layers=a.layers)
ctx_cap = a.ctx + 4 * K + 64


def mk(n_dec, chunk):
    nb = n_dec * ((ctx_cap + 15) // 16) + (4 * K + 8) * ((chunk + 15) // 16) + 64
    cfg = q.model_cfg(**P, num_blocks=nb, max_seq_len=8192, max_requests=n_dec + 64,
                      max_batch_tokens=chunk + n_dec + 2, max_batch_rows=n_dec + 2)
    e = q.Engine(cfg)
    e.qos_engine_load_synthetic(synth.SEED_WEIGHTS)
    e.qos_engine_set_option("shares_device", 1)   # no co-residency-dependent GEMM paths (two engines, one GPU)
    return cfg, e


class Stream:
    def __init__(self, n_dec, chunk):
        self.cfg, self.eng = mk(n_dec, chunk)
        self.n_dec, self.chunk = n_dec, chunk
        self.dec = list(range(1, n_dec + 1))
        for r in self.dec:
            self.eng.qos_kv_alloc(r, ctx_cap)
            self.eng.qos_kv_fill_synthetic(r, a.ctx, synth.SEED_KVFILL)
        self.ctx = {r: a.ctx for r in self.dec}
        self.toks = synth.request_tokens(0, max(1, chunk), self.cfg.vocab)
        self.nxt, self.live = 10_000, []
        self.out = torch.empty(n_dec + 2, dtype=torch.int32, device="cuda")

    def step(self, s, with_dec=True, with_chunk=True):
        pre = []
        if self.chunk and with_chunk:
            cr = self.nxt
            self.nxt += 1
            self.eng.qos_kv_alloc(cr, self.chunk)
            self.live.append(cr)
            pre = [(cr, 0, self.toks)]
        dec = []
        if with_dec:
            dec = [(r, self.ctx[r], (r * 7 + self.ctx[r]) % self.cfg.vocab) for r in self.dec]
            for r in self.dec:
                self.ctx[r] += 1
        self.eng.qos_hybrid_step(q.make_batch(pre, dec), None, q.QOS_F32, self.out.data_ptr(), 0, s.cuda_stream)
        while len(self.live) > 2:
            self.eng.qos_kv_free(self.live.pop(0))


sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
A = Stream(a.n_dec, 0)          # decode-only
B = Stream(a.n_dec, a.chunk)    # prefill-only (and the fused hybrid step)


def timed(fn):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(sa)
    sb.wait_event(e0)
    with Clk() as c:
        fn()
        eb = torch.cuda.Event()
        eb.record(sb)
        sa.wait_event(eb)
        e1.record(sa)
        torch.cuda.synchronize()
    return e0.elapsed_time(e1) / K, c.med()


def run_a():
    for _ in range(K):
        A.step(sa)


def run_b():
    for _ in range(K):
        B.step(sb, with_dec=False)


def run_ab():
    for _ in range(K):
        A.step(sa)
        B.step(sb, with_dec=False)


def run_h():
    for _ in range(K):
        B.step(sb)


for fn in (run_a, run_b, run_h):   # warm-up
    fn()
for rnd in range(2):
    res = {}
    for name, fn in (("A_decode_only", run_a), ("B_prefill_only", run_b), ("hybrid_fused", run_h)):
        res[name] = timed(fn)
    for ga in [int(x) for x in a.a_gemm_sms.split(",")]:
        for gb in [int(x) for x in a.gemm_sms.split(",")]:
            A.eng.qos_engine_set_option("gemm_sms", ga)
            B.eng.qos_engine_set_option("gemm_sms", gb)
            res[f"A||B gemm_sms A={ga} B={gb}"] = timed(run_ab)
    A.eng.qos_engine_set_option("gemm_sms", 0)
    B.eng.qos_engine_set_option("gemm_sms", 0)
    out = {k: {"ms_per_step": round(v[0], 3), "sm_mhz": v[1]} for k, v in res.items()}
    out["sum_A_B"] = round(res["A_decode_only"][0] + res["B_prefill_only"][0], 3)
    print(json.dumps({"round": rnd, "layers": a.layers, "chunk": a.chunk, "n_dec": a.n_dec, "ctx": a.ctx, **out}),
          flush=True)
A.eng.close()
B.eng.close()
