"""Hybrid-step benchmark (BASELINE.json metric: hybrid-step tokens/s & iteration latency vs chunk
size; %HBM / %tensor peak) on Llama-3-8B shapes (configs[1]).

A step = one qos_hybrid_step: a 2048-token prefill chunk of a fresh request (kv_start 0) fused
with 128 ongoing decodes at context ~4096 whose KV prefixes are resident in the paged cache
(synthetic KV) — one point of the configs[1] latency table (chunk 256-8192 x
0-256 decodes x ctx 1k-8k).  tokens/s = T / step latency with T = chunk + n_decode.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...   (N replicas, one per GPU; weak scaling)
    torchrun --nproc-per-node N bench.py --gpus N --tp N --model qwen2.5-14b   (configs[2]/[3]:
        one tensor-parallel model over the N ranks, cross-process peer group; strong scaling)

Rank 0 prints ONE JSON line.  `--impl reference` times the fp64 CPU oracle (the only other
place this file runs oracle/ code besides the cpu_baseline leg).
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

CHUNK, N_DEC, CTX = 2048, 128, 4096
WORKLOAD = f"llama3-8b hybrid step: chunk {CHUNK} @kv_start 0 + {N_DEC} decodes @ctx {CTX}"
# --workload: the headline hybrid step (configs[1]'s point above), or the prefill-node step of a
# PD-disaggregated deployment (one 8192-token chunk, no decodes: §4.1.3,
# SURVEY.md §8(f) NEXT-4)
WORKLOADS = {"hybrid": (CHUNK, N_DEC, CTX), "pd-prefill": (8192, 0, 0)}


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))
    except Exception:
        return {}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled every 200 ms during the timed region."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.index = index
        self.proc = None
        self.lines = []

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--id={self.index}", f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "200"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            threading.Thread(target=self._read, daemon=True).start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(2)
            except Exception:
                self.proc.kill()
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            f = [x.strip() for x in ln.split(",")]
            if len(f) < 7:
                continue
            try:
                sm.append(float(f[0]))
                mx = max(mx, float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


def _dist():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


# ------------------------------------------------------------------------------ our arm
class Workload:
    """The bench workload on one GPU: engine with Llama-3-8B shapes, 128 decode requests with
    synthetic ctx-4096 prefixes, and a fresh 2048-token chunk request per step.  Decodes advance
    one token per step (steady-state serving); each step's chunk request is freed after it."""

    def __init__(self, device: int, n_steps: int, chunk=CHUNK, n_dec=N_DEC, ctx=CTX, n_layers=None,
                 model="llama3-8b", tp=1, rank=0, group=None, max_tokens=None):
        import synth
        from paper_conf_asplos_goelmkar26_b200 import qoserve as q
        from paper_conf_asplos_goelmkar26_b200.presets import preset
        self.q = q
        self.chunk, self.n_dec = chunk, n_dec
        ctx_cap = ctx + n_steps + 2
        over = {} if n_layers is None else {"n_layers": n_layers}
        num_blocks = n_dec * ((ctx_cap + 15) // 16) + (n_steps + 4) * ((chunk + 15) // 16) + 64
        self.preset = preset(model, **over)
        self.cfg = q.model_cfg(**self.preset, num_blocks=num_blocks, max_seq_len=8192,
                               max_requests=n_dec + 64, max_batch_tokens=max(chunk + n_dec, max_tokens or 0),
                               max_batch_rows=n_dec + 1)
        self.eng = q.Engine(self.cfg, device=device, tp_rank=rank, tp_size=tp, group=group)
        self.eng.qos_engine_load_synthetic(synth.SEED_WEIGHTS)
        self.dec_reqs = list(range(1, n_dec + 1))
        for r in self.dec_reqs:
            self.eng.qos_kv_alloc(r, ctx_cap)
            self.eng.qos_kv_fill_synthetic(r, ctx, synth.SEED_KVFILL)
        self.ctx = {r: ctx for r in self.dec_reqs}
        self.tokens = synth.request_tokens(0, chunk, self.cfg.vocab)
        self._next_req = 10_000
        self.live = []
        self.tokens_per_step = chunk + n_dec

    def next_batch(self):
        cr = self._next_req
        self._next_req += 1
        self.eng.qos_kv_alloc(cr, self.chunk)
        self.live.append(cr)
        dec = [(r, self.ctx[r], (r * 7 + self.ctx[r]) % self.cfg.vocab) for r in self.dec_reqs]
        for r in self.dec_reqs:
            self.ctx[r] += 1
        return self.q.make_batch([(cr, 0, self.tokens)], dec)

    def retire(self):
        # the oldest enqueued step's chunk request leaves the engine; freeing right after the
        # (asynchronous) step is safe: later steps reusing its blocks are stream-ordered
        self.eng.qos_kv_free(self.live.pop(0))

    def step(self, batch, out_ptr, on_host, stream_ptr):
        self.eng.qos_hybrid_step(batch, None, self.q.QOS_F32, out_ptr, on_host, stream_ptr)
        self.retire()


def run_ours(args):
    import torch
    import torch.distributed as dist

    ws, rank, local = _dist()
    local = local % max(1, torch.cuda.device_count())
    torch.cuda.set_device(local)
    tp = args.tp
    shared_gpu = ws > torch.cuda.device_count()   # smoke runs of --tp on one GPU: NCCL refuses that
    if ws > 1:
        if shared_gpu:
            dist.init_process_group("gloo")
        else:
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    K, W = args.steps, args.warmup
    group = None
    if tp > 1:  # one model over the ranks: cross-process peer group (id from rank 0)
        from paper_conf_asplos_goelmkar26_b200 import qoserve as qq
        assert ws == tp, "--tp needs WORLD_SIZE == tp (one rank per GPU)"
        box = [qq.qos_group_unique_id() if rank == 0 else None]
        dist.broadcast_object_list(box, src=0)
        group = qq.Group(tp, box[0], rank)
    chunk, n_dec, ctx = WORKLOADS[args.workload]
    # the chunk-size sweep after the timed passes (the metric is tokens/s and latency vs chunk
    # size): the engine needs room for the largest chunk
    sweep_chunks = (256, 512, 1024, 2048, 4096, 8192) if (args.workload == "hybrid" and tp == 1 and
                                                          not args.no_sweep) else ()
    wl = Workload(local, W + 3 * K + 2, chunk=chunk, n_dec=n_dec, ctx=ctx, model=args.model, n_layers=args.layers,
                  tp=tp, rank=rank % tp, group=group)
    q, eng, T = wl.q, wl.eng, wl.tokens_per_step
    replicas = ws // tp
    stream = torch.cuda.current_stream()
    sptr = stream.cuda_stream
    out_tok = torch.empty(n_dec + 1, dtype=torch.int32, device="cuda")
    # -------- warm-up
    for _ in range(W):
        wl.step(wl.next_batch(), out_tok.data_ptr(), False, sptr)
    torch.cuda.synchronize()

    def timed_pass(instrument: bool):
        batches = [wl.next_batch() for _ in range(K)]
        eng.qos_engine_set_timing(instrument)
        if ws > 1:
            dist.barrier()
        torch.cuda.synchronize()
        evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in batches]
        ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        ev0.record(stream)
        for b, (e0, e1) in zip(batches, evs):
            e0.record(stream)
            wl.step(b, out_tok.data_ptr(), False, sptr)
            e1.record(stream)
        ev1.record(stream)
        torch.cuda.synchronize()
        if ws > 1:
            dist.barrier()
        per = eng.qos_last_step_timing() if instrument else None
        eng.qos_engine_set_timing(False)
        return ev0.elapsed_time(ev1) / K, [a.elapsed_time(b) for a, b in evs], per

    # -------- headline timed pass: device-resident outputs, no instrumentation
    clocks = ClockSampler(local)
    clocks.start()
    l0 = q.launch_count()
    ms_step, steps_ms, _ = timed_pass(False)
    launches = q.launch_count() - l0
    clk = clocks.stop()
    # -------- instrumented timed pass: CUDA events around every kernel class on the step stream;
    # a7 and a8 serialised so each kernel's own duration is attributed (overlap hides one in the other)
    eng.qos_engine_set_option("overlap_attn", 0)
    ms_instr, _, per_class = timed_pass(True)
    eng.qos_engine_set_option("overlap_attn", 1)
    # -------- e2e: a greedy serving loop through the public API.  Every step: the host builds the
    # descriptor (chunk tokens, decode positions) and the engine uploads it from pinned staging;
    # the decodes' tokens are the previous step's next tokens, read on the device
    # (qos_hybrid_step_ex), so step k+1 is built and enqueued while step k runs; every step's
    # next tokens are copied to pinned host memory and read on the host (one step behind).
    dec_rows = n_dec + 1
    dev_tok = [torch.empty(dec_rows, dtype=torch.int32, device="cuda") for _ in range(2)]
    pin_tok = [torch.empty(dec_rows, dtype=torch.int32, pin_memory=True) for _ in range(2)]
    done = [torch.cuda.Event() for _ in range(2)]
    first = torch.tensor([(r * 7 + wl.ctx[r]) % wl.cfg.vocab for r in wl.dec_reqs], dtype=torch.int32, device="cuda")
    torch.cuda.synchronize()
    read = 0
    t0 = time.perf_counter()
    src = first.data_ptr() if n_dec else None
    for k in range(K):
        i = k & 1
        b = wl.next_batch()
        if k >= 2:
            done[i].synchronize()  # step k-2's tokens were read below before it is overwritten
        eng.qos_hybrid_step_ex(b, None, wl.q.QOS_F32, dev_tok[i].data_ptr(), False, sptr, src)
        h2d, _ = eng.qos_last_step_io()
        wl.retire()
        pin_tok[i].copy_(dev_tok[i], non_blocking=True)
        done[i].record(stream)
        if k >= 1:
            done[i ^ 1].synchronize()
            read += int(pin_tok[i ^ 1][-1])  # the previous step's result, on the host
        # next step's decode tokens: rows 1.. (row 0 is the chunk); no decodes: nothing to feed
        src = dev_tok[i].data_ptr() + 4 if n_dec else None
    done[(K - 1) & 1].synchronize()
    read += int(pin_tok[(K - 1) & 1][-1])
    e2e_ms = (time.perf_counter() - t0) * 1e3 / K
    d2h = dec_rows * 4
    # the synchronous form (host outputs, the call returns after the step): host descriptor
    # building and the step's device time do not overlap
    batches = [wl.next_batch() for _ in range(K)]
    host_tok = np.empty(n_dec + 1, dtype=np.int32)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for b in batches:
        wl.step(b, host_tok.ctypes.data, True, sptr)
    e2e_sync_ms = (time.perf_counter() - t0) * 1e3 / K
    # -------- max over ranks
    if ws > 1:
        t = torch.tensor([ms_step, e2e_ms, ms_instr, e2e_sync_ms], device="cpu" if shared_gpu else "cuda")
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_step, e2e_ms, ms_instr, e2e_sync_ms = float(t[0]), float(t[1]), float(t[2]), float(t[3])
    peaks = _peaks()
    pr = wl.preset
    d, F, hd, Hkv = pr["d_model"], pr["ffn_dim"] // tp, pr["head_dim"], pr["n_kv_heads"] // tp
    L = pr["n_layers"]
    gu_ms, gu_n = per_class["gemm_gateup"]
    gu_flops = 2.0 * T * d * (2 * F)                    # algorithmic FLOPs per launch (one layer)
    gu_tfs = gu_flops / (gu_ms / gu_n * 1e-3) / 1e12
    peak_tc = peaks.get("bf16_tflops_sustained") or 1400.0
    da_ms, da_n = per_class.get("decode_attn", (0.0, 0))
    # decode attention: K+V bytes of every decode's (ctx+1) keys per layer;
    # the instrumented pass ran after warm-up + one timed pass, contexts grew 1 token per step
    mean_ctx = ctx + W + K + (K - 1) / 2.0
    da_bytes = 4.0 * hd * Hkv * n_dec * (mean_ctx + 1)
    da_gbs = da_bytes / (da_ms / da_n * 1e-3) / 1e9 if da_n else 0.0
    peak_hbm = peaks.get("hbm_gbs") or 6650.0
    # prefill attention (a7): causal FLOPs of the chunk per layer, chunk at kv_start 0
    pa_ms, pa_n = per_class.get("prefill_attn", (0.0, 0))
    H = pr["n_heads"] // tp
    pa_flops = 4.0 * hd * H * (chunk * (chunk + 1) / 2.0)
    pa_tfs = pa_flops / (pa_ms / pa_n * 1e-3) / 1e12 if pa_n else 0.0
    # step roofline: sum over the step's kernels of max(FLOPs / tensor peak,
    # bytes / HBM peak) against the measured step time
    Hq = pr["n_heads"] // tp
    V = pr["vocab"] // tp
    proj = [(d * (Hq + 2 * Hkv) * hd), (Hq * hd * d), (2 * d * F), (F * d)]   # weights per layer (elements)

    def step_terms(c, nd, cx, kv_bytes=None):
        Tt, R = c + nd, (1 if c else 0) + nd
        tg = sum(max(2.0 * Tt * w / (peak_tc * 1e12), 2.0 * w / (peak_hbm * 1e9)) for w in proj) * L
        th = max(2.0 * R * d * V / (peak_tc * 1e12), 2.0 * d * V / (peak_hbm * 1e9))
        kvb = kv_bytes if kv_bytes is not None else 4.0 * hd * Hkv * nd * (cx + 1)
        td = kvb * L / (peak_hbm * 1e9)
        tp_ = 4.0 * hd * Hq * (c * (c + 1) / 2.0) * L / (peak_tc * 1e12)
        return tg, th, td, tp_

    def step_roofline_ms(c, nd, cx):
        return sum(step_terms(c, nd, cx)) * 1e3

    t_gemm, t_head, t_dec, t_pre = step_terms(chunk, n_dec, ctx, kv_bytes=da_bytes)
    t_roof = (t_gemm + t_head + t_dec + t_pre) * 1e3
    # -------- chunk-size sweep (configs[1] row: chunk 256..8192 with the bench's 128 decodes @ctx
    # 4096): device-timed median of qos_profile_step on scratch requests (the bench's decode
    # requests are released first; their KV pool is reused)
    sweep = []
    if sweep_chunks:
        # a second engine with room for the largest chunk (the headline engine keeps exactly the
        # bench shape's workspace); the first one is released first
        eng.close()
        wl2 = Workload(local, 4, chunk=chunk, n_dec=n_dec, ctx=ctx, model=args.model, n_layers=args.layers,
                       max_tokens=max(sweep_chunks) + n_dec)
        for r in wl2.dec_reqs:
            wl2.eng.qos_kv_free(r)
        for c in sweep_chunks:
            ms_c, p95_c = wl2.eng.qos_profile_step(c, [ctx] * n_dec, reps=3, warmup=2)
            sweep.append({"chunk": c, "n_decode": n_dec, "ctx": ctx, "ms": round(ms_c, 3),
                          "tokens_per_s": round(replicas * (c + n_dec) / (ms_c * 1e-3), 1),
                          "roofline_frac": round(step_roofline_ms(c, n_dec, ctx) / ms_c, 4)})
        eng = wl2.eng
    roof_step = {"roofline_ms": round(t_roof, 3), "achieved_ms": round(ms_step, 3), "frac": round(t_roof / ms_step, 4),
                 "terms_ms": {"projections": round(t_gemm * 1e3, 3), "lm_head": round(t_head * 1e3, 3),
                              "decode_attn": round(t_dec * 1e3, 3), "prefill_attn": round(t_pre * 1e3, 3)},
                 "peaks": "bf16_tflops_sustained and hbm_gbs of MEASURED_PEAKS.json (of measured)"}
    traffic = None
    try:
        assert args.model == "llama3-8b" and tp == 1 and args.layers is None and args.workload == "hybrid"
        prof = json.load(open(os.path.join(ROOT, "profiles", "roofline_traffic.json")))
        traffic = prof.get("gemm_gateup", {}).get("dram_bytes_per_launch")
    except Exception:
        pass
    tag = args.model + (f" TP{tp}" if tp > 1 else "")
    rec = {
        "metric": (f"hybrid-step tokens/s ({tag}, chunk 2048 + 128 decodes @4k)" if args.workload == "hybrid" else
                   f"prefill-node step tokens/s ({tag}, chunk 8192, no decodes)"),
        "value": round(replicas * T / (ms_step * 1e-3), 1),
        "unit": "tokens/s",
        "n_gpus": ws, "steps": K, "warmup": W,
        "ms_per_step": round(ms_step, 4),
        "higher_is_better": True,
        "scaling": "weak" if tp == 1 else "strong",
        "vs_baseline": None,
        "dtype": "bf16",
        "data": "synthetic (seeded weights + synthetic KV prefixes; DESIGN.md §3)",
        "config": {"workload": (WORKLOAD.replace("llama3-8b", tag) if args.workload == "hybrid" else
                                f"{tag} PD-disaggregated prefill-node step: chunk {chunk} @kv_start 0, no decodes"),
                   "model": f"{args.model} ({L} layers, random-init)", "chunk_len": chunk,
                   "n_decode": n_dec, "ctx": ctx, "tokens_per_step": T,
                   "parallelism": f"replicas{ws}" if tp == 1 else f"tp{tp} (peer-memory collectives)",
                   "l2": ("inputs larger than L2 (16 GB weights + 69 GB KV streamed per step)" if tp == 1 and
                          args.model == "llama3-8b" and args.layers is None and n_dec else
                          "inputs larger than L2 (16 GB of weights streamed per step)" if not n_dec else
                          "inputs larger than L2 (weight shard + KV of 128 x 4k contexts streamed per step)")},
        "latency_ms": {"median": round(statistics.median(steps_ms), 4), "min": round(min(steps_ms), 4),
                       "max": round(max(steps_ms), 4), "instrumented_pass_serial_attention": round(ms_instr, 4)},
        "breakdown_ms_per_step": {k: round(v[0] / K, 4) for k, v in per_class.items() if v[1]},
        "roofline": {"kernel": "gemm_gateup (tcgen05, a11)", "bound": "tensor", "achieved": round(gu_tfs, 1),
                     "peak": peak_tc, "unit": "TFLOP/s", "frac": round(gu_tfs / peak_tc, 4),
                     "traffic": traffic,
                     "peak_source": "MEASURED_PEAKS.json bf16_tflops_sustained (of measured)"},
        "roofline_prefill_attn": {"bound": "tensor", "achieved": round(pa_tfs, 1), "peak": peak_tc, "unit": "TFLOP/s",
                                  "frac": round(pa_tfs / peak_tc, 4) if peak_tc else None,
                                  "note": f"{chunk}-token causal chunk from position 0"},
        "roofline_decode_attn": ({"bound": "hbm", "achieved": round(da_gbs, 1), "peak": peak_hbm, "unit": "GB/s",
                                  "frac": round(da_gbs / peak_hbm, 4),
                                  "peak_source": "MEASURED_PEAKS.json hbm_gbs (of measured)"} if n_dec else None),
        "roofline_step": roof_step,
        "chunk_sweep": sweep or None,
        "gpu_launches": int(launches),
        "clocks": clk,
        "e2e": {"value": round(replicas * T / (e2e_ms * 1e-3), 1), "unit": "tokens/s",
                "ms_per_step": round(e2e_ms, 4),
                "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
                "how": ("greedy serving loop, wall clock: host descriptor uploaded every step (pinned staging), "
                        "decode tokens fed from the previous step's device next_tokens (qos_hybrid_step_ex), "
                        "next_tokens copied to pinned host memory and read every step (one step behind)"),
                "sync_call": {"value": round(replicas * T / (e2e_sync_ms * 1e-3), 1), "ms_per_step": round(e2e_sync_ms, 4),
                              "how": "qos_hybrid_step with host descriptor and host next_tokens (outputs_on_host=1)"}},
    }
    if (rank == 0 and not args.no_cpu_baseline and tp == 1 and args.model == "llama3-8b" and args.layers is None
            and args.workload == "hybrid"):
        rec["cpu_baseline"] = cpu_baseline()
    eng.close()
    if group is not None:
        group.close()
    if ws > 1:
        dist.destroy_process_group()
    if rank == 0:
        print(json.dumps(rec), flush=True)


# ------------------------------------------------------------------------------ oracle (CPU)
def _oracle_setup():
    """The fp64 oracle on a bounded sample of the bench workload: ONE of the 32 layers
    (embedding + 1 layer + LM head) for the 2048-token chunk and 8 of the 128 decodes
    (synthetic ctx-4096 prefixes).  Weight / KV generation happens here, outside any timed
    region."""
    import synth
    from oracle.engine import OracleEngine
    from oracle.model import PRESETS, with_layers
    c = with_layers(PRESETS["llama3-8b"], 1)
    orc = OracleEngine(c, seed=synth.SEED_WEIGHTS, num_blocks=N_DEC * 260 + 200)
    b = synth.hybrid_batch(c.vocab, CHUNK, 8, CTX)
    orc.W.layer(0)
    orc.W.head()
    orc.W.final_norm()
    orc.kv_alloc(0, CHUNK)
    for d in b.decode:
        orc.kv_alloc(d.req, CTX + 1)
        orc.kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
    pre, dec = b.as_oracle()
    return orc, pre, dec


def _oracle_sample(state=None):
    """Time one sample step of the oracle (see _oracle_setup), extrapolated to the full step as
    t_step = 32 * (t_chunk + 16 * t_8dec)  (the head is counted 32x: pessimistic).  Re-running
    the sample rewinds the KV first (chunk positions 0..2047, decode position 4096 rewritten)."""
    orc, pre, dec = state if state is not None else _oracle_setup()
    # rewind the KV of a previous sample (untimed): the chunk starts again at position 0 and
    # each decode appends at position CTX
    orc.kv.pop(0, None)
    for r, layers in orc.kv.items():
        orc.kv[r] = [(k[:CTX], v[:CTX]) for k, v in layers]
    t0 = time.perf_counter()
    orc.hybrid_step(pre, [])
    t_chunk = time.perf_counter() - t0
    t0 = time.perf_counter()
    orc.hybrid_step([], dec)
    t_dec = time.perf_counter() - t0
    t_step = 32 * (t_chunk + (N_DEC / 8) * t_dec)
    return t_step, t_chunk + t_dec


def _cores():
    try:
        from threadpoolctl import threadpool_info
        th = [i.get("num_threads", 0) for i in threadpool_info() if i.get("user_api") == "blas"]
        if th:
            return int(max(th))
    except Exception:
        pass
    return os.cpu_count()


def cpu_baseline():
    t_step, t_meas = _oracle_sample()
    T = CHUNK + N_DEC
    return {"value": round(T / t_step, 3), "unit": "tokens/s", "cores": _cores(), "kind": "oracle",
            "sample": f"fp64 numpy oracle, 1 of 32 layers for the {CHUNK}-token chunk + 8 of {N_DEC} decodes "
                      f"(ctx {CTX}), measured {t_meas:.1f} s, extrapolated x32 layers and x16 decodes",
            "seconds_per_step_extrapolated": round(t_step, 2)}


def run_reference(args):
    ws, rank, local = _dist()
    if rank != 0:
        return
    if ws > 1:
        # torchrun sets OMP_NUM_THREADS=1 for multi-process jobs; the oracle's rank runs alone, so
        # give its BLAS the host's cores as in the single-process run
        try:
            from threadpoolctl import threadpool_limits
            threadpool_limits(limits=os.cpu_count(), user_api="blas")
        except Exception:
            pass
    for _ in range(args.warmup if args.warmup < 1 else 1):
        pass   # the oracle has no warm-up state; one untimed generation pass happens inside
    t_start = time.perf_counter()
    state = _oracle_setup()  # weights + KV prefixes generated once, untimed
    vals = []
    for _ in range(max(1, args.steps)):
        t_step, _ = _oracle_sample(state)
        vals.append(t_step)
        if time.perf_counter() - t_start > 120:   # keep the whole run within a few minutes
            break
    t_step = statistics.median(vals)
    T = CHUNK + N_DEC
    value = T / t_step
    rec = {"impl": "reference", "metric": "hybrid-step tokens/s (llama3-8b, chunk 2048 + 128 decodes @4k)",
           "value": round(value, 3), "unit": "tokens/s", "n_gpus": ws, "steps": len(vals), "warmup": args.warmup,
           "ms_per_step": round(t_step * 1e3, 1), "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f64", "data": "synthetic",
           "config": {"workload": WORKLOAD, "model": "llama3-8b (oracle, fp64)", "chunk_len": CHUNK,
                      "n_decode": N_DEC, "ctx": CTX, "parallelism": "cpu"},
           "cpu_baseline": {"value": round(value, 3), "unit": "tokens/s", "cores": _cores(), "kind": "oracle",
                            "sample": "each step: 1 of 32 layers, chunk + 8 of 128 decodes, extrapolated"},
           "e2e": {"value": round(value, 3), "unit": "tokens/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(rec), flush=True)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-sweep", action="store_true", help="skip the chunk-size sweep after the timed passes")
    ap.add_argument("--cpu-seconds", type=float, default=20.0)
    ap.add_argument("--tp", type=int, default=1, help="tensor-parallel degree (= WORLD_SIZE under torchrun)")
    ap.add_argument("--model", default="llama3-8b", help="llama3-8b | qwen2.5-14b | llama3-70b")
    ap.add_argument("--layers", type=int, default=None, help="fewer layers (smoke runs only)")
    ap.add_argument("--workload", default="hybrid", choices=sorted(WORKLOADS),
                    help="hybrid: the headline step; pd-prefill: the 8192-token prefill-node step (NEXT-4)")
    args = ap.parse_args()
    if args.warmup < 3 and args.impl == "ours":
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
