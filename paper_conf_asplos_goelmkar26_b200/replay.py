"""Trace replay (configs[4]): synthetic arrivals -> QoServe scheduler -> hybrid steps.

The virtual clock advances by each executed step's latency: the device-timed latency of the
real `qos_hybrid_step` (EngineExecutor) or the latency model's prediction (ModelExecutor).
Requests hold paged KV only while needed: blocks grow with each chunk /
decode and are freed when the request finishes.  Metrics follow PAPER.md:345-379 (TTFT, TBT,
TTLT), 1152-1155 (goodput: max load with <= 1% violations) and 1369-1371 (per-tier).
"""
from __future__ import annotations

import time

import numpy as np

from .scheduler import QoServeScheduler, Request, violated


class ModelExecutor:
    """Step latency from the fitted latency model (fast what-if simulation)."""

    def __init__(self, predict_ms):
        self.predict_ms = predict_ms

    def execute(self, chunks, decodes) -> float:
        return self.predict_ms([(r.prefill_done, n) for r, n in chunks], [r.ctx_len for r in decodes])

    def admit(self, chunks, decodes):
        return chunks

    def release(self, r: Request) -> None:
        pass


class EngineExecutor:
    """Runs every step on the GPU through the C ABI; greedy next tokens are fed back."""

    def __init__(self, engine, vocab: int, token_fn, stream=None):
        import torch
        from . import qoserve as q
        self.q = q
        self.eng = engine
        self.vocab = vocab
        self.token_fn = token_fn           # (req_id, positions slice) -> prompt token ids
        self.next_tok: dict[int, int] = {}
        self.stream = stream if stream is not None else torch.cuda.current_stream()
        self.out = torch.empty(4096, dtype=torch.int32, device="cuda")
        self.ev = (torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True))
        self.known: set[int] = set()

    def admit(self, chunks, decodes):
        """Grow KV for the step; chunks that do not fit wait (decodes are never dropped)."""
        ok = []
        for r, n in chunks:
            try:
                self.eng.qos_kv_alloc(r.req_id, r.prefill_done + n)
                self.known.add(r.req_id)
                ok.append((r, n))
            except self.q.QosError as e:
                if e.name != "OOM":
                    raise
        for r in decodes:
            self.eng.qos_kv_alloc(r.req_id, r.ctx_len + 1)
        return ok

    def execute(self, chunks, decodes) -> float:
        pre = [(r.req_id, r.prefill_done, self.token_fn(r.req_id, r.prefill_done, n)) for r, n in chunks]
        dec = [(r.req_id, r.ctx_len, self.next_tok.get(r.req_id, 0)) for r in decodes]
        b = self.q.make_batch(pre, dec)
        s = self.stream
        e0, e1 = self.ev
        e0.record(s)
        self.eng.qos_hybrid_step(b, None, self.q.QOS_F32, self.out.data_ptr(), False, s.cuda_stream)
        e1.record(s)
        e1.synchronize()
        toks = self.out[: len(pre) + len(dec)].cpu().numpy()
        for (r, _), t in zip(chunks, toks[: len(pre)]):
            self.next_tok[r.req_id] = int(t)
        for r, t in zip(decodes, toks[len(pre):]):
            self.next_tok[r.req_id] = int(t)
        return e0.elapsed_time(e1)

    def release(self, r: Request) -> None:
        if r.req_id in self.known:
            self.eng.qos_kv_free(r.req_id)
            self.known.discard(r.req_id)
        self.next_tok.pop(r.req_id, None)


def replay(trace, scheduler: QoServeScheduler, executor, max_steps: int = 10**9, log_chunks: bool = True):
    return summarize(*_run(trace, scheduler, executor, max_steps, log_chunks))


def replay_replicas(trace, n_replicas: int, make_scheduler, make_executor, max_steps: int = 10**9):
    """Round-robin load balancing over independent replicas (one TP1
    replica per GPU): request i goes to replica i mod n in arrival order; replicas share
    nothing, so each replays its share of the trace on its own clock.  Metrics are computed
    over all requests of all replicas."""
    order = sorted(range(len(trace)), key=lambda i: trace[i]["t_arrival"])
    reqs, done, t_end, steps, chunk_log, wall = [], [], 0.0, 0, [], 0.0
    for k in range(n_replicas):
        part = [trace[i] for i in order[k::n_replicas]]
        r, d, t, st, cl, w = _run(part, make_scheduler(), make_executor(), max_steps, True)
        reqs += r
        done += d
        t_end = max(t_end, t)
        steps += st
        chunk_log += cl
        wall += w
    out = summarize(reqs, done, t_end, steps, chunk_log, wall)
    out["replicas"] = n_replicas
    return out


def _run(trace, scheduler: QoServeScheduler, executor, max_steps: int, log_chunks: bool):
    reqs = [Request(**t) for t in trace]
    pending = sorted(reqs, key=lambda r: r.t_arrival)
    now, k, steps = 0.0, 0, 0
    done: list[Request] = []
    chunk_log = []
    wall0 = time.time()
    while (k < len(pending) or scheduler.prefill_q or scheduler.decode_q) and steps < max_steps:
        while k < len(pending) and pending[k].t_arrival <= now:
            scheduler.submit(pending[k])
            k += 1
        chunks, decodes = scheduler.create_batch(now)
        chunks = executor.admit(chunks, decodes)
        if not chunks and not decodes:
            if k < len(pending):
                now = max(now, pending[k].t_arrival)
                continue
            break
        ms = executor.execute(chunks, decodes)
        now += ms * 1e-3
        steps += 1
        if log_chunks:
            chunk_log.append((now, sum(n for _, n in chunks), len(decodes), ms))
        for r in scheduler.complete(chunks, decodes, now):
            executor.release(r)
            done.append(r)
    return reqs, done, now, steps, chunk_log, time.time() - wall0


def summarize(reqs, done, t_end, steps, chunk_log, wall_s):
    out = {"requests": len(reqs), "finished": len(done), "virtual_s": t_end, "steps": steps, "wall_s": wall_s}
    fin = [r for r in reqs if r.t_last is not None]
    viol = [violated(r) for r in reqs]
    out["violations_pct"] = 100.0 * float(np.mean(viol)) if reqs else 0.0
    for tier in ("Q1", "Q2", "Q3"):
        tr = [r for r in reqs if r.tier == tier]
        if not tr:
            continue
        d = {"n": len(tr), "violations_pct": 100.0 * float(np.mean([violated(r) for r in tr]))}
        ttft = [r.t_first - r.t_arrival for r in tr if r.t_first is not None]
        ttlt = [r.t_last - r.t_arrival for r in tr if r.t_last is not None]
        if ttft:
            d["ttft_p50"], d["ttft_p99"] = float(np.percentile(ttft, 50)), float(np.percentile(ttft, 99))
        if ttlt:
            d["ttlt_p50"], d["ttlt_p99"] = float(np.percentile(ttlt, 50)), float(np.percentile(ttlt, 99))
        out[tier] = d
    out["relegated_pct"] = 100.0 * float(np.mean([r.relegated for r in reqs])) if reqs else 0.0
    if chunk_log:
        cl = np.array(chunk_log)
        out["chunk_mean"] = float(cl[:, 1].mean())
        out["step_ms_mean"] = float(cl[:, 3].mean())
        out["tokens_per_s"] = float((cl[:, 1].sum() + cl[:, 2].sum()) / max(1e-9, cl[:, 3].sum() * 1e-3))
        out["chunk_series"] = [int(x) for x in cl[:1000, 1]]   # Fig. 9 / Fig. 15a analogue (1000 batches)
    del fin
    return out
