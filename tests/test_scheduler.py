"""QoServe host scheduler (NEXT-1) pins: Eq. 1-5 closed forms, the Alg. 1 comparator, dynamic
chunking against the latency model, relegation with hints, the Fig. 6 scenario, Table 2/3
fixtures, and a model-driven trace replay (CPU only)."""
import json
import math
import os

import numpy as np
import pytest

import synth
from paper_conf_asplos_goelmkar26_b200.replay import ModelExecutor, replay
from paper_conf_asplos_goelmkar26_b200.scheduler import (QOS_TIERS, DecodeHistory, QoServeScheduler, Request,
                                                         SchedulerConfig, violated)

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def lin_model(chunks, ctx):
    """A stand-in latency model: 5 ms + 10 us/token + 1 us per cached decode key / 1k."""
    T = sum(n for _, n in chunks) + len(ctx)
    return 5.0 + 0.01 * T + 1e-3 * sum(c + 1 for c in ctx) / 1000.0


def test_table3_tiers_match_paper():
    g = json.load(open(os.path.join(GOLD, "table3_qos.json")))
    for tier in ("Q1", "Q2", "Q3"):
        for k in ("interactive", "ttft", "tbt", "ttlt"):
            assert QOS_TIERS[tier][k] == g[tier][k]


def test_table2_lognormal_fits():
    g = json.load(open(os.path.join(GOLD, "table2_tokens.json")))["percentiles"]
    z90 = 1.2815515655446004
    for ds in ("azure_conv", "azure_code"):
        for part in ("prompt", "decode"):
            mu, sg = synth.LOGNORMAL[ds][part]
            assert abs(math.exp(mu) / g[ds][part]["p50"] - 1) < 0.01
            assert abs(math.exp(mu + z90 * sg) / g[ds][part]["p90"] - 1) < 0.01
    tr = synth.trace(5.0, 2000.0, "azure_conv")
    p = np.array([t["prompt_len"] for t in tr])
    assert abs(np.median(p) / 928 - 1) < 0.1                      # Table 2 p50
    tiers = np.array([t["tier"] for t in tr])
    for q in ("Q1", "Q2", "Q3"):
        assert abs((tiers == q).mean() - 1 / 3) < 0.05             # equal thirds
    gaps = np.diff([t["t_arrival"] for t in tr])
    assert abs(gaps.mean() - 0.2) < 0.02 and abs(gaps.std() / gaps.mean() - 1) < 0.1   # Poisson


def test_deadlines_eq1_to_eq3():
    a = Request(1, 10.0, 100, "Q1")
    assert a.d_first() == 16.0                                    # Eq. 1
    assert a.d_token(1) == 16.0 and abs(a.d_token(11) - 16.5) < 1e-12   # Eq. 2
    b = Request(2, 10.0, 100, "Q2")
    assert b.d_total() == 610.0                                   # Eq. 3


def test_hybrid_priority_eq4_eq5_and_comparator():
    s = QoServeScheduler(SchedulerConfig(alpha_ms_per_token=8.0), lin_model)
    a = Request(1, 0.0, 1000, "Q1")
    assert abs(s.priority(a) - (0 + 6 + 0.008 * 1000)) < 1e-12     # Eq. 4
    h = s.history
    for n in (10, 20, 30):
        h.observe("app", n)
    b = Request(2, 0.0, 500, "Q2", app_id="app", decoded=0)
    est = 20 + 2 * math.sqrt(np.var([10, 20, 30]))
    assert abs(h.estimate("app") - est) < 1e-9                    # mean + 2 sigma
    assert abs(s.priority(b) - (600 + 0.008 * (500 + est))) < 1e-9   # Eq. 5
    # comparator: relegated jobs last, then ascending priority
    c = Request(3, 100.0, 10, "Q1")
    b.relegated = True
    order = sorted([b, c, a], key=s.sort_key)
    assert [r.req_id for r in order] == [a.req_id, c.req_id, b.req_id]
    # alpha = 0 is EDF on the first deadline; large alpha favours short remaining work (SRPF-like)
    s0 = QoServeScheduler(SchedulerConfig(alpha_ms_per_token=0.0), lin_model)
    x, y = Request(4, 0.0, 8000, "Q1"), Request(5, 1.0, 10, "Q1")
    assert sorted([y, x], key=s0.sort_key)[0] is x
    s9 = QoServeScheduler(SchedulerConfig(alpha_ms_per_token=10.0), lin_model)
    assert sorted([x, y], key=s9.sort_key)[0] is y


def test_prefill_budget_follows_slack():
    s = QoServeScheduler(SchedulerConfig(max_chunk=4096, margin=0.0, chunk_step=64, min_chunk=64), lin_model)
    ctx = [1000] * 8
    assert s.prefill_budget(ctx, math.inf) == 4096                 # no decode constrains the step
    b1, b2 = s.prefill_budget(ctx, 0.010), s.prefill_budget(ctx, 0.030)
    assert 0 < b1 < b2
    assert lin_model([(0, b1)], ctx) <= 10.0 < lin_model([(0, b1 + 64)], ctx)
    assert s.prefill_budget(ctx, 0.001) == 0                       # decode-only step


def test_fig6_scenario_interactive_first_and_chunk_adapts():
    """PAPER.md:815-893 (Fig. 6): A (interactive) is served before D (non-interactive) despite
    arriving later; once A decodes, the chunk shrinks to keep its TBT; while A has slack, the
    chunk grows (B/D progress faster)."""
    s = QoServeScheduler(SchedulerConfig(max_chunk=2048, margin=0.0), lin_model)
    D = Request(1, 0.0, 3000, "Q2", decode_len=5)
    A = Request(2, 0.1, 600, "Q1", decode_len=50)
    s.submit(D)
    s.submit(A)
    chunks, decodes = s.create_batch(0.2)
    assert chunks[0][0] is A                                       # hybrid priority: A first
    now = 0.2
    sizes = []
    for _ in range(40):
        chunks, decodes = s.create_batch(now)
        if not chunks and not decodes:
            break
        sizes.append((sum(n for _, n in chunks), len(decodes)))
        now += lin_model([(0, sum(n for _, n in chunks))], [r.ctx_len for r in decodes]) * 1e-3
        s.complete(chunks, decodes, now)
    with_dec = [c for c, nd in sizes if nd > 0 and c > 0]
    without = [c for c, nd in sizes if nd == 0 and c > 0]
    assert with_dec and without and max(with_dec) < max(without)   # A's TBT bounds the chunk
    assert A.t_first is not None and not violated(A) or A.decoded < A.decode_len


def test_relegation_prefers_free_tier():
    s = QoServeScheduler(SchedulerConfig(max_chunk=256, margin=0.0), lambda c, x: 1000.0)  # 1 s steps
    late_free = Request(1, 0.0, 4000, "Q1", important=False)      # cannot make a 6 s TTFT
    late_paid = Request(2, 0.0, 4000, "Q1", important=True)
    s.submit(late_free)
    s.submit(late_paid)
    s.create_batch(0.5)
    assert late_free.relegated and not late_paid.relegated         # hint: free tier first
    s.create_batch(7.0)                                            # paid one has now missed TTFT
    assert late_paid.relegated


def test_model_replay_conserves_requests():
    tr = synth.trace(2.0, 30.0, "azure_code")
    s = QoServeScheduler(SchedulerConfig(max_chunk=2048), lin_model)
    out = replay(tr, s, ModelExecutor(lin_model))
    assert out["finished"] == out["requests"] == len(tr)
    assert 0 <= out["violations_pct"] <= 100
    assert out["tokens_per_s"] > 0 and len(out["chunk_series"]) > 0


def test_decode_history_default():
    h = DecodeHistory(default=77.0)
    assert h.estimate("new") == 77.0


def prefix_model(chunks, ctx):
    """Stand-in model whose chunk cost grows with the cached prefix (attention over it)."""
    T = sum(n for _, n in chunks) + len(ctx)
    return 5.0 + 0.01 * T + 1e-3 * sum(c + 1 for c in ctx) / 1000.0 + 2e-6 * sum(n * ks for ks, n in chunks)


def test_budget_prices_the_chunk_prefix():
    """Dynamic chunking prices the chunk at its request's cached prefix: later chunks of a
    long prompt get smaller budgets (attention grows for later chunks)."""
    s = QoServeScheduler(SchedulerConfig(max_chunk=4096, margin=0.0), prefix_model)
    ctx = [2000] * 16
    b0, b8k = s.prefill_budget(ctx, 0.030, 0), s.prefill_budget(ctx, 0.030, 8192)
    assert 0 < b8k < b0
    assert prefix_model([(8192, b8k)], ctx) <= 30.0 < prefix_model([(8192, b8k + 64)], ctx)


def test_medha_policy_shrinks_chunks_of_a_long_prefill():
    """NEXT-4 variant (Medha): one 10K-token prefill next to 500 decodes;
    with a fixed per-step target every step fits it and the chunk shrinks as the prefix grows."""
    cfg = SchedulerConfig(max_chunk=8192, margin=0.0, chunk_policy="medha", medha_target_ms=40.0, max_decodes=512,
                          max_rows=520)
    s = QoServeScheduler(cfg, prefix_model)
    decs = []
    for i in range(500):
        r = Request(1000 + i, 0.0, 1000, "Q2", decode_len=10 ** 6)
        r.prefill_done = r.prompt_len
        decs.append(r)
    s.decode_q.extend(decs)
    big = Request(1, 0.0, 10_000, "Q2", decode_len=500)
    s.submit(big)
    now, sizes = 0.0, []
    while big.prefill_rem > 0 and len(sizes) < 100:
        chunks, decodes = s.create_batch(now)
        c = sum(n for r, n in chunks if r is big)
        assert c > 0
        ms = prefix_model([(big.prefill_done, c)], [r.ctx_len for r in decodes])
        assert ms <= 40.0 + 1e-9
        sizes.append(c)
        now += ms * 1e-3
        s.complete(chunks, decodes, now)
    full = sizes[:-1]                      # the last chunk is the remainder
    assert len(full) >= 2 and all(a >= b for a, b in zip(full, full[1:])) and full[0] > full[-1]


def test_round_robin_replicas():
    """8 TP1 replicas with round-robin routing: every request is served
    once, and 8 replicas at 8x the load see no more violations than one replica at 1x."""
    from paper_conf_asplos_goelmkar26_b200.replay import replay_replicas
    tr8 = synth.trace(16.0, 20.0, "azure_conv")
    out8 = replay_replicas(tr8, 8, lambda: QoServeScheduler(SchedulerConfig(max_chunk=2048), lin_model),
                           lambda: ModelExecutor(lin_model))
    assert out8["requests"] == out8["finished"] == len(tr8) and out8["replicas"] == 8
    tr1 = synth.trace(2.0, 20.0, "azure_conv")
    out1 = replay(tr1, QoServeScheduler(SchedulerConfig(max_chunk=2048), lin_model), ModelExecutor(lin_model))
    assert out8["violations_pct"] <= out1["violations_pct"] + 1.0


def test_batches_respect_engine_capacity():
    """Every batch fits the engine (chunks + decodes <= max_rows), and no new prompt is started
    while the decode set is full (it would finish into a decode the engine cannot take)."""
    cfg = SchedulerConfig(max_chunk=4096, max_decodes=8, max_rows=10)
    s = QoServeScheduler(cfg, lambda chunks, ctx: 5.0 + 0.002 * sum(n for _, n in chunks) + 0.01 * len(ctx))
    for i in range(8):
        r = Request(100 + i, 0.0, 64, "Q2", decode_len=10 ** 6)
        r.prefill_done = r.prompt_len
        s.decode_q.append(r)
    fresh = [Request(i, 0.0, 32, "Q1", decode_len=4) for i in range(6)]
    for r in fresh:
        s.submit(r)
    chunks, decodes = s.create_batch(0.0)
    assert len(chunks) + len(decodes) <= cfg.max_rows
    assert not chunks                       # decode set full: no prompt is admitted
    s.decode_q = s.decode_q[:4]             # four decodes leave
    chunks, decodes = s.create_batch(0.0)
    assert chunks and len(chunks) + len(decodes) <= cfg.max_rows


def test_decode_set_never_exceeds_max_decodes():
    """Prompts that finish in the same batch count toward the decode limit: with 3 decodes
    running and max_decodes = 4, three short prompts must not all finish into the decode set
    (which would leave some decodes unscheduled while their TBT deadlines pass)."""
    cfg = SchedulerConfig(max_chunk=4096, max_decodes=4, max_rows=16, margin=0.0)
    s = QoServeScheduler(cfg, lambda chunks, ctx: 5.0 + 0.002 * sum(n for _, n in chunks) + 0.01 * len(ctx))
    for i in range(3):
        r = Request(100 + i, 0.0, 64, "Q1", decode_len=6)
        r.prefill_done = r.prompt_len
        r.decoded = 1
        s.decode_q.append(r)
    for i in range(3):
        s.submit(Request(i, 0.0, 32, "Q1", decode_len=3))
    now = 0.0
    for _ in range(60):
        chunks, decodes = s.create_batch(now)
        if not chunks and not decodes:
            break
        assert len(decodes) == len(s.decode_q) <= cfg.max_decodes       # every decode runs every step
        fin = sum(1 for r, n in chunks if n == r.prefill_rem)
        assert len(s.decode_q) + fin <= cfg.max_decodes
        now += 0.01
        s.complete(chunks, decodes, now)
        assert len(s.decode_q) <= cfg.max_decodes
    assert not s.decode_q and not s.prefill_q                            # everything finished


def test_partial_prefill_waits_one_token_short_of_a_full_decode_set():
    """A started prefill whose last chunk would finish into a full decode set is cut one token
    short; it completes once a decode slot frees."""
    cfg = SchedulerConfig(max_chunk=4096, max_decodes=2, max_rows=16, margin=0.0)
    s = QoServeScheduler(cfg, lambda chunks, ctx: 5.0)
    for i in range(2):
        r = Request(100 + i, 0.0, 64, "Q2", decode_len=3)
        r.prefill_done, r.decoded = r.prompt_len, 1
        s.decode_q.append(r)
    p = Request(1, 0.0, 100, "Q2", decode_len=2)
    p.prefill_done = 40
    s.submit(p)
    chunks, decodes = s.create_batch(0.0)
    assert chunks == [(p, 59)] and len(decodes) == 2
    s.complete(chunks, decodes, 0.01)
    chunks, decodes = s.create_batch(0.01)
    assert chunks == [] and len(decodes) == 2                           # still full: no finishing chunk
    s.complete(chunks, decodes, 0.02)                                   # both decodes finish (3 tokens)
    chunks, decodes = s.create_batch(0.02)
    assert chunks == [(p, 1)] and decodes == []


def test_preemption_stays_within_the_budget_and_token_capacity():
    """Selective preemption takes displaced in-flight prefills only from what is left of the
    budget C, and no batch exceeds the engine's token capacity (max_tokens)."""
    C = 256
    cfg = SchedulerConfig(max_chunk=C, min_chunk=64, chunk_step=64, max_decodes=64, max_rows=64, margin=0.0,
                          max_tokens=C + 8)
    # every step takes 1 s, so any started prompt with a 6 s TTFT is about to violate
    s = QoServeScheduler(cfg, lambda chunks, ctx: 1000.0)
    started = []
    for i in range(6):
        r = Request(i, 0.0, 4000, "Q1", decode_len=2)
        r.prefill_done = 100
        s.submit(r)
        started.append(r)
    for i in range(16):
        r = Request(100 + i, 0.0, 64, "Q2", decode_len=10 ** 6)
        r.prefill_done, r.decoded = r.prompt_len, 1
        s.decode_q.append(r)
    for t in (0.0, 1.0, 2.0, 3.0):
        chunks, decodes = s.create_batch(t)
        tok = sum(n for _, n in chunks)
        assert tok <= C and tok + len(decodes) <= cfg.max_tokens
    # the token capacity also caps an unconstrained budget
    s2 = QoServeScheduler(SchedulerConfig(max_chunk=4096, max_tokens=1000, max_decodes=64, max_rows=64),
                          lambda chunks, ctx: 1.0)
    for i in range(8):
        r = Request(100 + i, 0.0, 64, "Q2", decode_len=10 ** 6)
        r.prefill_done, r.decoded = r.prompt_len, 1
        s2.decode_q.append(r)
    s2.submit(Request(1, 0.0, 5000, "Q2"))
    chunks, decodes = s2.create_batch(0.0)
    assert sum(n for _, n in chunks) + len(decodes) == 1000


def test_fcfs_and_ablation_switches():
    """The ablation of the paper's Medha comparison ("only dynamic chunking under FCFS
    scheduling, disabling all other techniques"): fcfs serves prefills in
    arrival order where the hybrid priority (Eq. 4-5) would not; relegation off never relegates."""
    # a non-interactive request that arrived first vs an interactive one with an earlier
    # Eq. 4 priority: hybrid priority picks the interactive one, fcfs the earlier arrival
    early = Request(1, 0.0, 4000, "Q3", decode_len=10)
    late = Request(2, 1.0, 100, "Q1", decode_len=10)
    for fcfs, first in ((False, 2), (True, 1)):
        s = QoServeScheduler(SchedulerConfig(max_chunk=64, fcfs=fcfs), lin_model)
        s.submit(early)
        s.submit(late)
        chunks, _ = s.create_batch(2.0)
        assert chunks[0][0].req_id == first
    # an interactive prompt that cannot meet its TTFT: relegated with relegation on, not off
    for relegation in (True, False):
        s = QoServeScheduler(SchedulerConfig(max_chunk=64, relegation=relegation), lin_model)
        r = Request(3, 0.0, 100_000, "Q1", decode_len=10, important=False)
        s.submit(r)
        s.create_batch(5.9)
        assert r.relegated == relegation


def test_fixed_length_trace():
    tr = synth.trace(2.0, 30.0, "long_10k")
    assert len(tr) > 20 and all(t["prompt_len"] == 10_000 and t["decode_len"] == 500 for t in tr)
    assert {t["tier"] for t in tr} == {"Q1", "Q2", "Q3"}
