"""Tensor parallelism on the GPU (vLLM TP, §3.6): the sharded
engine — q/kv heads, FFN columns and vocab rows split over ranks, per-rank KV pools, the O/down
partials summed after each projection, the vocab slices gathered — against the UNSHARDED fp64
oracle, through the C ABI.

This run has one GPU, so the ranks are an in-process peer group (qos_group_create /
qos_engine_create_peer) of engines on cuda:0, one host thread per rank: the collectives are
the library's peer-memory kernels (fused reduce + residual add + RMSNorm, logits gather), the
same code that serves ranks on peer GPUs.  Every rank must return bit-identical logits (the
peer reduction sums in rank order on every rank).
"""
import os

import numpy as np
import pytest

import synth
from helpers import TOL_LOGITS, row_rel_err

pytestmark = pytest.mark.gpu


def _group_engines(preset_name, tp, **caps_over):
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    from paper_conf_asplos_goelmkar26_b200.presets import preset
    caps = dict(num_blocks=256, max_seq_len=4096, max_requests=64, max_batch_tokens=1024, max_batch_rows=32)
    model_over = {k: v for k, v in caps_over.items() if k not in caps}
    caps.update({k: v for k, v in caps_over.items() if k in caps})
    cfg = q.model_cfg(**preset(preset_name, **model_over), **caps)
    g = q.Group(tp)
    engs = [q.Engine(cfg, 0, r, tp, group=g) for r in range(tp)]
    return q, cfg, g, engs


def _close(g, engs):
    for e in engs:
        e.close()
    g.close()


def _oracle(preset, ffn_dim=None, **kw):
    import dataclasses

    from oracle.engine import OracleEngine
    from oracle.model import PRESETS, with_layers
    c = PRESETS[preset]
    if "n_layers" in kw:
        c = with_layers(c, kw.pop("n_layers"))
    if ffn_dim:
        c = dataclasses.replace(c, ffn_dim=ffn_dim)
    return OracleEngine(c, seed=0, **kw)


def _all(q, engs, fn):
    return q.run_ranks(fn, engs)


@pytest.mark.parametrize("preset,tp,ffn,twoshot,swab", [("tiny", 2, None, -1, 1), ("tiny", 2, None, 1, 1),
                                                         ("tiny", 2, None, 1, 0), ("tiny-qwen", 2, None, -1, 1),
                                                         ("tiny-mha", 2, None, -1, 1), ("tiny-mha", 4, 1024, -1, 1),
                                                         ("tiny-mha", 4, 1024, 0, 1), ("tiny-mha", 4, 1024, -1, 0)])
def test_tp_peer_group_tiny_scenario(preset, tp, ffn, twoshot, swab):
    # (tp 4 needs F/tp % 128 == 0: F = 1024 instead of 768); twoshot: one-shot / two-shot
    # reduction; swab = 0 puts the O / down projections on the one-pass tile kernels, whose
    # epilogue then stores each partial row straight into its owner's receive slot (tp_scatter)
    q, cfg, g, engs = _group_engines(preset, tp, **({"ffn_dim": ffn} if ffn else {}))
    for e in engs:
        e.qos_engine_set_option("tp_twoshot", twoshot)
        e.qos_engine_set_option("gemm_swab", swab)
    _all(q, engs, lambda r, e: e.qos_engine_load_synthetic(0))
    orc = _oracle(preset, ffn_dim=ffn, num_blocks=256)
    ctxs, warm, main, second = synth.tiny_scenario(cfg.vocab)
    for r, n in ctxs.items():
        _all(q, engs, lambda k, e: e.qos_kv_alloc(r, n + 2))
        orc.kv_alloc(r, n + 2)
    _all(q, engs, lambda k, e: e.qos_kv_alloc(0, 256))
    orc.kv_alloc(0, 256)
    for b in warm + [main, second]:
        kb = q.batch_from_synth(b)
        outs = _all(q, engs, lambda k, e: e.step_host(kb, cfg.vocab))
        ref = orc.hybrid_step(*b.as_oracle())
        for lg, tk in outs[1:]:  # every rank holds the same full logits
            assert np.array_equal(lg, outs[0][0]) and np.array_equal(tk, outs[0][1])
        lg, tk = outs[0]
        assert row_rel_err(lg, ref) <= TOL_LOGITS
        srt = np.sort(ref, 1)
        gap = (srt[:, -1] - srt[:, -2]) / np.abs(ref).max(1)
        rt = np.argmax(ref, 1)
        assert all(tk[i] == rt[i] or gap[i] <= 2 * TOL_LOGITS for i in range(len(rt)))
    for r in list(ctxs) + [0]:  # block tables identical on every rank and bit-exact vs the oracle
        for e in engs:
            assert e.qos_kv_table(r) == orc.kv_table(r)
            assert e.qos_kv_table_device(r) == orc.kv_table(r)
    _close(g, engs)


def test_tp_peer_group_matches_tp1_engine():
    """TP=2 and TP=1 runs of the same steps agree within the logits tolerance (different
    reduction order, same bf16 rounding points)."""
    from helpers import make_engine
    q, cfg, g, engs = _group_engines("tiny", 2)
    _, _, one = make_engine("tiny", num_blocks=256)
    one.qos_engine_load_synthetic(0)
    _all(q, engs, lambda r, e: e.qos_engine_load_synthetic(0))
    toks = synth.request_tokens(3, 200, cfg.vocab)
    one.qos_kv_alloc(3, 260)
    _all(q, engs, lambda r, e: e.qos_kv_alloc(3, 260))
    steps = [q.make_batch([(3, 0, toks[:120])], []), q.make_batch([(3, 120, toks[120:])], [])]
    steps += [q.make_batch([], [(3, 200 + i, int(toks[i]))]) for i in range(5)]
    for b in steps:
        l1, _ = one.step_host(b, cfg.vocab)
        l2 = _all(q, engs, lambda r, e: e.step_host(b, cfg.vocab))[0][0]
        assert row_rel_err(l2, l1) <= TOL_LOGITS
    one.close()
    _close(g, engs)


def test_tp_peer_group_profile_step_and_missing_rank_aborts():
    """qos_profile_step runs its steps through the collectives on every rank; a rank that never
    reaches a collective makes the others fail with QOS_ERR_COMM after the group timeout."""
    os.environ["QOS_GROUP_TIMEOUT_MS"] = "3000"
    try:
        q, cfg, g, engs = _group_engines("tiny", 2)
    finally:
        del os.environ["QOS_GROUP_TIMEOUT_MS"]
    _all(q, engs, lambda r, e: e.qos_engine_load_synthetic(0))
    ms = _all(q, engs, lambda r, e: e.qos_profile_step(64, [100, 300], reps=3))
    assert all(m[0] > 0 for m in ms)
    engs[0].qos_kv_alloc(5, 32)
    engs[1].qos_kv_alloc(5, 32)
    with pytest.raises(q.QosError) as ei:  # rank 1 never steps
        engs[0].step_host(q.make_batch([(5, 0, np.ones(8, np.int32))], []), cfg.vocab)
    assert ei.value.name == "COMM"
    with pytest.raises(q.QosError) as ei:  # the group stays aborted
        engs[1].step_host(q.make_batch([(5, 0, np.ones(8, np.int32))], []), cfg.vocab)
    assert ei.value.name == "COMM"
    with pytest.raises(q.QosError):  # engines first
        g.close()
    _close(g, engs)


@pytest.mark.slow
@pytest.mark.parametrize("tp", [2, 4])
def test_qwen14b_shapes_tp2_hybrid_step_sampled_parity(tp):
    """configs[2] launch shape: Qwen-2.5-14B (2 layers, full width: d 5120, 40 q / 8 kv heads,
    QKV bias, F 13824, V 152064) at TP2 and TP4 — a 2048-token chunk + 128 decodes @ ctx 4096
    with synthetic KV prefixes — sampled logits rows vs the unsharded oracle, ranks identical."""
    C, ND, CTX = 2048, 128, 4096
    q, cfg, g, engs = _group_engines("qwen2.5-14b", tp, n_layers=2,
                                     num_blocks=(C + ND * (CTX + 1)) // 16 + 200, max_seq_len=8192,
                                     max_batch_tokens=C + ND, max_batch_rows=ND + 1, max_requests=ND + 8)
    _all(q, engs, lambda r, e: e.qos_engine_load_synthetic(0))
    b = synth.hybrid_batch(cfg.vocab, C, ND, CTX)

    def prep(r, e):
        e.qos_kv_alloc(0, C)
        for d in b.decode:
            e.qos_kv_alloc(d.req, CTX + 1)
            e.qos_kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
    _all(q, engs, prep)
    kb = q.batch_from_synth(b)
    outs = _all(q, engs, lambda r, e: e.step_host(kb, cfg.vocab))
    assert all(np.array_equal(outs[0][0], o[0]) for o in outs[1:])
    lg = outs[0][0]
    orc = _oracle("qwen2.5-14b", n_layers=2, num_blocks=2 * (C // 16 + 1) + 8 * (CTX // 16 + 2))
    sample = [0, 77, 127]
    orc.kv_alloc(0, C)
    decs = []
    for j in sample:
        d = b.decode[j]
        orc.kv_alloc(d.req, CTX + 1)
        orc.kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
        decs.append((d.req, d.ctx_len, d.token))
    ref = orc.hybrid_step([(0, 0, [int(t) for t in b.prefill[0].tokens])], decs)
    got = np.concatenate([lg[:1], lg[[1 + j for j in sample]]])
    assert row_rel_err(got, ref) <= TOL_LOGITS
    _close(g, engs)


@pytest.mark.slow
def test_llama70b_shapes_tp8_hybrid_step_sampled_parity():
    """configs[3] launch shape at TP8: Llama-3-70B (2 layers, full width: d 8192, 64 q / 8 kv
    heads -> one kv head per rank, F 28672, V 128256) — a 512-token chunk at kv_start 1024 +
    32 decodes with log-uniform contexts on [1k, 32k] (synthetic KV prefixes) — sampled logits
    rows vs the unsharded oracle; all 8 ranks bit-identical."""
    C, KS, ND = 512, 1024, 32
    rng = np.random.default_rng(synth.SEED_CTX)
    ctx = [int(x) for x in np.exp(rng.uniform(np.log(1024), np.log(32768), ND)).astype(np.int64)]
    ctx[0] = 32767
    tot = C + KS + sum(c + 1 for c in ctx)
    q, cfg, g, engs = _group_engines("llama3-70b", 8, n_layers=2, num_blocks=tot // 16 + ND + 64,
                                     max_seq_len=32784, max_batch_tokens=C + ND, max_batch_rows=ND + 1,
                                     max_requests=ND + 8)
    _all(q, engs, lambda r, e: e.qos_engine_load_synthetic(0))
    b = synth.hybrid_batch(cfg.vocab, C, ND, ctx, kv_start=KS)

    def prep(r, e):
        e.qos_kv_alloc(0, KS + C)
        e.qos_kv_fill_synthetic(0, KS, synth.SEED_KVFILL)
        for d in b.decode:
            e.qos_kv_alloc(d.req, d.ctx_len + 1)
            e.qos_kv_fill_synthetic(d.req, d.ctx_len, synth.SEED_KVFILL)
    _all(q, engs, prep)
    kb = q.batch_from_synth(b)
    outs = _all(q, engs, lambda r, e: e.step_host(kb, cfg.vocab))
    for lg_r, _ in outs[1:]:
        assert np.array_equal(lg_r, outs[0][0])
    lg = outs[0][0]
    sample = [0, 13, 31]
    orc = _oracle("llama3-70b", n_layers=2,
                  num_blocks=(KS + C) // 16 + 1 + sum(ctx[j] // 16 + 2 for j in sample))
    orc.kv_alloc(0, KS + C)
    orc.kv_fill_synthetic(0, KS, synth.SEED_KVFILL)
    decs = []
    for j in sample:
        d = b.decode[j]
        orc.kv_alloc(d.req, d.ctx_len + 1)
        orc.kv_fill_synthetic(d.req, d.ctx_len, synth.SEED_KVFILL)
        decs.append((d.req, d.ctx_len, d.token))
    ref = orc.hybrid_step([(0, KS, [int(t) for t in b.prefill[0].tokens])], decs)
    got = np.concatenate([lg[:1], lg[[1 + j for j in sample]]])
    assert row_rel_err(got, ref) <= TOL_LOGITS
    _close(g, engs)


ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _ipc_worker(rank, tp, gid, preset_name, ffn, twoshot, out_q, swab=1):
    import sys
    sys.path.insert(0, ROOT)
    sys.path.insert(0, os.path.join(ROOT, "tests"))
    try:
        import torch
        torch.cuda.set_device(0)
        import synth as sy
        from paper_conf_asplos_goelmkar26_b200 import qoserve as q
        from paper_conf_asplos_goelmkar26_b200.presets import preset
        over = {"ffn_dim": ffn} if ffn else {}
        cfg = q.model_cfg(**preset(preset_name, **over), num_blocks=256, max_seq_len=4096, max_requests=64,
                          max_batch_tokens=1024, max_batch_rows=32)
        g = q.Group(tp, gid, rank)
        e = q.Engine(cfg, 0, rank, tp, group=g)
        e.qos_engine_set_option("tp_twoshot", twoshot)
        e.qos_engine_set_option("gemm_swab", swab)
        e.qos_engine_load_synthetic(0)
        ctxs, warm, main, second = sy.tiny_scenario(cfg.vocab)
        for r, n in ctxs.items():
            e.qos_kv_alloc(r, n + 2)
        e.qos_kv_alloc(0, 256)
        outs = [e.step_host(q.batch_from_synth(b), cfg.vocab) for b in warm + [main, second]]
        tables = {r: e.qos_kv_table(r) for r in list(ctxs) + [0]}
        e.close()
        g.close()
        out_q.put((rank, outs, tables, None))
    except Exception as ex:  # surfaced by the parent
        out_q.put((rank, None, None, repr(ex)))


@pytest.mark.parametrize("preset,tp,ffn,twoshot,swab", [("tiny", 2, None, 0, 1), ("tiny-mha", 4, 1024, 1, 1),
                                                         ("tiny-mha", 4, 1024, 1, 0)])
def test_tp_cross_process_group_tiny_scenario(preset, tp, ffn, twoshot, swab):
    """One process per rank (the torchrun layout), all on cuda:0: the group is opened from a
    shared-memory id, workspaces and sync events are exchanged as CUDA IPC handles, and the
    collectives read / store peer memory of other processes.  Results vs the unsharded oracle;
    all ranks bit-identical."""
    import multiprocessing as mp

    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    ctx = mp.get_context("spawn")
    out_q = ctx.Queue()
    gid = q.qos_group_unique_id()
    procs = [ctx.Process(target=_ipc_worker, args=(r, tp, gid, preset, ffn, twoshot, out_q, swab)) for r in range(tp)]
    for p in procs:
        p.start()
    res = {}
    try:
        for _ in range(tp):
            rank, outs, tables, err = out_q.get(timeout=600)
            assert err is None, (rank, err)
            res[rank] = (outs, tables)
    finally:
        for p in procs:
            p.join(timeout=60)
            if p.is_alive():
                p.kill()
    orc = _oracle(preset, ffn_dim=ffn, num_blocks=256)
    ctxs, warm, main, second = synth.tiny_scenario(1024)
    for r, n in ctxs.items():
        orc.kv_alloc(r, n + 2)
    orc.kv_alloc(0, 256)
    for k, b in enumerate(warm + [main, second]):
        ref = orc.hybrid_step(*b.as_oracle())
        lg0, tk0 = res[0][0][k]
        for rank in range(1, tp):
            assert np.array_equal(res[rank][0][k][0], lg0) and np.array_equal(res[rank][0][k][1], tk0)
        assert row_rel_err(lg0, ref) <= TOL_LOGITS
    for r in list(ctxs) + [0]:
        for rank in range(tp):
            assert res[rank][1][r] == orc.kv_table(r)
