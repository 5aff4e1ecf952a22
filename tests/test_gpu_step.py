"""End-to-end parity of qos_hybrid_step against the fp64 oracle (through the C ABI).

* tiny (configs[0]): chunked prefills of 4 prompts (splits {64, 100, 128}), then a 128-token
  chunk + 4 decodes, then a second chunk at kv_start 128 + decodes; logits rel-err <= 1e-2,
  greedy tokens identical, KV tables (host and device mirror) bit-exact vs the oracle's
  allocator (north star); batch-composition and chunk-split invariance on the GPU.
* Llama-3-8B shapes (2 layers, full width) at the bench batch shape (2048-token chunk +
  128 decodes @ ctx 4096 with synthetic KV): sampled rows vs the oracle.
"""
import numpy as np
import pytest

import synth
from helpers import TOL_LOGITS, make_engine, row_rel_err

pytestmark = pytest.mark.gpu


def _oracle(preset, **kw):
    from oracle.engine import OracleEngine
    from oracle.model import PRESETS, with_layers
    c = PRESETS[preset]
    if "n_layers" in kw:
        c = with_layers(c, kw.pop("n_layers"))
    return OracleEngine(c, seed=0, **kw)


def _run_tiny(preset):
    q, cfg, eng = make_engine(preset, num_blocks=256)
    eng.qos_engine_load_synthetic(0)
    orc = _oracle(preset, num_blocks=256)
    ctxs, warm, main, second = synth.tiny_scenario(cfg.vocab)
    for r, n in ctxs.items():
        eng.qos_kv_alloc(r, n + 2)
        orc.kv_alloc(r, n + 2)
    eng.qos_kv_alloc(0, 256)
    orc.kv_alloc(0, 256)
    errs = []
    for k, b in enumerate(warm + [main, second]):
        lg, tk = eng.step_host(q.batch_from_synth(b), cfg.vocab)
        ref = orc.hybrid_step(*b.as_oracle())
        errs.append(row_rel_err(lg, ref))
        srt = np.sort(ref, 1)
        gap = (srt[:, -1] - srt[:, -2]) / np.abs(ref).max(1)
        rt = np.argmax(ref, 1)
        for i in range(len(rt)):
            # identical greedy tokens unless the oracle's top-2 gap is inside the tolerance
            # (reading s11); logged either way
            assert tk[i] == rt[i] or gap[i] <= 2 * TOL_LOGITS, (k, i, errs[-1], gap[i], tk[i], rt[i])
    for r in list(ctxs) + [0]:
        assert eng.qos_kv_table(r) == orc.kv_table(r)
        assert eng.qos_kv_table_device(r) == orc.kv_table(r)
        assert eng.qos_kv_cached_len(r) == orc.cached_len(r)
    return q, cfg, eng, orc, max(errs)


@pytest.mark.parametrize("preset", ["tiny", "tiny-mha", "tiny-qwen"])
def test_tiny_scenario_parity(preset):
    q, cfg, eng, orc, err = _run_tiny(preset)
    assert err <= TOL_LOGITS, err
    eng.close()


def test_tiny_greedy_decode_loop_tokens_identical():
    """Autoregressive decode: feed each step's argmax back in; the GPU and
    the oracle must produce the same token sequence (north star: greedy tokens identical)."""
    q, cfg, eng, orc, _ = _run_tiny("tiny")
    ctxs = {1: 39, 2: 202, 3: 313, 4: 514}        # after tiny_scenario (+2 steps)
    toks = {r: 5 + r for r in ctxs}
    for r, n in ctxs.items():
        eng.qos_kv_alloc(r, n + 40)
        orc.kv_alloc(r, n + 40)
    for step in range(30):
        dec = [(r, ctxs[r], toks[r]) for r in sorted(ctxs)]
        lg, tk = eng.step_host(q.make_batch([], dec), cfg.vocab)
        ref = orc.hybrid_step([], dec)
        rt = np.argmax(ref, 1)
        # argmax must be identical unless the oracle's top-2 gap is inside the tolerance
        srt = np.sort(ref, 1)
        gap = (srt[:, -1] - srt[:, -2]) / np.abs(ref).max(1)
        for i, r in enumerate(sorted(ctxs)):
            if gap[i] > 2 * TOL_LOGITS:
                assert tk[i] == rt[i], (step, r)
            toks[r] = int(rt[i])
            ctxs[r] += 1
        assert row_rel_err(lg, ref) <= TOL_LOGITS
    eng.close()


def test_device_token_feedback_loop_matches_host_loop():
    """qos_hybrid_step_ex: a greedy loop whose decode tokens are the previous step's DEVICE
    next_tokens (steps enqueued back to back, no host round trip between them) gives exactly the
    logits and tokens of the same loop fed back through the host, which the oracle checks.  The
    steps also carry a prefill chunk each (chunk row first, so the decode tokens are
    next_tokens + 1 of the previous step) and the descriptor's decode tokens are wrong on purpose."""
    import torch
    from oracle.engine import OracleEngine
    from oracle.model import PRESETS
    V = 1024
    runs = []
    for mode in ("host", "device"):
        q, cfg, eng = make_engine("tiny", num_blocks=256)
        eng.qos_engine_load_synthetic(0)
        prompts = {r: synth.request_tokens(r, 20 + 7 * r, V) for r in (1, 2, 3)}
        for r, p in prompts.items():
            eng.qos_kv_alloc(r, len(p) + 12)
        lg, tk = eng.step_host(q.make_batch([(r, 0, p) for r, p in prompts.items()], []), V)
        toks = {r: int(tk[i]) for i, r in enumerate(prompts)}
        if mode == "host":
            init_toks = dict(toks)
        ctx = {r: len(p) for r, p in prompts.items()}
        outs = []
        if mode == "device":
            st = torch.cuda.current_stream()
            dev = [torch.empty(4, dtype=torch.int32, device="cuda") for _ in range(10)]
            dlg = [torch.empty((4, V), dtype=torch.float32, device="cuda") for _ in range(10)]
            first = torch.tensor([toks[r] for r in sorted(prompts)], dtype=torch.int32, device="cuda")
        for k in range(10):
            chunk_req = 100 + k
            eng.qos_kv_alloc(chunk_req, 16)
            pre = [(chunk_req, 0, synth.request_tokens(chunk_req, 16, V))]
            if mode == "host":
                dec = [(r, ctx[r], toks[r]) for r in sorted(prompts)]
                lg, tk = eng.step_host(q.make_batch(pre, dec), V)
                outs.append((lg, tk))
                toks = {r: int(tk[1 + i]) for i, r in enumerate(sorted(prompts))}
            else:
                dec = [(r, ctx[r], 0) for r in sorted(prompts)]  # ignored: tokens come from the device
                src = first.data_ptr() if k == 0 else dev[k - 1].data_ptr() + 4
                eng.qos_hybrid_step_ex(q.make_batch(pre, dec), dlg[k].data_ptr(), q.QOS_F32, dev[k].data_ptr(), False,
                                       st.cuda_stream, src)
            for r in prompts:
                ctx[r] += 1
        if mode == "device":
            torch.cuda.synchronize()
            outs = [(dlg[k].cpu().numpy(), dev[k].cpu().numpy()) for k in range(10)]
        runs.append(outs)
        eng.close()
    for (la, ta), (lb, tb) in zip(*runs):
        assert np.array_equal(la, lb) and np.array_equal(ta, tb)
    # and the host loop against the oracle for the first decode step (same descriptor)
    orc = OracleEngine(PRESETS["tiny"], seed=0, num_blocks=256)
    prompts = {r: synth.request_tokens(r, 20 + 7 * r, V) for r in (1, 2, 3)}
    for r, p in prompts.items():
        orc.kv_alloc(r, len(p) + 12)
    ref0 = orc.hybrid_step([(r, 0, list(p)) for r, p in prompts.items()], [])
    orc.kv_alloc(100, 16)
    dec = [(r, len(prompts[r]), init_toks[r]) for r in sorted(prompts)]
    ref = orc.hybrid_step([(100, 0, list(synth.request_tokens(100, 16, V)))], dec)
    assert row_rel_err(runs[0][0][0], ref) <= TOL_LOGITS


def test_batch_composition_and_split_invariance_on_gpu():
    q, cfg, eng = make_engine("tiny", num_blocks=256)
    eng.qos_engine_load_synthetic(0)
    toks = synth.request_tokens(7, 150, cfg.vocab)
    other = synth.request_tokens(8, 90, cfg.vocab)
    eng.qos_kv_alloc(7, 150)
    eng.qos_kv_alloc(8, 90)
    eng.qos_kv_alloc(9, 150)
    # (a) req 7 in one chunk, mixed with req 8's chunk
    la, _ = eng.step_host(q.make_batch([(7, 0, toks), (8, 0, other)], []), cfg.vocab)
    # (b) req 9 = same tokens, split 64 + 50 + 36, alone
    eng.step_host(q.make_batch([(9, 0, toks[:64])], []), cfg.vocab)
    eng.step_host(q.make_batch([(9, 64, toks[64:114])], []), cfg.vocab)
    lb, _ = eng.step_host(q.make_batch([(9, 114, toks[114:])], []), cfg.vocab)
    # bf16 activations make the two schedules differ only by rounding
    assert row_rel_err(la[:1], lb) <= TOL_LOGITS
    eng.close()


def test_step_errors_leave_state_unchanged():
    q, cfg, eng = make_engine("tiny", num_blocks=8)
    eng.qos_engine_load_synthetic(0)
    eng.qos_kv_alloc(1, 20)
    with pytest.raises(q.QosError) as ei:
        eng.step_host(q.make_batch([(1, 0, np.zeros(33, np.int32))], []), cfg.vocab)
    assert ei.value.name == "NOT_ALLOCATED"
    with pytest.raises(q.QosError) as ei:
        eng.step_host(q.make_batch([(1, 5, np.zeros(3, np.int32))], []), cfg.vocab)
    assert ei.value.name == "BAD_KV_START"
    with pytest.raises(q.QosError) as ei:
        eng.step_host(q.make_batch([], [(42, 0, 1)]), cfg.vocab)
    assert ei.value.name == "UNKNOWN_REQ"
    with pytest.raises(q.QosError) as ei:
        eng.step_host(q.make_batch([(1, 0, np.array([cfg.vocab], np.int32))], []), cfg.vocab)
    assert ei.value.name == "INVALID_ARG"
    with pytest.raises(q.QosError) as ei:
        eng.step_host(q.make_batch([], []), cfg.vocab)                       # empty batch
    assert ei.value.name == "INVALID_ARG"
    with pytest.raises(q.QosError) as ei:                                    # a request twice in one step
        eng.step_host(q.make_batch([(1, 0, np.zeros(3, np.int32))], [(1, 0, 1)]), cfg.vocab)
    assert ei.value.name == "INVALID_ARG"
    with pytest.raises(q.QosError) as ei:                                    # rows > max_batch_rows (32)
        eng.step_host(q.make_batch([(1, 0, np.zeros(1, np.int32))], [(1000 + i, 0, 1) for i in range(32)]),
                      cfg.vocab)
    assert ei.value.name == "INVALID_ARG"
    assert eng.qos_kv_cached_len(1) == 0
    free = eng.qos_kv_free_blocks()
    with pytest.raises(q.QosError) as ei:
        eng.qos_kv_alloc(2, 16 * 8)
    assert ei.value.name == "OOM" and eng.qos_kv_free_blocks() == free
    eng.step_host(q.make_batch([(1, 0, np.ones(20, np.int32))], []), cfg.vocab)
    assert eng.qos_kv_cached_len(1) == 20
    with pytest.raises(q.QosError) as ei:
        eng.qos_kv_free(99)
    assert ei.value.name == "UNKNOWN_REQ"
    eng.close()


def test_engine_refuses_a_decode_work_list_beyond_its_workspace():
    """max_batch_rows x kv heads must fit the decode item workspace (65536 items): a config
    that could exceed it is refused at creation instead of looping in the split search."""
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    with pytest.raises(q.QosError) as ei:
        make_engine("tiny", max_batch_tokens=40000, max_batch_rows=40000)   # 40000 x 2 kv heads
    assert ei.value.name == "UNSUPPORTED"
    q_, cfg, eng = make_engine("tiny", max_batch_tokens=32768, max_batch_rows=32768)   # exactly 65536
    eng.close()


def test_free_realloc_fill_is_ordered_after_an_inflight_step():
    """qos_kv_free returns blocks at once; a fill of a new request that reuses them runs on the
    engine's internal stream, which must wait for the step still reading them (step enqueued
    asynchronously with device outputs on the caller's stream)."""
    import torch
    q, cfg, eng = make_engine("tiny", num_blocks=64)
    eng.qos_engine_load_synthetic(0)
    ctx = 600
    eng.qos_kv_alloc(1, ctx + 1)
    eng.qos_kv_fill_synthetic(1, ctx, 2)
    b = q.make_batch([], [(1, ctx, 7)])
    ref_lg, _ = eng.step_host(b, cfg.vocab)
    eng.qos_kv_free(1)
    eng.qos_kv_alloc(1, ctx + 1)                 # the same blocks again (lowest free first)
    eng.qos_kv_fill_synthetic(1, ctx, 2)
    lg = torch.empty((1, cfg.vocab), dtype=torch.float32, device="cuda")
    s = torch.cuda.Stream()
    for _ in range(3):
        with torch.cuda.stream(s):
            eng.qos_hybrid_step(b, lg.data_ptr(), q.QOS_F32, 0, 0, s.cuda_stream)
        # while the step may still run: free, take the blocks for another request, overwrite them
        eng.qos_kv_free(1)
        eng.qos_kv_alloc(2, ctx + 1)
        eng.qos_kv_fill_synthetic(2, ctx, 99)
        s.synchronize()
        assert row_rel_err(lg.cpu().numpy(), ref_lg) == 0.0
        eng.qos_kv_free(2)
        eng.qos_kv_alloc(1, ctx + 1)
        eng.qos_kv_fill_synthetic(1, ctx, 2)
    eng.close()


def test_kv_tables_match_oracle_under_churn():
    from oracle.kv import BlockAllocator, OracleOOM
    q, cfg, eng = make_engine("tiny", num_blocks=300)
    a = BlockAllocator(300)
    rng = np.random.default_rng(3)
    live = {}
    for _ in range(500):
        if live and rng.random() < 0.3:
            r = int(rng.choice(list(live)))
            eng.qos_kv_free(r)
            a.free(r)
            del live[r]
        else:
            r = int(rng.integers(0, 50))
            n = max(int(rng.integers(0, 800)), live.get(r, 0))
            try:
                a.alloc(r, n)
                ok = True
            except OracleOOM:
                ok = False
            if ok:
                eng.qos_kv_alloc(r, n)
                live[r] = n
            else:
                with pytest.raises(q.QosError):
                    eng.qos_kv_alloc(r, n)
    for r in live:
        assert eng.qos_kv_table(r) == a.table(r)
        assert eng.qos_kv_table_device(r) == a.table(r)
    assert eng.qos_kv_free_blocks() == a.n_free
    eng.close()


@pytest.mark.slow
@pytest.mark.parametrize("split", [None, 512])
def test_llama8b_shapes_bench_batch_sampled_parity(split):
    """2-layer Llama-3-8B (full width) at the bench launch shape: a 2048-token chunk at
    kv_start 0 + 128 decodes @ ctx 4096 whose prefixes hold synthetic KV.
    Default decode_split: one 4097-key item per (decode, kv head); 512: 8 splits merged by the
    last arriving item."""
    C, ND, CTX = 2048, 128, 4096
    q, cfg, eng = make_engine("llama3-8b", n_layers=2, num_blocks=(C + ND * (CTX + 1)) // 16 + 200,
                              max_seq_len=8192, max_batch_tokens=C + ND, max_batch_rows=ND + 1,
                              max_requests=ND + 8)
    eng.qos_engine_load_synthetic(0)
    if split:
        eng.qos_engine_set_option("decode_split", split)
    b = synth.hybrid_batch(cfg.vocab, C, ND, CTX)
    eng.qos_kv_alloc(0, C)
    for d in b.decode:
        eng.qos_kv_alloc(d.req, CTX + 1)
        eng.qos_kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
    lg, tk = eng.step_host(q.batch_from_synth(b), cfg.vocab)
    orc = _oracle("llama3-8b", n_layers=2, num_blocks=2 * (C // 16 + 1) + 8 * (CTX // 16 + 2))
    sample = [0, 1, 63, 127]
    orc.kv_alloc(0, C)
    pre = [(0, 0, [int(t) for t in b.prefill[0].tokens])]
    decs = []
    for j in sample:
        d = b.decode[j]
        orc.kv_alloc(d.req, CTX + 1)
        orc.kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
        decs.append((d.req, d.ctx_len, d.token))
    ref = orc.hybrid_step(pre, decs)
    got = np.concatenate([lg[:1], lg[[1 + j for j in sample]]])
    err = row_rel_err(got, ref)
    assert err <= TOL_LOGITS, err
    eng.close()


@pytest.mark.parametrize("opts", [{"overlap_attn": 0}, {"gemm_splitk": 1}, {"pdl": 0}, {"gemm_swab": 0},
                                  {"gemm_streamk": 0}, {"gemm_streamk": 2, "gemm_swab": 0},
                                  {"gemm_swab": 2}, {"decode_round_split": 0}, {"fa_poly": 0}, {"fa_poly": 2},
                                  {"fa_qtiles": 2}, {"fa_persist": 0}, {"gemm_2cta": 0},
                                  {"norm_fold": 0}, {"gemm_swab": 0, "norm_fold": 1}, {"attn_order": 1}, {"gemm_swab": 0, "gemm_2cta": 0}, {"decode_stages": 4},
                                  {"decode_split": 64}, {"decode_split": 4096}, {"decode_persist": 1},
                                  {"dual_stream": 1, "dual_min_prefill": 1, "dual_min_decode": 1},
                                  {"add_split": 0}, {"shares_device": 1}])
def test_execution_options_do_not_change_results(opts):
    """qos_engine_set_option variants (serial attention, no split-K, two-stream sub-batches)
    stay within tolerance of the oracle and give the same greedy tokens."""
    q, cfg, eng = make_engine("tiny", num_blocks=256)
    eng.qos_engine_load_synthetic(0)
    for k, v in opts.items():
        eng.qos_engine_set_option(k, v)
    orc = _oracle("tiny", num_blocks=256)
    ctxs, warm, main, second = synth.tiny_scenario(cfg.vocab)
    for r, n in ctxs.items():
        eng.qos_kv_alloc(r, n + 2)
        orc.kv_alloc(r, n + 2)
    eng.qos_kv_alloc(0, 256)
    orc.kv_alloc(0, 256)
    for b in warm + [main, second]:
        lg, tk = eng.step_host(q.batch_from_synth(b), cfg.vocab)
        ref = orc.hybrid_step(*b.as_oracle())
        assert row_rel_err(lg, ref) <= TOL_LOGITS
    with pytest.raises(q.QosError):
        eng.qos_engine_set_option("no_such_option", 1)
    with pytest.raises(q.QosError):
        eng.qos_engine_set_option("decode_split", 100)  # not a power of two
    eng.qos_engine_set_option("pdl", 1)  # process-wide: restore the defaults
    eng.qos_engine_set_option("fa_poly", 4)
    eng.close()


@pytest.mark.slow
@pytest.mark.parametrize("add_split", [1, 0])
def test_llama8b_mid_t_step_parity(add_split):
    """Mid-size step at full Llama-3-8B width (2 layers): a 512-token chunk at kv_start 0 + 128
    decodes @ ctx 1024 (T = 640).  The down projection (K = 14336) runs the ordered in-place
    split-K of the tile kernel here (3 K slices of 128 x 256 tiles, round 2); add_split = 0 is
    the whole-tile path.  Sampled rows vs the oracle within 1e-2, and the split step is
    bit-identical when repeated (slice order fixed)."""
    C, ND, CTX = 512, 128, 1024
    q, cfg, eng = make_engine("llama3-8b", n_layers=2, num_blocks=(2 * C + ND * (CTX + 2)) // 16 + 400,
                              max_seq_len=4096, max_batch_tokens=C + ND, max_batch_rows=ND + 1,
                              max_requests=ND + 8)
    eng.qos_engine_load_synthetic(0)
    eng.qos_engine_set_option("add_split", add_split)
    b = synth.hybrid_batch(cfg.vocab, C, ND, CTX)
    for d in b.decode:
        eng.qos_kv_alloc(d.req, CTX + 1)
        eng.qos_kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
    outs = []
    for rep in range(2):   # the same step twice on fresh chunk requests (decode KV rewritten in place)
        b.prefill[0].req = 1000 + rep
        eng.qos_kv_alloc(1000 + rep, C)
        lg, _ = eng.step_host(q.batch_from_synth(b), cfg.vocab)
        outs.append(lg)
        for d in b.decode:   # rewind the decodes: their position-CTX entries are rewritten next time
            eng.qos_kv_free(d.req)
            eng.qos_kv_alloc(d.req, CTX + 1)
            eng.qos_kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
    assert np.array_equal(outs[0][1:], outs[1][1:])
    orc = _oracle("llama3-8b", n_layers=2, num_blocks=C // 16 + 4 + 4 * (CTX // 16 + 2))
    sample = [0, 77, 127]
    orc.kv_alloc(0, C)
    pre = [(0, 0, [int(t) for t in b.prefill[0].tokens])]
    decs = []
    for j in sample:
        d = b.decode[j]
        orc.kv_alloc(d.req, CTX + 1)
        orc.kv_fill_synthetic(d.req, CTX, synth.SEED_KVFILL)
        decs.append((d.req, d.ctx_len, d.token))
    ref = orc.hybrid_step(pre, decs)
    got = np.concatenate([outs[0][:1], outs[0][[1 + j for j in sample]]])
    assert row_rel_err(got, ref) <= TOL_LOGITS, row_rel_err(got, ref)
    eng.close()


def test_capacity_boundaries_step_parity():
    """Edge of every capacity at once: a chunk of exactly max_batch_tokens - 1 tokens whose last
    position is max_seq_len - 1 (the last block-table column), a decode at position
    max_seq_len - 1, and R = max_batch_rows; logits vs the oracle, then one position further is
    refused without changing state."""
    q, cfg, eng = make_engine("tiny", num_blocks=256, max_seq_len=1024, max_batch_tokens=512, max_batch_rows=2)
    eng.qos_engine_load_synthetic(0)
    orc = _oracle("tiny", num_blocks=256)
    for alloc, fill in ((eng.qos_kv_alloc, eng.qos_kv_fill_synthetic), (orc.kv_alloc, orc.kv_fill_synthetic)):
        alloc(1, 1024)
        fill(1, 1024 - 511, synth.SEED_KVFILL)
        alloc(2, 1024)
        fill(2, 1023, synth.SEED_KVFILL)
    rng = np.random.default_rng(3)
    toks = [int(x) for x in rng.integers(0, cfg.vocab, 511)]
    b = q.make_batch([(1, 1024 - 511, np.array(toks, np.int32))], [(2, 1023, 5)])
    lg, _ = eng.step_host(b, cfg.vocab)
    ref = orc.hybrid_step([(1, 1024 - 511, toks)], [(2, 1023, 5)])
    assert row_rel_err(lg, ref) <= TOL_LOGITS
    assert eng.qos_kv_cached_len(1) == 1024 and eng.qos_kv_cached_len(2) == 1024
    with pytest.raises(q.QosError):                       # position 1024 >= max_seq_len / past the table
        eng.step_host(q.make_batch([], [(2, 1024, 5)]), cfg.vocab)
    assert eng.qos_kv_cached_len(2) == 1024
    eng.close()


def test_long_context_step_parity():
    """Maximum context (configs[3]: up to 32k): a 100-token chunk at kv_start 16000 and decodes
    at ctx 32767 / 20000 / 17, all prefixes synthetic KV, through qos_hybrid_step vs the oracle
    (logits rows <= 1e-2, same greedy tokens) — long block tables, many decode splits."""
    q, cfg, eng = make_engine("tiny", num_blocks=4600, max_seq_len=32784, max_requests=8)
    eng.qos_engine_load_synthetic(0)
    orc = _oracle("tiny", num_blocks=4600)
    rng = np.random.default_rng(5)
    plan = {1: 16000, 2: 32767, 3: 20000, 4: 17}
    for r, n in plan.items():
        total = n + (100 if r == 1 else 1)
        eng.qos_kv_alloc(r, total)
        orc.kv_alloc(r, total)
        eng.qos_kv_fill_synthetic(r, n, synth.SEED_KVFILL)
        orc.kv_fill_synthetic(r, n, synth.SEED_KVFILL)
    toks = [int(x) for x in rng.integers(0, cfg.vocab, 100)]
    decs = [(r, plan[r], int(rng.integers(0, cfg.vocab))) for r in (2, 3, 4)]
    b = q.make_batch([(1, plan[1], np.array(toks, np.int32))], decs)
    lg, tk = eng.step_host(b, cfg.vocab)
    ref = orc.hybrid_step([(1, plan[1], toks)], decs)
    assert row_rel_err(lg, ref) <= TOL_LOGITS
    top = np.argsort(ref, axis=1)
    gap = ref[np.arange(len(ref)), top[:, -1]] - ref[np.arange(len(ref)), top[:, -2]]
    clear = gap > 2 * TOL_LOGITS * np.abs(ref).max(axis=1)
    assert np.array_equal(np.asarray(tk)[clear], top[clear, -1])
    eng.close()


@pytest.mark.parametrize("fold", [1, 0])
def test_norm_fold_large_step_parity(fold):
    """The RMSNorm folded into the projections (taken from 1536 tokens per step: the O / down
    epilogues write r, bf16(r * g) and per-block sums of squares, the QKV / gate-up epilogues
    scale rows by 1/rms) against the oracle on a 1700-token chunk + decodes, tiny shapes."""
    q, cfg, eng = make_engine("tiny", num_blocks=512, max_batch_tokens=2048, max_seq_len=4096)
    eng.qos_engine_load_synthetic(0)
    eng.qos_engine_set_option("norm_fold", fold)
    orc = _oracle("tiny", num_blocks=512)
    rng = np.random.default_rng(11)
    toks = [int(x) for x in rng.integers(0, cfg.vocab, 1700)]
    eng.qos_kv_alloc(1, 1700)
    orc.kv_alloc(1, 1700)
    decs = []
    for r, n in ((2, 40), (3, 300)):
        eng.qos_kv_alloc(r, n + 1)
        orc.kv_alloc(r, n + 1)
        eng.qos_kv_fill_synthetic(r, n, synth.SEED_KVFILL)
        orc.kv_fill_synthetic(r, n, synth.SEED_KVFILL)
        decs.append((r, n, int(rng.integers(0, cfg.vocab))))
    lg, tk = eng.step_host(q.make_batch([(1, 0, np.array(toks, np.int32))], decs), cfg.vocab)
    ref = orc.hybrid_step([(1, 0, toks)], decs)
    assert row_rel_err(lg, ref) <= TOL_LOGITS
    eng.close()
