"""Kernel-level parity on the B200 (one test per SURVEY.md §8(a) row), through the C ABI.

Inputs are seeded on the host, rounded to bf16, and fed to both the CUDA op and the fp64
oracle; outputs are compared with the north-star tolerances (metric of reading s9).
"""
import numpy as np
import pytest

from helpers import TOL_ATTN, bf16_bits, bits_to_f64, f16_bits, f16_bits_to_f64, make_engine, row_rel_err

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def torch_cuda():
    import torch
    assert torch.cuda.is_available()
    return torch


def _dev_bf16(torch, x):
    return torch.from_numpy(bf16_bits(x).view(np.int16)).view(torch.bfloat16).cuda()


# ------------------------------------------------------------------ weights (generator spec)
def test_weights_bit_exact_tiny():
    from oracle import gen
    from oracle.model import PRESETS, tensor_names
    q, cfg, eng = make_engine("tiny-qwen")
    eng.qos_engine_load_synthetic(0)
    c = PRESETS["tiny-qwen"]
    for l in range(c.n_layers):
        nm = tensor_names(c, l)
        for key, kind, shape, fan in [("wq", "linear", (256, 256), 256), ("wk", "linear", (128, 256), 256),
                                      ("wv", "linear", (128, 256), 256), ("wo", "linear", (256, 256), 256),
                                      ("wg", "linear", (768, 256), 256), ("wu", "linear", (768, 256), 256),
                                      ("wd", "linear", (256, 768), 768), ("ln1", "norm", (1, 256), 1),
                                      ("ln2", "norm", (1, 256), 1)]:
            ref = gen.gen_bits(0, nm[key], kind, 0, shape[0] * shape[1], fan).reshape(shape)
            got = eng.qos_engine_read_weight(nm[key], 0, shape[0], shape[1])
            assert np.array_equal(got, ref), nm[key]
    for name, kind, shape in [("model.embed_tokens.weight", "embed", (1024, 256)),
                              ("lm_head.weight", "linear", (1024, 256)), ("model.norm.weight", "norm", (1, 256))]:
        ref = gen.gen_bits(0, name, kind, 0, shape[0] * shape[1], shape[1]).reshape(shape)
        assert np.array_equal(eng.qos_engine_read_weight(name, 0, shape[0], shape[1]), ref), name
    eng.close()


def test_weights_bit_exact_8b_sampled():
    from oracle import gen
    q, cfg, eng = make_engine("llama3-8b", n_layers=2, num_blocks=64, max_batch_tokens=256, max_batch_rows=16)
    eng.qos_engine_load_synthetic(0)
    checks = [("model.layers.1.mlp.gate_proj.weight", 14336, 4096, 4096, [0, 63, 64, 5000, 14335]),
              ("model.layers.1.mlp.up_proj.weight", 14336, 4096, 4096, [0, 65, 14335]),
              ("model.layers.0.mlp.down_proj.weight", 4096, 14336, 14336, [0, 4095]),
              ("model.layers.0.self_attn.o_proj.weight", 4096, 4096, 4096, [7, 4000]),
              ("model.layers.0.self_attn.k_proj.weight", 1024, 4096, 4096, [0, 1023]),
              ("lm_head.weight", 128256, 4096, 4096, [0, 128255]),
              ("model.embed_tokens.weight", 128256, 4096, 1, [77])]
    for name, rows, cols, fan, sample in checks:
        kind = "embed" if "embed" in name else "linear"
        for r in sample:
            ref = gen.gen_bits(0, name, kind, r * cols, cols, fan)
            got = eng.qos_engine_read_weight(name, r, 1, cols)[0]
            assert np.array_equal(got, ref), (name, r)
    eng.close()


# ------------------------------------------------------------------ GEMM (a4, a9, a11, a12, a13)
@pytest.mark.parametrize("M,N,K", [(1, 256, 64), (77, 384, 320), (128, 512, 256), (300, 96, 128),
                                   (700, 1024, 512), (2176, 1536, 1024)])
@pytest.mark.parametrize("epi", ["store_f32", "store_bf16", "add_f32", "bias_bf16"])
def test_gemm_parity(torch_cuda, M, N, K, epi):
    torch = torch_cuda
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(M * 7 + N + K)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    B = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (N, K)) / np.sqrt(K)))
    ref = A @ B.T                                   # numpy fp64 (the oracle's GEMM primitive)
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, B)
    bias = None
    if epi in ("store_f32", "add_f32"):
        init = rng.uniform(-1, 1, (M, N)).astype(np.float32) if epi == "add_f32" else np.zeros((M, N), np.float32)
        dC = torch.from_numpy(init.copy()).cuda()
        ref = ref + init.astype(np.float64)
    else:
        dC = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        if epi == "bias_bf16":
            bvals = bits_to_f64(bf16_bits(rng.uniform(-0.02, 0.02, N)))
            bias = torch.from_numpy(bvals.astype(np.float32)).cuda()
            ref = ref + bvals
    q.qos_op_gemm(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, N, K, epi,
                  bias.data_ptr() if bias is not None else None)
    torch.cuda.synchronize()
    got = dC.float().cpu().numpy()
    tol = 1e-5 if epi in ("store_f32", "add_f32") else 8e-3   # fp32 out vs bf16 rounding (2^-8)
    assert row_rel_err(got, ref) <= tol


@pytest.mark.parametrize("M,F,K", [(1, 128, 64), (200, 384, 256), (1000, 768, 512)])
def test_gemm_silu_gate_parity(torch_cuda, M, F, K):
    torch = torch_cuda
    from oracle.model import swiglu_mlp, silu
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(F + K)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    Wg = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (F, K)) / np.sqrt(K)))
    Wu = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (F, K)) / np.sqrt(K)))
    # QOS_EPI_SILU_GATE interleave: rows [128j, 128j+64) gate rows [64j, ...), then 64 up rows
    Bi = np.empty((2 * F, K))
    for j in range(F // 64):
        Bi[128 * j:128 * j + 64] = Wg[64 * j:64 * j + 64]
        Bi[128 * j + 64:128 * j + 128] = Wu[64 * j:64 * j + 64]
    ref = silu(A @ Wg.T) * (A @ Wu.T)
    dC = torch.empty((M, F), dtype=torch.bfloat16, device="cuda")
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, Bi)     # keep the device inputs alive
    q.qos_op_gemm(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, 2 * F, K, "silu_gate")
    torch.cuda.synchronize()
    assert row_rel_err(dC.float().cpu().numpy(), ref) <= 8e-3
    del swiglu_mlp


# ------------------------------------------------------------------ RMSNorm (a3)
def test_rmsnorm_parity(torch_cuda):
    torch = torch_cuda
    from oracle.model import rms_norm
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(5)
    for T, d in [(1, 256), (33, 4096), (7, 5120), (3, 8192)]:
        x = rng.standard_normal((T, d)).astype(np.float32)
        g = bits_to_f64(bf16_bits(rng.uniform(0.9, 1.1, d)))
        out = torch.empty((T, d), dtype=torch.bfloat16, device="cuda")
        dx, dg = torch.from_numpy(x).cuda(), _dev_bf16(torch, g)   # keep the device inputs alive
        q.qos_op_rmsnorm(dx.data_ptr(), dg.data_ptr(), out.data_ptr(), T, d, 1e-5)
        torch.cuda.synchronize()
        assert row_rel_err(out.float().cpu().numpy(), rms_norm(x.astype(np.float64), g, 1e-5)) <= 8e-3


# ------------------------------------------------------------------ QKV + RoPE + KV append (a4, a5, a6)
@pytest.mark.parametrize("preset,over", [("tiny", {}), ("tiny-qwen", {}),
                                         ("llama3-8b", dict(n_layers=1, num_blocks=128))])
def test_qkv_rope_append_parity(preset, over):
    """The fused QKV GEMM epilogue: q = RoPE(h Wq^T (+bq)), k = RoPE(h Wk^T (+bk)) -> cache,
    v = h Wv^T (+bv) -> cache, against the oracle on the same bf16 h and generated weights."""
    from oracle.model import PRESETS as OP, Weights, apply_rope, with_layers
    q, cfg, eng = make_engine(preset, **over)
    eng.qos_engine_load_synthetic(0)
    c = OP[preset] if "n_layers" not in over else with_layers(OP[preset], over["n_layers"])
    w = Weights(c, seed=0).layer(0)
    H, Hkv, hd, d = cfg.n_heads, cfg.n_kv_heads, cfg.head_dim, cfg.d_model
    rng = np.random.default_rng(11)
    eng.qos_kv_alloc(1, 300)
    eng.qos_kv_alloc(2, 1500)
    # a 45-token chunk at kv_start 200 of req 1 + a decode of req 2 at position 1400
    b = q.make_batch([(1, 200, np.zeros(45, np.int32))], [(2, 1400, 0)])
    T = 46
    pos = np.array(list(range(200, 245)) + [1400])
    h = bits_to_f64(bf16_bits(rng.standard_normal((T, d))))
    qo = eng.qos_op_qkv_rope_append(0, b, bf16_bits(h), H * hd)
    qq, kk, vv = h @ w["wq"].T, h @ w["wk"].T, h @ w["wv"].T
    if c.qkv_bias:
        qq, kk, vv = qq + w["bq"], kk + w["bk"], vv + w["bv"]
    qr = apply_rope(qq.reshape(T, H, hd), pos, c.rope_theta)
    kr = apply_rope(kk.reshape(T, Hkv, hd), pos, c.rope_theta)
    vr = vv.reshape(T, Hkv, hd)
    # fp32-accumulated GEMM + one bf16 rounding of the stored value
    assert row_rel_err(bits_to_f64(qo).reshape(T * H, hd), qr.reshape(T * H, hd)) <= 8e-3
    k1, v1 = eng.qos_kv_read(0, 1, 200, 45, Hkv, hd)
    k2, v2 = eng.qos_kv_read(0, 2, 1400, 1, Hkv, hd)
    assert row_rel_err(bits_to_f64(np.concatenate([k1, k2])).reshape(-1, hd), kr.reshape(-1, hd)) <= 8e-3
    # V is cached in fp16 (reading r-v16)
    assert row_rel_err(f16_bits_to_f64(np.concatenate([v1, v2])).reshape(-1, hd), vr.reshape(-1, hd)) <= 2e-3
    eng.close()


# ------------------------------------------------------------------ attention (a7, a8)
ATTN_CASES = [
    # (preset, overrides, chunks [(kv_start, len)], decode ctxs, scale)
    ("tiny", {}, [(0, 1), (0, 37), (100, 128)], [0, 15, 16, 17, 300], 1.0),
    ("llama3-8b", dict(n_layers=1, num_blocks=2048), [(0, 200), (4096, 64)], [1, 1000, 5000], 1.0),
    ("llama3-8b", dict(n_layers=1, num_blocks=2048), [(31, 129)], [2047, 4095], 3.0),
    ("tiny-mha", {}, [(5, 77)], [33, 64], 1.0),
    ("llama3-70b", dict(n_layers=1, n_heads=8, n_kv_heads=1, d_model=1024, ffn_dim=1024, num_blocks=1024),
     [(0, 48)], [700, 3000], 1.0),   # group 8 = Llama-3-70B at TP8
    # configs[3] maximum context: a chunk deep into a 20k prefix and a decode over 32k keys
    ("llama3-70b", dict(n_layers=1, n_heads=8, n_kv_heads=1, d_model=1024, ffn_dim=1024, num_blocks=4096,
                        max_seq_len=32784), [(20000, 96)], [32767], 1.0),
    # GQA group 5 (Qwen-2.5-14B per rank at TP2): 125 valid rows per q tile, not 128
    ("qwen2.5-14b", dict(n_layers=1, n_heads=10, n_kv_heads=2, d_model=1280, ffn_dim=1024, num_blocks=1024),
     [(0, 300), (100, 77)], [500, 31], 1.0),
    # the bench chunk: 512 work items (more than 2 per SM), so persistent CTAs run several each
    ("llama3-8b", dict(n_layers=1, num_blocks=2048), [(0, 2048), (512, 700)], [100], 1.0),
]


@pytest.mark.parametrize("qtiles,persist,pair,dpersist", [(1, 1, 0, 0), (1, 0, 0, 0), (2, 0, 0, 0), (1, 1, 1, 0),
                                                     (1, 1, 0, 1)])
@pytest.mark.parametrize("case", range(len(ATTN_CASES)))
def test_attention_parity(case, qtiles, persist, pair, dpersist):
    """Prefill + decode attention (fp32 output) vs the fp64 oracle; prefill with 1 or 2 q tiles
    per CTA sharing every K/V tile (odd tile counts padded with a duplicate), the persistent
    single-tile kernel (several work items per CTA), and the persistent CTA-pair kernel
    (cta_group::2, hd 128; hd 64 presets fall back to the single-CTA kernel); decode attention
    one CTA per item or persistent CTAs over the item list (dpersist)."""
    from oracle.model import causal_attention
    preset, over, chunks, ctxs, scale = ATTN_CASES[case]
    q, cfg, eng = make_engine(preset, **{"max_seq_len": 8192, "max_batch_tokens": 4096, **over})
    eng.qos_engine_set_option("fa_qtiles", qtiles)
    eng.qos_engine_set_option("fa_persist", persist)
    eng.qos_engine_set_option("fa_pair", pair)
    eng.qos_engine_set_option("decode_persist", dpersist)
    H, Hkv, hd = cfg.n_heads, cfg.n_kv_heads, cfg.head_dim
    g = H // Hkv
    rng = np.random.default_rng(100 + case)
    prefill, decode, qrows, refs = [], [], [], []
    req = 0
    for ks, n in chunks:
        P = ks + n
        eng.qos_kv_alloc(req, P)
        K = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (P, Hkv, hd)) * scale))
        V = f16_bits_to_f64(f16_bits(rng.uniform(-1, 1, (P, Hkv, hd))))
        eng.qos_kv_write(0, req, 0, bf16_bits(K), f16_bits(V))
        Q = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (n, H, hd)) * scale))
        prefill.append((req, ks, np.zeros(n, np.int32)))
        qrows.append(Q)
        refs.append(causal_attention(Q, K, V, ks, g))
        req += 1
    for c in ctxs:
        eng.qos_kv_alloc(req, c + 1)
        K = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (c + 1, Hkv, hd)) * scale))
        V = f16_bits_to_f64(f16_bits(rng.uniform(-1, 1, (c + 1, Hkv, hd))))
        eng.qos_kv_write(0, req, 0, bf16_bits(K), f16_bits(V))
        Q = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (1, H, hd)) * scale))
        decode.append((req, c, 0))
        qrows.append(Q)
        refs.append(causal_attention(Q, K, V, c, g))
        req += 1
    b = q.make_batch(prefill, decode)
    Qall = np.concatenate(qrows)
    out = eng.qos_op_attention(0, b, bf16_bits(Qall))
    ref = np.concatenate(refs)
    err = row_rel_err(out.reshape(-1, hd), ref.reshape(-1, hd))
    assert err <= TOL_ATTN, err
    eng.close()


@pytest.mark.parametrize("M,N,K,ks", [(1, 512, 1024, 4), (130, 1024, 4096, 8), (256, 768, 512, 2), (77, 384, 640, 3)])
@pytest.mark.parametrize("epi", ["store_f32", "store_bf16", "add_f32", "bias_bf16", "silu_gate"])
def test_gemm_splitk_parity(torch_cuda, M, N, K, ks, epi):
    """Split-K (weight-bound small-M GEMMs): slices reduced in order by the last CTA."""
    torch = torch_cuda
    from oracle.model import silu
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(M + N + K + ks)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    B = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (N, K)) / np.sqrt(K)))
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, B)
    ref = A @ B.T
    bias = None
    if epi == "silu_gate":
        g = np.concatenate([ref[:, 128 * j:128 * j + 64] for j in range(N // 128)], axis=1)
        u = np.concatenate([ref[:, 128 * j + 64:128 * j + 128] for j in range(N // 128)], axis=1)
        ref = silu(g) * u
        dC = torch.empty((M, N // 2), dtype=torch.bfloat16, device="cuda")
    elif epi in ("store_f32", "add_f32"):
        init = rng.uniform(-1, 1, (M, N)).astype(np.float32) if epi == "add_f32" else np.zeros((M, N), np.float32)
        dC = torch.from_numpy(init.copy()).cuda()
        ref = ref + init.astype(np.float64)
    else:
        dC = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        if epi == "bias_bf16":
            bvals = bits_to_f64(bf16_bits(rng.uniform(-0.02, 0.02, N)))
            bias = torch.from_numpy(bvals.astype(np.float32)).cuda()
            ref = ref + bvals
    for _ in range(2):   # twice: the arrival counters must be reset by the reducing CTA
        if epi == "add_f32":
            dC.copy_(torch.from_numpy(init.copy()).cuda())
        q.qos_op_gemm_ex(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, N, K, epi,
                         bias.data_ptr() if bias is not None else None, ks)
        torch.cuda.synchronize()
        got = dC.float().cpu().numpy()
        tol = 1e-5 if epi in ("store_f32", "add_f32") else 8e-3
        assert row_rel_err(got, ref) <= tol


@pytest.mark.parametrize("M,N,K,ks", [(512, 4096, 4096, 2), (288, 4096, 14336, 3), (1000, 4096, 2048, 3),
                                      (777, 1280, 2048, 4), (512, 4096, 14336, 0), (640, 4096, 4096, 0)])
def test_gemm_ordered_split_add_parity(torch_cuda, M, N, K, ks):
    """Ordered in-place split-K of EPI_ADD_F32 (the O / down projections of mid-size steps):
    every K slice red.adds its fp32 partial into C after the previous slice of its tile, so the
    result is deterministic (bit-identical run to run) and within fp32 rounding of the fp64
    product; 768 units at (1000, 4096, 2048, 3) exercise several units per CTA and slices
    waiting on other CTAs; ks = 0 is the engine's automatic (tile width, slices) choice."""
    torch = torch_cuda
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(M + N + K + ks)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    B = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (N, K)) / np.sqrt(K)))
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, B)
    init = rng.uniform(-1, 1, (M, N)).astype(np.float32)
    ref = A @ B.T + init.astype(np.float64)
    dC = torch.from_numpy(init.copy()).cuda()
    outs = []
    for _ in range(3):   # the tile counters must be back at 0 after every launch
        dC.copy_(torch.from_numpy(init.copy()).cuda())
        q.qos_op_gemm_ex(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, N, K, "add_f32", None, ks)
        torch.cuda.synchronize()
        outs.append(dC.cpu().numpy().copy())
    # fp32 accumulation error grows with the reduction length: 1e-5 at K <= 4096 (the tolerance
    # of the whole-tile GEMM tests), scaled with sqrt(K / 4096) for the down projection's K
    # (the unsplit K = 14336 tile accumulates 896 MMA K-steps in one TMEM accumulator)
    tol = 1e-5 * max(1.0, np.sqrt(K / 4096))
    assert row_rel_err(outs[0], ref) <= tol, row_rel_err(outs[0], ref)
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])


@pytest.mark.parametrize("M,N,K", [(1, 256, 64), (77, 512, 320), (300, 768, 128), (1000, 4096, 512),
                                   (2176, 1024, 1024), (4100, 512, 256)])
@pytest.mark.parametrize("epi", ["store_f32", "store_bf16", "add_f32", "bias_bf16", "silu_gate"])
def test_gemm_2cta_parity(torch_cuda, M, N, K, epi):
    """CTA-pair kernel (ksplit = -3; tcgen05 cta_group::2, 256 x 256 tiles over 2 SMs): every
    epilogue, ragged M (half-empty and fully-empty 128-row halves of a pair tile), more tiles
    than CTA pairs (persistent loop over both TMEM accumulators)."""
    torch = torch_cuda
    from oracle.model import silu
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(M * 5 + N + K)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    B = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (N, K)) / np.sqrt(K)))
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, B)
    ref = A @ B.T
    bias = None
    init = None
    if epi == "silu_gate":
        g = np.concatenate([ref[:, 128 * j:128 * j + 64] for j in range(N // 128)], axis=1)
        u = np.concatenate([ref[:, 128 * j + 64:128 * j + 128] for j in range(N // 128)], axis=1)
        ref = silu(g) * u
        dC = torch.empty((M, N // 2), dtype=torch.bfloat16, device="cuda")
    elif epi in ("store_f32", "add_f32"):
        init = rng.uniform(-1, 1, (M, N)).astype(np.float32) if epi == "add_f32" else np.zeros((M, N), np.float32)
        dC = torch.from_numpy(init.copy()).cuda()
        ref = ref + init.astype(np.float64)
    else:
        dC = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        if epi == "bias_bf16":
            bvals = bits_to_f64(bf16_bits(rng.uniform(-0.02, 0.02, N)))
            bias = torch.from_numpy(bvals.astype(np.float32)).cuda()
            ref = ref + bvals
    outs = []
    for _ in range(2):
        if init is not None:
            dC.copy_(torch.from_numpy(init.copy()).cuda())
        q.qos_op_gemm_ex(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, N, K, epi,
                         bias.data_ptr() if bias is not None else None, -3)
        torch.cuda.synchronize()
        outs.append(dC.float().cpu().numpy())
    tol = 1e-5 if epi in ("store_f32", "add_f32") else 8e-3
    assert row_rel_err(outs[0], ref) <= tol
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("M,N,K", [(1, 128, 64), (16, 4096, 4096), (17, 1024, 2048), (100, 640, 1536),
                                   (256, 512, 8192), (300, 384, 1024)])
@pytest.mark.parametrize("epi", ["store_f32", "store_bf16", "add_f32", "bias_bf16", "silu_gate"])
def test_gemm_swab_parity(torch_cuda, M, N, K, epi):
    """Weight-streaming swap-AB stream-K kernel (ksplit < 0): every epilogue, ragged token
    counts, tiles cut across CTAs (K up to 8192), two token tiles (M = 300); run twice —
    the per-tile arrival counters must be reset, and the fixed-order reduction makes the two
    results bit-identical."""
    torch = torch_cuda
    from oracle.model import silu
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(M * 3 + N + K)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    B = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (N, K)) / np.sqrt(K)))
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, B)
    ref = A @ B.T
    bias = None
    init = None
    if epi == "silu_gate":
        g = np.concatenate([ref[:, 128 * j:128 * j + 64] for j in range(N // 128)], axis=1)
        u = np.concatenate([ref[:, 128 * j + 64:128 * j + 128] for j in range(N // 128)], axis=1)
        ref = silu(g) * u
        dC = torch.empty((M, N // 2), dtype=torch.bfloat16, device="cuda")
    elif epi in ("store_f32", "add_f32"):
        init = rng.uniform(-1, 1, (M, N)).astype(np.float32) if epi == "add_f32" else np.zeros((M, N), np.float32)
        dC = torch.from_numpy(init.copy()).cuda()
        ref = ref + init.astype(np.float64)
    else:
        dC = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        if epi == "bias_bf16":
            bvals = bits_to_f64(bf16_bits(rng.uniform(-0.02, 0.02, N)))
            bias = torch.from_numpy(bvals.astype(np.float32)).cuda()
            ref = ref + bvals
    outs = []
    for _ in range(2):
        if init is not None:
            dC.copy_(torch.from_numpy(init.copy()).cuda())
        q.qos_op_gemm_ex(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, N, K, epi,
                         bias.data_ptr() if bias is not None else None, -1)
        torch.cuda.synchronize()
        outs.append(dC.float().cpu().numpy())
        tol = 1e-5 if epi in ("store_f32", "add_f32") else 8e-3
        assert row_rel_err(outs[-1], ref) <= tol
    assert np.array_equal(outs[0], outs[1])


@pytest.mark.parametrize("M,N,K", [(1, 256, 1024), (300, 512, 640), (2176, 1536, 1024), (777, 1280, 2048)])
@pytest.mark.parametrize("epi", ["store_f32", "store_bf16", "add_f32", "bias_bf16", "silu_gate"])
def test_gemm_streamk_parity(torch_cuda, M, N, K, epi):
    """Tile kernel in stream-K mode (ksplit = -2): tiles cut across CTAs, cooperative
    fixed-order reduction; run twice (counter reset) and bit-identical."""
    torch = torch_cuda
    from oracle.model import silu
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    rng = np.random.default_rng(M * 5 + N + K)
    A = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (M, K))))
    B = bits_to_f64(bf16_bits(rng.uniform(-1, 1, (N, K)) / np.sqrt(K)))
    dA, dB = _dev_bf16(torch, A), _dev_bf16(torch, B)
    ref = A @ B.T
    bias = None
    init = None
    if epi == "silu_gate":
        g = np.concatenate([ref[:, 128 * j:128 * j + 64] for j in range(N // 128)], axis=1)
        u = np.concatenate([ref[:, 128 * j + 64:128 * j + 128] for j in range(N // 128)], axis=1)
        ref = silu(g) * u
        dC = torch.empty((M, N // 2), dtype=torch.bfloat16, device="cuda")
    elif epi in ("store_f32", "add_f32"):
        init = rng.uniform(-1, 1, (M, N)).astype(np.float32) if epi == "add_f32" else np.zeros((M, N), np.float32)
        dC = torch.from_numpy(init.copy()).cuda()
        ref = ref + init.astype(np.float64)
    else:
        dC = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        if epi == "bias_bf16":
            bvals = bits_to_f64(bf16_bits(rng.uniform(-0.02, 0.02, N)))
            bias = torch.from_numpy(bvals.astype(np.float32)).cuda()
            ref = ref + bvals
    outs = []
    for _ in range(2):
        if init is not None:
            dC.copy_(torch.from_numpy(init.copy()).cuda())
        q.qos_op_gemm_ex(dA.data_ptr(), dB.data_ptr(), dC.data_ptr(), M, N, K, epi,
                         bias.data_ptr() if bias is not None else None, -2)
        torch.cuda.synchronize()
        outs.append(dC.float().cpu().numpy())
        tol = 1e-5 if epi in ("store_f32", "add_f32") else 8e-3
        assert row_rel_err(outs[-1], ref) <= tol
    assert np.array_equal(outs[0], outs[1])
