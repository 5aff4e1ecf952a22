"""Pins of the fp64 oracle against things other than itself (CPU only).

Each test pins one oracle function to a published constant, a closed form, an invariant, a
library routine, or brute force — chosen so that a plausible mistake (dropped term, wrong
sign or index, transposed operand) fails at least one of them.
"""
import numpy as np
import pytest
import torch
import torch.nn.functional as F

from oracle import gen
from oracle.model import (PRESETS, apply_rope, attention_one, causal_attention, rms_norm,
                          rope_inv_freq, silu, softmax, swiglu_mlp)

RNG = np.random.default_rng(1234)


# ------------------------------------------------------------------ generator primitives
def test_splitmix64_published_vector():
    # Vigna's reference splitmix64: state 0 -> first output 0xE220A8397B1DCDAF,
    # second 0x6E789E6AA1B965F4 (state advanced by the golden gamma).
    assert gen.splitmix64_int(0) == 0xE220A8397B1DCDAF
    assert gen.splitmix64_int(0x9E3779B97F4A7C15) == 0x6E789E6AA1B965F4


def test_splitmix64_vectorised_matches_scalar():
    zs = [0, 1, 2, 12345678901234567, (1 << 64) - 1, 0xDEADBEEFCAFEBABE]
    v = gen.splitmix64_np(np.array(zs, dtype=np.uint64))
    assert [int(x) for x in v] == [gen.splitmix64_int(z) for z in zs]


def test_fnv1a64_published_vectors():
    assert gen.fnv1a64(b"") == 0xCBF29CE484222325
    assert gen.fnv1a64(b"a") == 0xAF63DC4C8601EC8C
    assert gen.fnv1a64(b"foobar") == 0x85944171F73967E8


def test_bf16_rne_matches_torch():
    x = (RNG.standard_normal(100000) * np.exp(RNG.uniform(-20, 20, 100000))).astype(np.float32)
    x[:6] = [1.0, 1.0 + 2**-8, 1.0 + 3 * 2**-8, -0.0, 65504.0, 1e-40]
    ours = gen.bf16_rne_bits(x)
    ref = torch.from_numpy(x).to(torch.bfloat16).view(torch.int16).numpy().view(np.uint16)
    assert np.array_equal(ours, ref)
    assert ours[0] == 0x3F80 and ours[1] == 0x3F80 and ours[2] == 0x3F82  # ties to even


def test_generator_distribution_and_kinds():
    a = gen._a_values(0, "t", 0, 200000).astype(np.float64)
    assert a.min() >= -1.0 and a.max() < 1.0
    assert abs(a.mean()) < 0.01 and abs(a.var() - 1 / 3) < 0.01
    # k is 24-bit -> a has at most 24 significant bits (exact in fp32)
    assert np.all(np.round(a * 2**23) == a * 2**23)
    w = gen.gen_tensor(0, "w", "linear", (64, 4096), fan_in=4096)
    assert abs(w.std() - 1 / np.sqrt(3 * 4096)) < 0.02 / np.sqrt(4096)
    g = gen.gen_tensor(0, "g", "norm", (4096,))
    assert g.min() >= 0.9 - 2**-8 and g.max() <= 1.1 + 2**-7  # bf16 spacing
    b = gen.gen_tensor(0, "b", "bias", (4096,))
    assert np.abs(b).max() <= 0.02 + 1e-4
    # row slicing is consistent with the flat index
    full = gen.gen_tensor(7, "x", "embed", (10, 33))
    part = gen.gen_tensor(7, "x", "embed", (10, 33), row_start=4, row_end=7)
    assert np.array_equal(full[4:7], part)
    # different names / seeds give different streams
    assert not np.array_equal(gen.gen_tensor(0, "x", "embed", (4, 8)), gen.gen_tensor(1, "x", "embed", (4, 8)))


def test_generator_golden_values():
    # the vectorised generator against the scalar spec written out element by element
    # (splitmix64_int, explicit fp32 multiply, RNE rounding)
    name = "model.layers.0.self_attn.q_proj.weight"
    base = 0 ^ gen.fnv1a64(name.encode())
    for i in (0, 1, 4095, 123456):
        k = gen.splitmix64_int((base + i) & gen.MASK64) >> 40
        a = np.float32((k - 2**23) / 2**23)
        w32 = np.float32(a * np.float32(1 / np.sqrt(4096.0)))
        expect = gen.bf16_rne_bits(np.array([w32]))[0]
        got = gen.gen_bits(0, name, "linear", i, 1, fan_in=4096)[0]
        assert got == expect


# ------------------------------------------------------------------ norm / rope / mlp
def test_rms_norm_vs_torch():
    x = RNG.standard_normal((7, 256))
    g = RNG.uniform(0.9, 1.1, 256)
    ref = F.rms_norm(torch.from_numpy(x), (256,), torch.from_numpy(g), eps=1e-5).numpy()
    assert np.allclose(rms_norm(x, g, 1e-5), ref, rtol=1e-13, atol=1e-13)


def test_rms_norm_closed_form():
    x = np.full((1, 64), 3.0)
    out = rms_norm(x, np.ones(64), 0.0)
    assert np.allclose(out, 1.0)


def test_rope_identity_norm_and_relative_position():
    hd, theta = 128, 500000.0
    x = RNG.standard_normal((5, 3, hd))
    assert np.allclose(apply_rope(x, np.zeros(5), theta), x, atol=0)
    pos = np.array([0, 1, 17, 4095, 32767])
    r = apply_rope(x, pos, theta)
    assert np.allclose(np.linalg.norm(r, axis=-1), np.linalg.norm(x, axis=-1), rtol=1e-12)
    q = RNG.standard_normal((1, 1, hd))
    k = RNG.standard_normal((1, 1, hd))
    def dot(m, n):
        return float(np.sum(apply_rope(q, np.array([m]), theta) * apply_rope(k, np.array([n]), theta)))
    assert np.isclose(dot(10, 3), dot(107, 100), rtol=1e-10)
    assert np.isclose(dot(5000, 4000), dot(1000, 0), rtol=1e-9)


def test_rope_matches_complex_rotation():
    # independent formulation: pair (x_i, x_{i+hd/2}) as the complex number x_i + j*x_{i+hd/2}
    # rotated by angle pos * theta^(-2i/hd)
    hd, theta = 64, 10000.0
    x = RNG.standard_normal((4, 2, hd))
    pos = np.array([0, 3, 100, 511])
    z = x[..., : hd // 2] + 1j * x[..., hd // 2:]
    ang = pos[:, None, None] * (theta ** (-np.arange(0, hd, 2) / hd))[None, None, :]
    zr = z * np.exp(1j * ang)
    ref = np.concatenate([zr.real, zr.imag], axis=-1)
    assert np.allclose(apply_rope(x, pos, theta), ref, rtol=1e-12, atol=1e-12)
    assert np.isclose(rope_inv_freq(theta, hd)[1], theta ** (-2 / hd))


def test_silu_and_swiglu_vs_torch():
    x = RNG.standard_normal(1000) * 5
    assert np.allclose(silu(x), F.silu(torch.from_numpy(x)).numpy(), rtol=1e-14, atol=1e-15)
    h = RNG.standard_normal((3, 32))
    Wg, Wu, Wd = RNG.standard_normal((48, 32)), RNG.standard_normal((48, 32)), RNG.standard_normal((32, 48))
    th = torch.from_numpy(h)
    ref = (F.silu(th @ torch.from_numpy(Wg).T) * (th @ torch.from_numpy(Wu).T)) @ torch.from_numpy(Wd).T
    assert np.allclose(swiglu_mlp(h, Wg, Wu, Wd), ref.numpy(), rtol=1e-12)


# ------------------------------------------------------------------ attention
def test_softmax_rows_sum_to_one():
    s = RNG.standard_normal((50, 300)) * 30
    p = softmax(s)
    assert np.allclose(p.sum(-1), 1.0, atol=1e-12)
    assert np.all(p >= 0)


def test_attention_one_brute_force():
    hd, n = 16, 9
    q, K, V = RNG.standard_normal(hd), RNG.standard_normal((n, hd)), RNG.standard_normal((n, hd))
    w = [np.exp(sum(q[i] * K[j, i] for i in range(hd)) / np.sqrt(hd)) for j in range(n)]
    z = sum(w)
    ref = [sum(w[j] / z * V[j, i] for j in range(n)) for i in range(hd)]
    assert np.allclose(attention_one(q, K, V), ref, rtol=1e-12)


def test_attention_special_cases():
    hd = 8
    V = RNG.standard_normal((5, hd))
    # equal scores -> mean of V
    assert np.allclose(attention_one(np.zeros(hd), RNG.standard_normal((5, hd)), V), V.mean(0))
    # one dominant key -> its value row
    K = np.zeros((5, hd))
    K[3, 0] = 1e4
    q = np.zeros(hd)
    q[0] = 1.0
    assert np.allclose(attention_one(q, K, V), V[3])


@pytest.mark.parametrize("H,Hkv", [(4, 4), (4, 2), (8, 1)])
def test_causal_attention_vs_torch_sdpa(H, Hkv):
    n, hd = 37, 16
    Q = RNG.standard_normal((n, H, hd))
    K = RNG.standard_normal((n, Hkv, hd))
    V = RNG.standard_normal((n, Hkv, hd))
    g = H // Hkv
    tq = torch.from_numpy(Q).permute(1, 0, 2)
    tk = torch.from_numpy(K).permute(1, 0, 2).repeat_interleave(g, dim=0)
    tv = torch.from_numpy(V).permute(1, 0, 2).repeat_interleave(g, dim=0)
    ref = F.scaled_dot_product_attention(tq, tk, tv, is_causal=True).permute(1, 0, 2).numpy()
    assert np.allclose(causal_attention(Q, K, V, 0, g), ref, rtol=1e-11, atol=1e-12)


def test_causal_attention_with_prefix_equals_suffix_rows_of_full():
    H, Hkv, hd, P, n = 4, 2, 16, 40, 13
    Q = RNG.standard_normal((P + n, H, hd))
    K = RNG.standard_normal((P + n, Hkv, hd))
    V = RNG.standard_normal((P + n, Hkv, hd))
    full = causal_attention(Q, K, V, 0, 2)
    part = causal_attention(Q[P:], K, V, P, 2)
    assert np.allclose(full[P:], part, rtol=1e-13, atol=1e-14)


def test_presets_shapes():
    c = PRESETS["llama3-8b"]
    body = c.n_layers * (c.d_model * (c.n_heads + 2 * c.n_kv_heads) * c.head_dim
                         + c.n_heads * c.head_dim * c.d_model + 3 * c.d_model * c.ffn_dim)
    assert abs(body / 1e9 - 6.98) < 0.01          # SURVEY.md §8 preset table: 6.98 B body params
    assert c.n_heads % c.n_kv_heads == 0
