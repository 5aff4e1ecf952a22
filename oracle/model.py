"""fp64 reference math of one decoder layer stack (test infrastructure only).

The paper names only the models (Table 1: Llama3-8B GQA, Qwen-7B MHA,
Llama3-70B GQA) and never their equations; per SURVEY.md §8(c) reading s1-s3 the oracle uses
the public Llama / Qwen2 convention: pre-norm RMSNorm, rotate-half RoPE, GQA with contiguous
head groups, SwiGLU MLP, untied LM head, optional QKV bias (Qwen).  Every function below is
the textbook definition written out in fp64; no blocking, fusion or reordering.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from . import gen


@dataclass(frozen=True)
class ModelConfig:
    """Model shape (SURVEY.md §8 preset table; dims of public configs are [ext])."""
    name: str
    n_layers: int
    d_model: int
    n_heads: int
    n_kv_heads: int
    head_dim: int
    ffn_dim: int
    vocab: int
    rope_theta: float
    rms_eps: float
    qkv_bias: bool = False
    block_size: int = 16


PRESETS = {
    # configs[0]: L=2, d=256, 4 heads, block 16; Hkv/F/V/theta are our reading s15
    "tiny": ModelConfig("tiny", 2, 256, 4, 2, 64, 768, 1024, 10000.0, 1e-5),
    "tiny-mha": ModelConfig("tiny-mha", 2, 256, 4, 4, 64, 768, 1024, 10000.0, 1e-5),
    "tiny-qwen": ModelConfig("tiny-qwen", 2, 256, 4, 2, 64, 768, 1024, 1e6, 1e-6, qkv_bias=True),
    "llama3-8b": ModelConfig("llama3-8b", 32, 4096, 32, 8, 128, 14336, 128256, 500000.0, 1e-5),
    "qwen2.5-14b": ModelConfig("qwen2.5-14b", 48, 5120, 40, 8, 128, 13824, 152064, 1e6, 1e-6,
                               qkv_bias=True),
    "llama3-70b": ModelConfig("llama3-70b", 80, 8192, 64, 8, 128, 28672, 128256, 500000.0, 1e-5),
}


def with_layers(cfg: ModelConfig, n_layers: int) -> ModelConfig:
    """Same shapes, fewer layers (parity runs at full width)."""
    d = dict(cfg.__dict__)
    d["n_layers"] = n_layers
    d["name"] = f"{cfg.name}-L{n_layers}"
    return ModelConfig(**d)


# ----------------------------------------------------------------------------- primitives

def rms_norm(x: np.ndarray, g: np.ndarray, eps: float) -> np.ndarray:
    """RMSNorm over the last axis: x / sqrt(mean(x^2) + eps) * g   (reading s1)."""
    return x / np.sqrt(np.mean(x * x, axis=-1, keepdims=True) + eps) * g


def rope_inv_freq(theta: float, head_dim: int) -> np.ndarray:
    """inv_freq_i = theta^(-2i/hd), i < hd/2   (reading s2)."""
    i = np.arange(head_dim // 2, dtype=np.float64)
    return theta ** (-(2.0 * i) / head_dim)


def apply_rope(x: np.ndarray, pos: np.ndarray, theta: float) -> np.ndarray:
    """Rotate-half RoPE (pairs (i, i+hd/2)) of x[..., n, heads, hd] at positions pos[n]."""
    hd = x.shape[-1]
    half = hd // 2
    ang = np.asarray(pos, dtype=np.float64)[:, None] * rope_inv_freq(theta, hd)[None, :]
    cos = np.cos(ang)[:, None, :]
    sin = np.sin(ang)[:, None, :]
    x1 = x[..., :half]
    x2 = x[..., half:]
    return np.concatenate([x1 * cos - x2 * sin, x2 * cos + x1 * sin], axis=-1)


def softmax(s: np.ndarray) -> np.ndarray:
    """Row softmax over the last axis (max-subtracted; exact in the limit)."""
    m = np.max(s, axis=-1, keepdims=True)
    e = np.exp(s - m)
    return e / np.sum(e, axis=-1, keepdims=True)


def attention_one(q: np.ndarray, K: np.ndarray, V: np.ndarray) -> np.ndarray:
    """o = softmax(q K^T / sqrt(hd)) V for ONE query row q[hd] over keys K[n, hd], V[n, hd]
    (reading s3: scale 1/sqrt(hd))."""
    s = K @ q / np.sqrt(q.shape[-1])
    return softmax(s[None, :])[0] @ V


def causal_attention(Q: np.ndarray, K: np.ndarray, V: np.ndarray, q_pos0: int,
                     group: int) -> np.ndarray:
    """Causal GQA attention.

    Q[n, H, hd] are queries at positions q_pos0 .. q_pos0+n-1; K, V[P, Hkv, hd] hold the
    keys/values of positions 0..P-1 (P >= q_pos0+n).  Query at position p attends keys
    0..p; head h uses kv head h // group (reading s3).  Returns O[n, H, hd].
    """
    n, H, hd = Q.shape
    out = np.empty_like(Q)
    pos = q_pos0 + np.arange(n)
    key = np.arange(K.shape[0])
    mask = key[None, :] <= pos[:, None]                       # [n, P]
    for h in range(H):
        kvh = h // group
        s = Q[:, h, :] @ K[:, kvh, :].T / np.sqrt(hd)          # [n, P]
        s = np.where(mask, s, -np.inf)
        out[:, h, :] = softmax(s) @ V[:, kvh, :]
    return out


def silu(x: np.ndarray) -> np.ndarray:
    """SiLU(x) = x * sigmoid(x)."""
    return x / (1.0 + np.exp(-x))


def swiglu_mlp(h: np.ndarray, Wg: np.ndarray, Wu: np.ndarray, Wd: np.ndarray) -> np.ndarray:
    """(silu(h Wg^T) * (h Wu^T)) Wd^T  with HF weight layout W[out, in]."""
    return (silu(h @ Wg.T) * (h @ Wu.T)) @ Wd.T


# ----------------------------------------------------------------------------- weights

def tensor_names(cfg: ModelConfig, layer: int) -> dict:
    p = f"model.layers.{layer}."
    return {
        "ln1": p + "input_layernorm.weight",
        "wq": p + "self_attn.q_proj.weight",
        "wk": p + "self_attn.k_proj.weight",
        "wv": p + "self_attn.v_proj.weight",
        "bq": p + "self_attn.q_proj.bias",
        "bk": p + "self_attn.k_proj.bias",
        "bv": p + "self_attn.v_proj.bias",
        "wo": p + "self_attn.o_proj.weight",
        "ln2": p + "post_attention_layernorm.weight",
        "wg": p + "mlp.gate_proj.weight",
        "wu": p + "mlp.up_proj.weight",
        "wd": p + "mlp.down_proj.weight",
    }


@dataclass
class Weights:
    """Lazily generated fp64 (bf16-exact) weights of one model."""
    cfg: ModelConfig
    seed: int = 0
    cache_layers: bool = True
    _layers: dict = field(default_factory=dict)
    _embed_rows: dict = field(default_factory=dict)
    _head: np.ndarray | None = None
    _final_norm: np.ndarray | None = None

    def layer(self, l: int) -> dict:
        if l in self._layers:
            return self._layers[l]
        c = self.cfg
        nm = tensor_names(c, l)
        d, hd = c.d_model, c.head_dim
        w = {
            "ln1": gen.gen_tensor(self.seed, nm["ln1"], "norm", (d,)),
            "wq": gen.gen_tensor(self.seed, nm["wq"], "linear", (c.n_heads * hd, d), fan_in=d),
            "wk": gen.gen_tensor(self.seed, nm["wk"], "linear", (c.n_kv_heads * hd, d), fan_in=d),
            "wv": gen.gen_tensor(self.seed, nm["wv"], "linear", (c.n_kv_heads * hd, d), fan_in=d),
            "wo": gen.gen_tensor(self.seed, nm["wo"], "linear", (d, c.n_heads * hd),
                                 fan_in=c.n_heads * hd),
            "ln2": gen.gen_tensor(self.seed, nm["ln2"], "norm", (d,)),
            "wg": gen.gen_tensor(self.seed, nm["wg"], "linear", (c.ffn_dim, d), fan_in=d),
            "wu": gen.gen_tensor(self.seed, nm["wu"], "linear", (c.ffn_dim, d), fan_in=d),
            "wd": gen.gen_tensor(self.seed, nm["wd"], "linear", (d, c.ffn_dim), fan_in=c.ffn_dim),
        }
        if c.qkv_bias:
            w["bq"] = gen.gen_tensor(self.seed, nm["bq"], "bias", (c.n_heads * hd,))
            w["bk"] = gen.gen_tensor(self.seed, nm["bk"], "bias", (c.n_kv_heads * hd,))
            w["bv"] = gen.gen_tensor(self.seed, nm["bv"], "bias", (c.n_kv_heads * hd,))
        if self.cache_layers:
            self._layers[l] = w
        return w

    def embed(self, tokens) -> np.ndarray:
        """Rows E[tok] of model.embed_tokens.weight [V, d] (generated row by row)."""
        c = self.cfg
        out = np.empty((len(tokens), c.d_model))
        for i, t in enumerate(tokens):
            t = int(t)
            if t not in self._embed_rows:
                self._embed_rows[t] = gen.gen_tensor(self.seed, "model.embed_tokens.weight",
                                                     "embed", (c.vocab, c.d_model),
                                                     row_start=t, row_end=t + 1)[0]
            out[i] = self._embed_rows[t]
        return out

    def final_norm(self) -> np.ndarray:
        if self._final_norm is None:
            self._final_norm = gen.gen_tensor(self.seed, "model.norm.weight", "norm",
                                              (self.cfg.d_model,))
        return self._final_norm

    def head(self) -> np.ndarray:
        """lm_head.weight [V, d] (untied; reading s1)."""
        if self._head is None:
            c = self.cfg
            rows = []
            step = max(1, (1 << 24) // c.d_model)
            for r0 in range(0, c.vocab, step):
                rows.append(gen.gen_tensor(self.seed, "lm_head.weight", "linear",
                                           (c.vocab, c.d_model), fan_in=c.d_model,
                                           row_start=r0, row_end=min(c.vocab, r0 + step)))
            self._head = np.concatenate(rows, axis=0)
        return self._head


# ----------------------------------------------------------------------------- forward

def layer_qkv(cfg: ModelConfig, w: dict, h: np.ndarray, pos: np.ndarray):
    """q, k, v of normalised inputs h[n, d] at positions pos[n]; RoPE applied to q and k."""
    n = h.shape[0]
    q = h @ w["wq"].T
    k = h @ w["wk"].T
    v = h @ w["wv"].T
    if cfg.qkv_bias:
        q = q + w["bq"]
        k = k + w["bk"]
        v = v + w["bv"]
    q = q.reshape(n, cfg.n_heads, cfg.head_dim)
    k = k.reshape(n, cfg.n_kv_heads, cfg.head_dim)
    v = v.reshape(n, cfg.n_kv_heads, cfg.head_dim)
    return apply_rope(q, pos, cfg.rope_theta), apply_rope(k, pos, cfg.rope_theta), v


def logits_of(cfg: ModelConfig, W: Weights, x_last: np.ndarray) -> np.ndarray:
    """logits = RMSNorm(x) * g_f  @  W_lm^T   for rows x_last[r, d]."""
    return rms_norm(x_last, W.final_norm(), cfg.rms_eps) @ W.head().T
