"""Seeded synthetic inputs shared by the oracle runs and the CUDA runs.

This module holds NO arithmetic of the method (no norm, attention, GEMM, RoPE, ...): only the
recipes that decide *which* requests, tokens, lengths and batches are fed to both sides
(DESIGN.md §3 "input recipe").  Seeds follow SURVEY.md §8(d): weights 0, tokens 1, KV fill 2,
ctx draws 3, arrivals 4.

Workload shapes come from the paper: chunked prefill + co-located decodes,
Table 2 prompt/decode token percentiles, Poisson arrivals
(PAPER.md:1008-1010), three equal QoS thirds (Table 3 1039-1048).
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

SEED_WEIGHTS = 0
SEED_TOKENS = 1
SEED_KVFILL = 2
SEED_CTX = 3
SEED_ARRIVALS = 4

_M64 = (1 << 64) - 1


def _mix(z: np.ndarray) -> np.ndarray:
    # splitmix64 finaliser, used here purely as a seeded integer source for token ids
    z = z + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def request_tokens(req: int, n: int, vocab: int, seed: int = SEED_TOKENS, start: int = 0) -> np.ndarray:
    """Token ids of request ``req`` at positions [start, start+n): uniform in [0, vocab)."""
    base = np.uint64(((seed * 0x9E3779B97F4A7C15) ^ (int(req) * 0xD1B54A32D192ED03)) & _M64)
    pos = np.arange(start, start + n, dtype=np.uint64)
    return (_mix(pos + base) % np.uint64(vocab)).astype(np.int32)


@dataclass
class Chunk:
    req: int
    kv_start: int
    tokens: np.ndarray           # int32 [chunk_len]

    @property
    def chunk_len(self) -> int:
        return int(len(self.tokens))


@dataclass
class Decode:
    req: int
    ctx_len: int
    token: int


@dataclass
class Batch:
    prefill: list = field(default_factory=list)   # [Chunk]
    decode: list = field(default_factory=list)    # [Decode]

    @property
    def n_tokens(self) -> int:
        return sum(c.chunk_len for c in self.prefill) + len(self.decode)

    def as_oracle(self):
        return ([(c.req, c.kv_start, [int(t) for t in c.tokens]) for c in self.prefill],
                [(d.req, d.ctx_len, int(d.token)) for d in self.decode])


def split_prompt(req: int, prompt_len: int, chunk_sizes, vocab: int, seed: int = SEED_TOKENS):
    """Chunks that prefill positions [0, prompt_len) of ``req`` with a cycling list of chunk
    sizes (exercises arbitrary chunk splits)."""
    toks = request_tokens(req, prompt_len, vocab, seed)
    out, s, i = [], 0, 0
    while s < prompt_len:
        n = min(int(chunk_sizes[i % len(chunk_sizes)]), prompt_len - s)
        out.append(Chunk(req, s, toks[s:s + n]))
        s += n
        i += 1
    return out


def tiny_scenario(vocab: int):
    """configs[0]: one 128-token prefill chunk + 4 decodes (ctx <= 512).

    Returns (warm_steps, main_batch, second_batch):
      * warm_steps — batches that prefill the 4 decode requests' prompts (ctx {37, 200, 311,
        512}) in chunks cycling over {64, 100, 128}, several requests per step;
      * main_batch  — req 0 chunk (kv_start 0, len 128) + the 4 decodes at position ctx;
      * second_batch — req 0 chunk (kv_start 128, len 128) + decodes at ctx+1 (paged prefix).
    """
    ctxs = {1: 37, 2: 200, 3: 311, 4: 512}
    per_req = {r: split_prompt(r, n, (64, 100, 128), vocab) for r, n in ctxs.items()}
    warm = []
    k = 0
    while any(per_req.values()):
        b = Batch()
        for r in sorted(per_req):
            if per_req[r]:
                b.prefill.append(per_req[r].pop(0))
        warm.append(b)
        k += 1
    t0 = request_tokens(0, 256, vocab)
    main = Batch([Chunk(0, 0, t0[:128])],
                 [Decode(r, n, int(request_tokens(r, 1, vocab, start=n)[0])) for r, n in ctxs.items()])
    second = Batch([Chunk(0, 128, t0[128:256])],
                   [Decode(r, n + 1, int(request_tokens(r, 1, vocab, start=n + 1)[0]))
                    for r, n in ctxs.items()])
    return ctxs, warm, main, second


def ctx_draw(n: int, lo: int, hi: int, seed: int = SEED_CTX, kind: str = "uniform") -> np.ndarray:
    """Decode context lengths: uniform on [lo, hi] or log-uniform (70B config)."""
    rng = np.random.default_rng(seed)
    if kind == "uniform":
        return rng.integers(lo, hi + 1, size=n).astype(np.int64)
    if kind == "loguniform":
        return np.exp(rng.uniform(np.log(lo), np.log(hi), size=n)).astype(np.int64)
    raise ValueError(kind)


def hybrid_batch(vocab: int, chunk_len: int, n_decode: int, ctx, kv_start: int = 0,
                 chunk_req: int = 0, first_decode_req: int = 1, seed: int = SEED_TOKENS) -> Batch:
    """One hybrid step: a prefill chunk of ``chunk_len`` tokens at ``kv_start`` + ``n_decode``
    decodes with context lengths ``ctx`` (int or sequence).  The decodes' prefixes are
    expected to be cached (KV-fill or earlier prefills)."""
    ctx = [int(ctx)] * n_decode if np.isscalar(ctx) else [int(c) for c in ctx]
    b = Batch()
    if chunk_len > 0:
        b.prefill.append(Chunk(chunk_req, kv_start,
                               request_tokens(chunk_req, chunk_len, vocab, seed, start=kv_start)))
    for j in range(n_decode):
        r = first_decode_req + j
        b.decode.append(Decode(r, ctx[j], int(request_tokens(r, 1, vocab, seed, start=ctx[j])[0])))
    return b


# Table 2 p50 / p90 token counts -> lognormal (mu, sigma) fitted to them
# ("po0" read as p90).
LOGNORMAL = {
    "azure_code": {"prompt": (7.565, 0.917), "decode": (2.079, 1.312)},
    "azure_conv": {"prompt": (6.833, 1.106), "decode": (3.714, 1.655)},
}


# fixed-length synthetic workloads: (prompt tokens, decode tokens) of every request
FIXED = {"long_10k": (10_000, 500)}   # the paper's Medha comparison trace


def trace(qps: float, duration_s: float, dataset: str = "azure_conv", seed: int = SEED_ARRIVALS,
          low_priority_frac: float = 0.2, max_total: int = 8192):
    """Synthetic request stream shaped like the paper's workloads: Poisson arrivals at `qps`
    (PAPER.md:1008-1010), prompt / decode lengths lognormal fitted to Table 2,
    three equal QoS thirds Q1/Q2/Q3 (Table 3), a `low_priority_frac` share of
    free-tier requests, prompt + decode <= max_total (Llama-3-8B window).
    Returns a list of dicts (pure data; the scheduler builds its Request objects from them)."""
    rng = np.random.default_rng(seed)
    fixed = FIXED.get(dataset)
    if fixed is None:
        mu_p, sg_p = LOGNORMAL[dataset]["prompt"]
        mu_d, sg_d = LOGNORMAL[dataset]["decode"]
    t, out, i = 0.0, [], 0
    while True:
        t += rng.exponential(1.0 / qps)
        if t > duration_s:
            break
        if fixed is not None:   # fixed lengths; the window check does not apply (max_total unused)
            p, d = fixed
        else:
            p = int(np.clip(np.exp(rng.normal(mu_p, sg_p)), 16, max_total - 16))
            d = int(np.clip(np.exp(rng.normal(mu_d, sg_d)), 1, max_total - p))
        tier = ("Q1", "Q2", "Q3")[int(rng.integers(0, 3))]
        out.append({"req_id": i, "t_arrival": t, "prompt_len": p, "decode_len": d, "tier": tier,
                    "app_id": f"{dataset}-{tier}", "important": bool(rng.random() >= low_priority_frac)})
        i += 1
    return out
