"""OracleEngine: the plain fp64 definition of a QoServe hybrid step (test infrastructure only).

Semantics replayed from the C ABI (include/qoserve.h):

* a step = all decodes + prefill chunk(s) selected by the scheduler (§3.1
  step 1; Alg. 1 lines 2, 17-20 = PAPER.md:755, 770-773), run as one fused token batch
  (§3.3).  The oracle runs every request on its own — the plain definition
  that the fused, chunked, paged GPU batch must reproduce.
* a prefill chunk {req, kv_start, tokens} processes positions kv_start .. kv_start+len-1,
  attending to the request's cached prefix plus itself (causal);  kv_start must equal the
  cached length (strict append).  One logits row per chunk: its last token (reading s8).
* a decode {req, ctx_len, token} processes one token at position ctx_len over ctx_len+1 keys
  (reading s7).  Decodes are never preempted.
* output rows: chunks in descriptor order, then decodes in descriptor order.
* KV blocks: own allocator (oracle.kv), same policy; tables must match the GPU's bit-exactly.
"""
from __future__ import annotations

import numpy as np

from . import gen
from .kv import BlockAllocator
from .model import (ModelConfig, Weights, causal_attention, layer_qkv, logits_of, rms_norm,
                    swiglu_mlp)


class OracleBadKVStart(Exception):
    pass


class OracleNotAllocated(Exception):
    pass


class OracleEngine:
    def __init__(self, cfg: ModelConfig, seed: int = 0, num_blocks: int = 4096,
                 cache_layers: bool = True):
        self.cfg = cfg
        self.W = Weights(cfg, seed=seed, cache_layers=cache_layers)
        self.alloc = BlockAllocator(num_blocks, cfg.block_size)
        # per request: list over layers of (K[P, Hkv, hd], V[P, Hkv, hd]) in fp64
        self.kv: dict[int, list] = {}

    # ------------------------------------------------------------------ KV management
    def kv_alloc(self, req: int, n_tokens_total: int) -> None:
        self.alloc.alloc(req, n_tokens_total)

    def kv_free(self, req: int) -> None:
        self.alloc.free(req)
        self.kv.pop(req, None)

    def kv_table(self, req: int) -> list[int]:
        return self.alloc.table(req)

    def cached_len(self, req: int) -> int:
        st = self.kv.get(req)
        return 0 if st is None else st[0][0].shape[0]

    def kv_fill_synthetic(self, req: int, n_tokens: int, seed: int) -> None:
        """Cache positions [0, n_tokens) of ``req`` with the synthetic KV of oracle.gen
        (used at bench sizes where the prefix is not produced by a prefill)."""
        self._check_alloc(req, n_tokens)
        c = self.cfg
        self.kv[req] = [
            (gen.kvfill_rows(seed, l, "k", req, 0, n_tokens, c.n_kv_heads, c.head_dim),
             gen.kvfill_rows(seed, l, "v", req, 0, n_tokens, c.n_kv_heads, c.head_dim))
            for l in range(c.n_layers)]

    def _check_alloc(self, req: int, n_tokens: int) -> None:
        have = len(self.alloc.tables.get(req, []))
        if have * self.cfg.block_size < n_tokens:
            raise OracleNotAllocated(f"req {req}: {have} blocks < {n_tokens} tokens")

    # ------------------------------------------------------------------ forward
    def forward_run(self, req: int, tokens, start: int, record: dict | None = None) -> np.ndarray:
        """Plain causal forward of tokens at positions start.. of one request; appends its
        K/V to the request's cache and returns the final residual stream x[n, d]."""
        c = self.cfg
        if self.cached_len(req) != start:
            raise OracleBadKVStart(f"req {req}: cached {self.cached_len(req)} != start {start}")
        self._check_alloc(req, start + len(tokens))
        n = len(tokens)
        pos = start + np.arange(n)
        x = self.W.embed(tokens)
        if req not in self.kv:
            z = np.zeros((0, c.n_kv_heads, c.head_dim))
            self.kv[req] = [(z, z) for _ in range(c.n_layers)]
        group = c.n_heads // c.n_kv_heads
        for l in range(c.n_layers):
            w = self.W.layer(l)
            h = rms_norm(x, w["ln1"], c.rms_eps)
            q, k, v = layer_qkv(c, w, h, pos)
            K, V = self.kv[req][l]
            K = np.concatenate([K, k], axis=0)
            V = np.concatenate([V, v], axis=0)
            self.kv[req][l] = (K, V)
            o = causal_attention(q, K, V, start, group)
            if record is not None:
                record.setdefault("q", []).append(q)
                record.setdefault("attn", []).append(o)
            x = x + o.reshape(n, c.n_heads * c.head_dim) @ w["wo"].T
            h2 = rms_norm(x, w["ln2"], c.rms_eps)
            x = x + swiglu_mlp(h2, w["wg"], w["wu"], w["wd"])
        return x

    def hybrid_step(self, prefill, decode) -> np.ndarray:
        """prefill: list of (req, kv_start, tokens); decode: list of (req, ctx_len, token).
        Returns fp64 logits [n_prefill + n_decode, V]."""
        reqs = [p[0] for p in prefill] + [d[0] for d in decode]
        if len(set(reqs)) != len(reqs):
            raise ValueError("a request appears twice in one step")
        last = []
        for req, kv_start, tokens in prefill:
            x = self.forward_run(req, list(tokens), kv_start)
            last.append(x[-1])
        for req, ctx_len, token in decode:
            x = self.forward_run(req, [token], ctx_len)
            last.append(x[-1])
        if not last:
            return np.zeros((0, self.cfg.vocab))
        return logits_of(self.cfg, self.W, np.stack(last))

    def hybrid_step_layer_major(self, prefill, decode) -> np.ndarray:
        """hybrid_step with the loops exchanged: layer by layer, every request of the step
        through that layer (each layer's weights are needed once, not once per request — the
        form that makes full-depth bench-size checks affordable).  Per request the operations
        and their order are exactly forward_run's, so the result is identical (pinned in
        tests/test_oracle_model.py)."""
        c = self.cfg
        runs = [(req, list(tokens), kv_start) for req, kv_start, tokens in prefill] + \
               [(req, [token], ctx_len) for req, ctx_len, token in decode]
        reqs = [r[0] for r in runs]
        if len(set(reqs)) != len(reqs):
            raise ValueError("a request appears twice in one step")
        if not runs:
            return np.zeros((0, c.vocab))
        xs, poss = [], []
        for req, tokens, start in runs:
            if self.cached_len(req) != start:
                raise OracleBadKVStart(f"req {req}: cached {self.cached_len(req)} != start {start}")
            self._check_alloc(req, start + len(tokens))
            if req not in self.kv:
                z = np.zeros((0, c.n_kv_heads, c.head_dim))
                self.kv[req] = [(z, z) for _ in range(c.n_layers)]
            xs.append(self.W.embed(tokens))
            poss.append(start + np.arange(len(tokens)))
        group = c.n_heads // c.n_kv_heads
        for l in range(c.n_layers):
            w = self.W.layer(l)
            for i, (req, tokens, start) in enumerate(runs):
                x, n = xs[i], len(tokens)
                h = rms_norm(x, w["ln1"], c.rms_eps)
                q, k, v = layer_qkv(c, w, h, poss[i])
                K, V = self.kv[req][l]
                K = np.concatenate([K, k], axis=0)
                V = np.concatenate([V, v], axis=0)
                self.kv[req][l] = (K, V)
                o = causal_attention(q, K, V, start, group)
                x = x + o.reshape(n, c.n_heads * c.head_dim) @ w["wo"].T
                h2 = rms_norm(x, w["ln2"], c.rms_eps)
                xs[i] = x + swiglu_mlp(h2, w["wg"], w["wu"], w["wd"])
        return logits_of(c, self.W, np.stack([x[-1] for x in xs]))


def greedy(logits: np.ndarray) -> np.ndarray:
    """Greedy argmax per row, lowest index on ties (reading s11; np.argmax returns the first
    maximal index)."""
    return np.argmax(logits, axis=-1).astype(np.int64)
