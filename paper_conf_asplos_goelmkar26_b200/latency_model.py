"""Iteration-time model of the hybrid step for QoServe's dynamic chunking.

The paper predicts batch latency with a random forest trained on Vidur's per-op profiles and
uses it to pick the largest chunk that keeps every decode's next-token deadline
(GET_PREFILL_BUDGET, Alg. 1 line 7 = PAPER.md:760; §3.6.1; "<10% error",
"err on the side of under-predicting" PAPER.md:941-944).  Here the model is fitted to the
engine's OWN device-timed steps (`qos_profile_step`) with features that follow the step's
work and the engine's tiling:

    t(batch) = c0 * Wgemm(T) + c1 * T + c2 * Bdec + c3 * n_dec + c4 * [n_dec > 0] + c5 + c6 * Fdiag
               + c7 * Wstream(T) + c8 * Fprefix + c9 * Wpair(T) + c10 * Npair(T) + c11 * Ntile(T)

* Wgemm(T): sum over the projections run by the single-CTA tile kernel (csrc/gemm.cu) of (waves
  of 128 x BN tiles over the SMs) x (k-blocks per tile) x BN/256 — the tensor-core GEMM time
  with the engine's tile-quantisation (same BN choice), T = sum(chunk_len) + n_decode; the O
  and down projections below the fold threshold enter with the cost of the engine's ordered
  split-K choice (`add_split`, mirroring gemm_pick_add_split) in the same units;
* Wpair(T): the same for the projections run by the CTA-pair kernel (256 x 256 tiles over 2
  SMs, same selection rule as gemm2_eligible): (waves of pair tiles over SMs/2) x k-blocks —
  a separate term because its per-k-block cost differs;
* Npair(T), Ntile(T): how many of the 4 projections run on the pair / single-CTA tile kernel
  (per-launch prologue, pipeline fill and exposed last-wave epilogue, x L layers);
* Wstream(T): weight elements N*K of the projections run by the weight-streaming kernel
  (csrc/gemm_swab.cu, same selection rule as swab_prefer) — HBM-bound;
* T: per-token elementwise work (norms, RoPE/append, embedding);
* Bdec = sum_j (ctx_j + 1): decode-attention KV bytes (HBM-bound);
* n_dec and [n_dec > 0]: per-decode and per-launch latency of the split-K decode attention;
* Fdiag = sum_c len_c (len_c + 1) / 2 and Fprefix = sum_c len_c * kv_start_c: prefill-attention
  work on the chunk's own (causal, masked diagonal tiles) and on its cached prefix (unmasked
  tiles, measured ~1.6x more efficient per FLOP on B200) — kept apart, as their costs differ.

Least squares (numpy, relative weights) over profiled points; `predict` is host arithmetic.
The north star asks iteration latency to be predictable within 5% across chunks 256-8192.
"""
from __future__ import annotations

import json
import math
from dataclasses import dataclass, field

import numpy as np

N_FEAT = 14
FOLD_MIN_TOKENS = 1536   # kFoldMinTokens (csrc/internal.h)


@dataclass
class StepShape:
    chunks: list = field(default_factory=list)   # [(kv_start, chunk_len)]
    ctx: list = field(default_factory=list)      # decode context lengths

    @property
    def T(self) -> int:
        return sum(n for _, n in self.chunks) + len(self.ctx)


@dataclass(frozen=True)
class GemmShapes:
    """(N, K) of the QKV, O, gate/up and down projections of one TP rank + the SM count."""
    gemms: tuple = ((6144, 4096), (4096, 4096), (28672, 4096), (4096, 14336))
    num_sms: int = 148

    @staticmethod
    def for_model(d_model, n_heads, n_kv_heads, head_dim, ffn_dim, tp=1, num_sms=148):
        nqkv = (n_heads + 2 * n_kv_heads) // tp * head_dim
        return GemmShapes(((nqkv, d_model), (d_model, n_heads // tp * head_dim), (2 * ffn_dim // tp, d_model),
                           (d_model, ffn_dim // tp)), num_sms)


def _bn(M: int, N: int, sms: int) -> int:      # mirrors gemm_pick_bn (csrc/gemm.cu)
    if N % 256:
        return 128
    mt = (M + 127) // 128
    w128 = -(-(mt * (N // 128)) // sms)
    w256 = -(-(mt * (N // 256)) // sms)
    return 256 if w256 * 630 < w128 * 445 else 128


def swab_prefer(M: int, N: int, sms: int) -> bool:   # mirrors swab_prefer (csrc/gemm_swab.cu)
    if N % 128:
        return False
    if M <= 64:
        return True
    if M > 256:
        return False
    return ((M + 127) // 128) * (N // 128) * 4 < sms


def swab_prefer_k(M: int, N: int, K: int, sms: int) -> bool:   # mirrors swab_prefer_k (csrc/gemm_swab.cu)
    if swab_prefer(M, N, sms):
        return True
    if N % 128 or M > 128 or K < 8192:
        return False
    return ((M + 127) // 128) * (N // 128) * 2 < sms


def pair_eligible(M: int, N: int, K: int, sms: int) -> bool:   # mirrors gemm2_eligible (csrc/gemm.cu)
    if N % 256 or K % 64:
        return False
    t1 = ((M + 127) // 128) * (N // 256)
    t2 = ((M + 255) // 256) * (N // 256)
    if t1 < sms:
        return False
    return -(-t2 // (sms // 2)) <= -(-t1 // sms)


def pair_work(T: int, g: GemmShapes) -> float:
    return float(sum(-(-(((T + 255) // 256) * (N // 256)) // (g.num_sms // 2)) * (K // 64)
                     for N, K in g.gemms if T > 0 and pair_eligible(T, N, K, g.num_sms)))


def add_split(M: int, N: int, K: int, sms: int, max_tiles: int = 4096):
    """(BN, slices, cost in cycles) of an EPI_ADD_F32 projection; mirrors gemm_pick_add_split
    (csrc/gemm.cu): waves x k-blocks per unit x c(BN) + (slices - 1) x E(BN)."""
    mt, kb = (M + 127) // 128, K // 64
    best = best1 = None
    for bn in (128, 256):
        if bn == 256 and N % 256:
            continue
        tiles = mt * ((N + bn - 1) // bn)
        ckb, epi = (687, 8500) if bn == 256 else (403, 5600)
        for ks in (1, 2, 3, 4):
            if ks > 1 and (kb < 128 or kb // ks < 8 or tiles > max_tiles):
                break
            cost = -(-tiles * ks // sms) * (-(-kb // ks)) * ckb + (ks - 1) * epi
            if ks == 1 and (best1 is None or cost < best1[2]):
                best1 = (bn, 1, cost)
            if best is None or cost < best[2]:
                best = (bn, ks, cost)
    return best if best[1] > 1 and best[2] * 100 <= best1[2] * 85 else best1


# the projections with the residual-add epilogue (O and down): ordered split-K below the fold
ADD_GEMMS = (1, 3)


def gemm_work(T: int, g: GemmShapes, fold: bool = False) -> float:
    if T <= 0:
        return 0.0
    tot = 0.0
    for i, (N, K) in enumerate(g.gemms):
        if swab_prefer_k(T, N, K, g.num_sms) or pair_eligible(T, N, K, g.num_sms):
            continue
        if i in ADD_GEMMS and not fold:
            tot += add_split(T, N, K, g.num_sms)[2] / 630.0
            continue
        bn = _bn(T, N, g.num_sms)
        tiles = ((T + 127) // 128) * ((N + bn - 1) // bn)   # whole tiles
        tot += math.ceil(tiles / g.num_sms) * (K // 64) * (bn / 256)
    return tot


def stream_work(T: int, g: GemmShapes) -> float:
    return float(sum(N * K for N, K in g.gemms if T > 0 and swab_prefer_k(T, N, K, g.num_sms)))


def features(s: StepShape, g: GemmShapes = GemmShapes()) -> np.ndarray:
    nd = len(s.ctx)
    n_pair = sum(1 for N, K in g.gemms if s.T > 0 and pair_eligible(s.T, N, K, g.num_sms))
    n_stream = sum(1 for N, K in g.gemms if s.T > 0 and swab_prefer_k(s.T, N, K, g.num_sms))
    fold = 1.0 if (s.T >= FOLD_MIN_TOKENS and n_stream == 0) else 0.0   # mirrors run_layers' norm fold
    return np.array([gemm_work(s.T, g, fold > 0) / 100.0, s.T / 1000.0, sum(c + 1 for c in s.ctx) / 1e6, nd / 100.0,
                     1.0 if nd else 0.0, 1.0, sum(n * (n + 1) / 2 for ks, n in s.chunks) / 1e7,
                     stream_work(s.T, g) / 1e8, sum(n * ks for ks, n in s.chunks) / 1e7, pair_work(s.T, g) / 100.0,
                     float(n_pair), float(len(g.gemms) - n_pair - n_stream), fold, fold * s.T / 1000.0])


class LatencyModel:
    def __init__(self, shapes: GemmShapes = GemmShapes()):
        self.shapes = shapes
        self.coef = None

    def fit(self, shapes, ms):
        X = np.stack([features(s, self.shapes) for s in shapes])
        y = np.asarray(ms, dtype=np.float64)
        w = 1.0 / y                         # relative least squares: every point counts alike
        self.coef, *_ = np.linalg.lstsq(X * w[:, None], y * w, rcond=None)
        return self

    def predict(self, s: StepShape) -> float:
        return float(features(s, self.shapes) @ self.coef)

    def to_json(self) -> str:
        return json.dumps({"gemms": [list(x) for x in self.shapes.gemms], "num_sms": self.shapes.num_sms,
                           "coef": [float(x) for x in self.coef]})

    @classmethod
    def from_json(cls, s: str) -> "LatencyModel":
        d = json.loads(s)
        m = cls(GemmShapes(tuple(tuple(x) for x in d["gemms"]), d["num_sms"]))
        m.coef = np.asarray(d["coef"])
        return m
