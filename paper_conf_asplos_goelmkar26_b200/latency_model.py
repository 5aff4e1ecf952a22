"""Iteration-time model of the hybrid step for QoServe's dynamic chunking.

The paper predicts batch latency with a random forest trained on Vidur's per-op profiles and
uses it to pick the largest chunk that keeps every decode's next-token deadline
(GET_PREFILL_BUDGET, Alg. 1 line 7 = PAPER.md:760; §3.6.1; "<10% error",
"err on the side of under-predicting" PAPER.md:941-944).  Here the model is fitted to the
engine's OWN device-timed steps (`qos_profile_step`), with features taken from the step's
roofline work:

    t(batch) = G(T) + a * Bdec + b * Fpre + c

* G(T): piecewise-linear in T = sum(chunk_len) + n_decode (hat basis on knots) — the dense
  projections, norms, RoPE/append, LM head (their cost depends on T only, with the GEMM tile
  steps of 128 rows);
* Bdec = sum_j (ctx_j + 1): decode-attention KV bytes are proportional (HBM-bound);
* Fpre = sum_c [len_c * kv_start_c + len_c (len_c + 1) / 2]: prefill-attention work.

Least squares (numpy) over profiled points; `predict` is pure host arithmetic.  The north
star asks iteration latency to be predictable within 5% across chunk sizes 256-8192.
"""
from __future__ import annotations

import json
from dataclasses import dataclass, field

import numpy as np

KNOTS = (1, 64, 128, 256, 512, 768, 1024, 1536, 2048, 3072, 4096, 5120, 6144, 7168, 8192, 8448)


@dataclass
class StepShape:
    chunks: list = field(default_factory=list)   # [(kv_start, chunk_len)]
    ctx: list = field(default_factory=list)      # decode context lengths

    @property
    def T(self) -> int:
        return sum(n for _, n in self.chunks) + len(self.ctx)


def features(s: StepShape, knots=KNOTS) -> np.ndarray:
    T = s.T
    k = np.asarray(knots, dtype=np.float64)
    hat = np.zeros(len(k))
    if T <= k[0]:
        hat[0] = 1.0
    elif T >= k[-1]:
        hat[-1] = 1.0
    else:
        i = int(np.searchsorted(k, T) - 1)
        w = (T - k[i]) / (k[i + 1] - k[i])
        hat[i], hat[i + 1] = 1 - w, w
    bdec = float(sum(c + 1 for c in s.ctx)) / 1e6
    fpre = float(sum(n * ks + n * (n + 1) / 2 for ks, n in s.chunks)) / 1e7
    return np.concatenate([hat, [bdec, fpre]])


class LatencyModel:
    def __init__(self, knots=KNOTS):
        self.knots = tuple(knots)
        self.coef = None

    def fit(self, shapes, ms):
        X = np.stack([features(s, self.knots) for s in shapes])
        y = np.asarray(ms, dtype=np.float64)
        # relative least squares (weights 1/y) so every chunk size counts the same
        w = 1.0 / y
        # only knots that carry weight enter the fit; the rest interpolate to neighbours
        used = X[:, :len(self.knots)].sum(0) > 0
        cols = np.concatenate([used, [True, True]])
        coef, *_ = np.linalg.lstsq(X[:, cols] * w[:, None], y * w, rcond=None)
        full = np.zeros(X.shape[1])
        full[cols] = coef
        # fill unused knots by linear interpolation between used ones
        kx = np.asarray(self.knots, dtype=np.float64)
        ui = np.where(used)[0]
        if len(ui) >= 2:
            full[:len(kx)] = np.interp(kx, kx[ui], full[ui])
        self.coef = full
        return self

    def predict(self, s: StepShape) -> float:
        return float(features(s, self.knots) @ self.coef)

    def max_chunk(self, budget_ms: float, ctx, kv_start: int = 0, lo: int = 256, hi: int = 8192,
                  step: int = 256, margin: float = 0.05) -> int:
        """Largest chunk on the grid whose predicted step time fits budget*(1-margin); 0 if
        none (a decode-only step).  The margin under-predicts chunk size."""
        best = 0
        for c in range(lo, hi + 1, step):
            if self.predict(StepShape([(kv_start, c)], list(ctx))) <= budget_ms * (1 - margin):
                best = c
        return best

    def to_json(self) -> str:
        return json.dumps({"knots": list(self.knots), "coef": [float(x) for x in self.coef]})

    @classmethod
    def from_json(cls, s: str) -> "LatencyModel":
        d = json.loads(s)
        m = cls(d["knots"])
        m.coef = np.asarray(d["coef"])
        return m
