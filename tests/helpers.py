"""Shared test helpers (no method arithmetic): tolerance metric of reading s9, bf16 packing of
host inputs, engine construction."""
from __future__ import annotations

import numpy as np

# Tolerances of BASELINE.json:north_star, metric of reading s9:
# per row max_i |g_i - o_i| / max_i |o_i|, max over rows.
TOL_LOGITS = 1e-2
TOL_ATTN = 2e-3


def row_rel_err(got: np.ndarray, ref: np.ndarray) -> float:
    got = np.asarray(got, dtype=np.float64).reshape(-1, np.shape(ref)[-1])
    ref = np.asarray(ref, dtype=np.float64).reshape(-1, np.shape(ref)[-1])
    den = np.maximum(np.abs(ref).max(axis=1), 1e-300)
    return float(np.max(np.abs(got - ref).max(axis=1) / den))


def bf16_bits(x: np.ndarray) -> np.ndarray:
    """fp64/fp32 values -> bf16 bits (RNE via fp32)."""
    u = np.ascontiguousarray(np.asarray(x, dtype=np.float32)).view(np.uint32).astype(np.uint64)
    u = u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))
    return (u >> np.uint64(16)).astype(np.uint16)


def bits_to_f64(b: np.ndarray) -> np.ndarray:
    return (np.asarray(b, dtype=np.uint16).astype(np.uint32) << np.uint32(16)).view(np.float32).astype(np.float64)


def f16_bits(x: np.ndarray) -> np.ndarray:
    """fp64/fp32 values -> IEEE fp16 bits (RNE via fp32; the cached V format, reading r-v16)."""
    return np.ascontiguousarray(np.asarray(x, dtype=np.float32)).astype(np.float16).view(np.uint16)


def f16_bits_to_f64(b: np.ndarray) -> np.ndarray:
    return np.ascontiguousarray(b, dtype=np.uint16).view(np.float16).astype(np.float64)


def make_engine(preset_name: str, **over):
    from paper_conf_asplos_goelmkar26_b200 import qoserve as q
    from paper_conf_asplos_goelmkar26_b200.presets import preset
    caps = dict(num_blocks=1024, max_seq_len=4096, max_requests=64, max_batch_tokens=1024, max_batch_rows=32)
    model_over = {k: v for k, v in over.items() if k not in caps}
    caps.update({k: v for k, v in over.items() if k in caps})
    cfg = q.model_cfg(**preset(preset_name, **model_over), **caps)
    return q, cfg, q.Engine(cfg)
