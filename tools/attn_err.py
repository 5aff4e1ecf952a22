"""Attention numerics report: worst row-relative error of qos_op_attention (fp32 output) vs the
fp64 oracle on the ATTN_CASES of tests/test_gpu_ops.py, split into prefill and decode rows.

  python tools/attn_err.py
"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.join(ROOT, "tests"))

import numpy as np  # noqa: E402

from helpers import bf16_bits, bits_to_f64, f16_bits, f16_bits_to_f64, make_engine, row_rel_err  # noqa: E402
from test_gpu_ops import ATTN_CASES  # noqa: E402
from oracle.model import causal_attention  # noqa: E402

for case, (preset, over, chunks, ctxs, scale) in enumerate(ATTN_CASES):
    q, cfg, eng = make_engine(preset, **{"max_seq_len": 8192, **over})
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
    npre = sum(n for _, n in chunks)
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
    out = eng.qos_op_attention(0, b, bf16_bits(np.concatenate(qrows)))
    ref = np.concatenate(refs)
    ep = row_rel_err(out[:npre].reshape(-1, hd), ref[:npre].reshape(-1, hd))
    ed = row_rel_err(out[npre:].reshape(-1, hd), ref[npre:].reshape(-1, hd))
    print(f"case {case} {preset} scale {scale}: prefill {ep:.2e}  decode {ed:.2e}", flush=True)
    eng.close()
