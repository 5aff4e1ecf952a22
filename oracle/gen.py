"""Synthetic-weight and synthetic-KV generator of the oracle (test infrastructure only).

The paper loads real checkpoints from Hugging Face (§A.3.5); there is no
network here, so both sides draw the SAME bf16 bits from a counter-based generator whose
*specification* is fixed in SURVEY.md §8(c) step 1 and DESIGN.md §3 ("weights"):

    z    = (seed XOR fnv1a64(tensor_name)) + i            (mod 2^64, i = flat row-major index)
    k    = splitmix64(z) >> 40                            (24-bit integer)
    a    = (k - 2^23) / 2^23                              (= 2u-1 with u = k/2^24; exact in fp32)
    linear  w = bf16_rne( fp32( a * fp32(1/sqrt(fan_in)) ) )
    embed   w = bf16_rne( a )
    norm    w = bf16_rne( fp32( 1 + fp32(0.1 * a) ) )
    bias    w = bf16_rne( fp32( 0.02 * a ) )
    kvfill  K: w = bf16_rne( a ),  V: w = fp16_rne( a )   (reading r-v16: the cache
            holds V in fp16)   name "kvfill.{layer}.{k|v}.{req}", i = (pos*Hkv + h)*hd + j

This module is an independent numpy implementation of that spec.  The CUDA library has its
own implementation (device kernel); the two are compared bit-for-bit on the generated bf16
bits (tests/test_gpu_weights.py).  Nothing here is shared
with the product path.
"""
from __future__ import annotations

import numpy as np

MASK64 = (1 << 64) - 1
FNV_OFFSET = 0xCBF29CE484222325
FNV_PRIME = 0x100000001B3


def fnv1a64(data: bytes) -> int:
    """FNV-1a 64-bit hash of a byte string (plain Python ints)."""
    h = FNV_OFFSET
    for b in data:
        h ^= b
        h = (h * FNV_PRIME) & MASK64
    return h


def splitmix64_np(z: np.ndarray) -> np.ndarray:
    """splitmix64 finaliser on a uint64 array (numpy uint64 arithmetic wraps mod 2^64)."""
    z = z + np.uint64(0x9E3779B97F4A7C15)
    z = (z ^ (z >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
    z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
    return z ^ (z >> np.uint64(31))


def splitmix64_int(z: int) -> int:
    """Scalar splitmix64 with Python ints (used to pin the vectorised version)."""
    z = (z + 0x9E3779B97F4A7C15) & MASK64
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31)


def bf16_rne_bits(x32: np.ndarray) -> np.ndarray:
    """Round fp32 values to bf16 (round-to-nearest-even); returns uint16 bit patterns."""
    u = np.ascontiguousarray(x32, dtype=np.float32).view(np.uint32).astype(np.uint64)
    u = u + np.uint64(0x7FFF) + ((u >> np.uint64(16)) & np.uint64(1))
    return (u >> np.uint64(16)).astype(np.uint16)


def f16_rne_bits(x32: np.ndarray) -> np.ndarray:
    """Round fp32 values to IEEE fp16 (round-to-nearest-even, numpy's conversion); uint16 bits."""
    return np.ascontiguousarray(x32, dtype=np.float32).astype(np.float16).view(np.uint16)


def f16_bits_to_f64(bits: np.ndarray) -> np.ndarray:
    """Exact widening of fp16 bit patterns to fp64."""
    return np.ascontiguousarray(bits, dtype=np.uint16).view(np.float16).astype(np.float64)


def bf16_bits_to_f64(bits: np.ndarray) -> np.ndarray:
    """Exact widening of bf16 bit patterns to fp64."""
    return (bits.astype(np.uint32) << np.uint32(16)).view(np.float32).astype(np.float64)


def f64_to_bf16_f64(x: np.ndarray) -> np.ndarray:
    """Round fp64 values to bf16 via fp32 (RNE at each step) and widen back (used only to
    build bf16-exact *inputs* for kernel-level tests)."""
    return bf16_bits_to_f64(bf16_rne_bits(np.asarray(x, dtype=np.float64).astype(np.float32)))


def _a_values(seed: int, name: str, start: int, count: int) -> np.ndarray:
    base = (int(seed) ^ fnv1a64(name.encode())) & MASK64
    idx = np.arange(start, start + count, dtype=np.uint64)
    z = idx + np.uint64(base)
    k = (splitmix64_np(z) >> np.uint64(40)).astype(np.int64)
    # a = (k - 2^23) / 2^23, exact in fp32 (24 significant bits)
    return ((k - (1 << 23)).astype(np.float32)) / np.float32(1 << 23)


def gen_bits(seed: int, name: str, kind: str, start: int, count: int, fan_in: int = 1) -> np.ndarray:
    """bf16 bit patterns of elements [start, start+count) of tensor ``name`` (fp16 bit patterns
    for kind "kvfill_v", the synthetic cached V)."""
    a = _a_values(seed, name, start, count)
    if kind == "kvfill_v":
        return f16_rne_bits(a)
    if kind == "linear":
        s = np.float32(1.0 / np.sqrt(np.float64(fan_in)))
        w = a * s                                   # fp32 multiply, RNE
    elif kind in ("embed", "kvfill"):
        w = a
    elif kind == "norm":
        w = np.float32(1.0) + np.float32(0.1) * a   # fp32 ops, RNE each
    elif kind == "bias":
        w = np.float32(0.02) * a
    else:
        raise ValueError(kind)
    return bf16_rne_bits(w.astype(np.float32))


def gen_tensor(seed: int, name: str, kind: str, shape, fan_in: int = 1,
               row_start: int = 0, row_end: int | None = None) -> np.ndarray:
    """fp64 array (exact bf16 values) of rows [row_start, row_end) of a row-major tensor."""
    shape = tuple(int(s) for s in shape)
    if len(shape) == 1:
        return bf16_bits_to_f64(gen_bits(seed, name, kind, 0, shape[0], fan_in))
    rows, cols = shape
    row_end = rows if row_end is None else row_end
    n = (row_end - row_start) * cols
    bits = gen_bits(seed, name, kind, row_start * cols, n, fan_in)
    return bf16_bits_to_f64(bits).reshape(row_end - row_start, cols)


def kvfill_rows(seed: int, layer: int, which: str, req: int, pos0: int, pos1: int,
                n_kv_heads: int, head_dim: int) -> np.ndarray:
    """Synthetic cached K or V of request ``req`` for positions [pos0, pos1) at ``layer``:
    fp64 array [pos1-pos0, n_kv_heads, head_dim] of bf16-exact K / fp16-exact V values
    (reading r-v16)."""
    name = f"kvfill.{layer}.{which}.{req}"
    per_pos = n_kv_heads * head_dim
    if which == "v":
        bits = gen_bits(seed, name, "kvfill_v", pos0 * per_pos, (pos1 - pos0) * per_pos)
        return f16_bits_to_f64(bits).reshape(pos1 - pos0, n_kv_heads, head_dim)
    bits = gen_bits(seed, name, "kvfill", pos0 * per_pos, (pos1 - pos0) * per_pos)
    return bf16_bits_to_f64(bits).reshape(pos1 - pos0, n_kv_heads, head_dim)
