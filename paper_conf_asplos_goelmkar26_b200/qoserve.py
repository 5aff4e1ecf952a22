"""Thin ctypes binding of libqoserve.so (include/qoserve.h, include/qoserve_ops.h).

Argument marshalling only: every step of the hybrid iteration runs in the library's sm_100a
kernels.  The functions below carry the C names; ``Engine`` bundles them for one engine and
uses PyTorch only to allocate the device arenas (weights, KV pool, workspace) and to supply
CUDA streams.  If the shared library is missing this module raises at import — there is no
CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libqoserve.so")

if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} not built: run `python -m paper_conf_asplos_goelmkar26_b200.build` "
                      "(or __graft_entry__.build()); there is no CPU fallback")
lib = C.CDLL(LIB_PATH)

QOS_OK = 0
ERRORS = {-1: "INVALID_ARG", -2: "OOM", -3: "UNKNOWN_REQ", -4: "BAD_KV_START", -5: "NOT_ALLOCATED",
          -6: "CUDA", -7: "COMM", -8: "UNSUPPORTED"}
QOS_F32, QOS_BF16 = 0, 1
EPI = {"store_bf16": 0, "store_f32": 1, "bias_bf16": 2, "silu_gate": 3, "add_f32": 4}
TIMING_CLASSES = ["meta", "embed", "norm", "gemm_qkv", "rope_append", "prefill_attn", "decode_attn", "gemm_o",
                  "gemm_gateup", "gemm_down", "allreduce", "head", "argmax"]


class QosError(RuntimeError):
    def __init__(self, code: int, where: str):
        self.code = code
        self.name = ERRORS.get(code, str(code))
        super().__init__(f"{where}: QOS_ERR_{self.name}: {lib.qos_last_error().decode()}")


class qos_model_cfg(C.Structure):
    _fields_ = [("n_layers", C.c_int32), ("d_model", C.c_int32), ("n_heads", C.c_int32),
                ("n_kv_heads", C.c_int32), ("head_dim", C.c_int32), ("ffn_dim", C.c_int32),
                ("vocab", C.c_int32), ("rope_theta", C.c_float), ("rms_eps", C.c_float),
                ("qkv_bias", C.c_int32), ("block_size", C.c_int32), ("num_blocks", C.c_int64),
                ("max_seq_len", C.c_int32), ("max_requests", C.c_int32),
                ("max_batch_tokens", C.c_int32), ("max_batch_rows", C.c_int32)]


class qos_mem_sizes(C.Structure):
    _fields_ = [("weight_bytes", C.c_uint64), ("kv_bytes", C.c_uint64), ("workspace_bytes", C.c_uint64)]


class qos_mem(C.Structure):
    _fields_ = [("weights", C.c_void_p), ("kv", C.c_void_p), ("workspace", C.c_void_p)]


class qos_shard(C.Structure):
    _fields_ = [("n_heads", C.c_int32), ("n_kv_heads", C.c_int32), ("ffn", C.c_int32), ("vocab", C.c_int32),
                ("head0", C.c_int32), ("kv_head0", C.c_int32), ("ffn0", C.c_int32), ("vocab0", C.c_int32)]


class qos_prefill_chunk(C.Structure):
    _fields_ = [("req", C.c_int64), ("kv_start", C.c_int32), ("chunk_len", C.c_int32),
                ("tokens", C.POINTER(C.c_int32))]


class qos_decode(C.Structure):
    _fields_ = [("req", C.c_int64), ("ctx_len", C.c_int32), ("token", C.c_int32)]


class qos_batch(C.Structure):
    _fields_ = [("n_prefill", C.c_int32), ("prefill", C.POINTER(qos_prefill_chunk)),
                ("n_decode", C.c_int32), ("decode", C.POINTER(qos_decode))]


_P = C.c_void_p
_SIGS = {
    "qos_engine_mem_sizes": [C.POINTER(qos_model_cfg), C.c_int, C.POINTER(qos_mem_sizes)],
    "qos_engine_create": [C.POINTER(qos_model_cfg), C.c_int, C.c_int, C.c_int, C.c_char_p,
                          C.POINTER(qos_mem), C.POINTER(_P)],
    "qos_engine_destroy": [_P],
    "qos_group_create": [C.c_int, C.POINTER(_P)],
    "qos_group_destroy": [_P],
    "qos_group_unique_id": [C.c_char_p],
    "qos_group_open": [C.c_char_p, C.c_int, C.c_int, C.POINTER(_P)],
    "qos_engine_create_peer": [C.POINTER(qos_model_cfg), C.c_int, C.c_int, _P, C.POINTER(qos_mem), C.POINTER(_P)],
    "qos_nccl_unique_id": [C.c_char_p],
    "qos_shard_plan": [C.POINTER(qos_model_cfg), C.c_int, C.c_int, C.POINTER(qos_shard)],
    "qos_engine_load_synthetic": [_P, C.c_uint64],
    "qos_engine_read_weight": [_P, C.c_char_p, C.c_int64, C.c_int64, _P],
    "qos_kv_alloc": [_P, C.c_int64, C.c_int32],
    "qos_kv_free": [_P, C.c_int64],
    "qos_kv_table": [_P, C.c_int64, C.POINTER(C.c_int32), C.c_int32, C.POINTER(C.c_int32)],
    "qos_kv_table_device": [_P, C.c_int64, C.POINTER(C.c_int32), C.c_int32, C.POINTER(C.c_int32)],
    "qos_kv_cached_len": [_P, C.c_int64, C.POINTER(C.c_int32)],
    "qos_kv_free_blocks": [_P, C.POINTER(C.c_int64)],
    "qos_kv_fill_synthetic": [_P, C.c_int64, C.c_int32, C.c_uint64],
    "qos_hybrid_step": [_P, C.POINTER(qos_batch), _P, C.c_int, _P, C.c_int, _P],
    "qos_hybrid_step_ex": [_P, C.POINTER(qos_batch), _P, C.c_int, _P, C.c_int, _P, _P],
    "qos_profile_step": [_P, C.c_int32, C.c_int32, C.POINTER(C.c_int32), C.c_int32, C.POINTER(C.c_float)],
    "qos_profile_step_ex": [_P, C.c_int32, C.c_int32, C.c_int32, C.POINTER(C.c_int32), C.c_int32, C.c_int32,
                            C.POINTER(C.c_float), C.POINTER(C.c_float)],
    "qos_engine_set_option": [_P, C.c_char_p, C.c_int64],
    "qos_engine_set_timing": [_P, C.c_int],
    "qos_last_step_timing": [_P, C.POINTER(C.c_float), C.POINTER(C.c_int32)],
    "qos_last_step_io": [_P, C.POINTER(C.c_int64), C.POINTER(C.c_int64)],
    "qos_engine_launch_count": [_P, C.POINTER(C.c_int64)],
    "qos_op_gemm": [_P, _P, _P, C.c_int64, C.c_int64, C.c_int64, C.c_int, _P, _P],
    "qos_op_gemm_ex": [_P, _P, _P, C.c_int64, C.c_int64, C.c_int64, C.c_int, _P, C.c_int, _P],
    "qos_op_rmsnorm": [_P, _P, _P, C.c_int32, C.c_int32, C.c_float, _P],
    "qos_kv_write": [_P, C.c_int32, C.c_int64, C.c_int32, C.c_int32, _P, _P],
    "qos_kv_read": [_P, C.c_int32, C.c_int64, C.c_int32, C.c_int32, _P, _P],
    "qos_op_qkv_rope_append": [_P, C.c_int32, C.POINTER(qos_batch), _P, _P],
    "qos_op_attention": [_P, C.c_int32, C.POINTER(qos_batch), _P, _P],
}
EXPORTED = sorted(list(_SIGS) + ["qos_strerror", "qos_last_error"])
for _name, _args in _SIGS.items():
    _f = getattr(lib, _name)
    _f.argtypes = _args
    _f.restype = C.c_int
lib.qos_strerror.argtypes = [C.c_int]
lib.qos_strerror.restype = C.c_char_p
lib.qos_last_error.argtypes = []
lib.qos_last_error.restype = C.c_char_p


def _chk(code: int, where: str) -> None:
    if code != QOS_OK:
        raise QosError(code, where)


def _call(name: str, *args) -> None:
    _chk(getattr(lib, name)(*args), name)


# module-level functions with the C names (marshalling only)
def qos_engine_mem_sizes(cfg: qos_model_cfg, tp_size: int = 1) -> qos_mem_sizes:
    out = qos_mem_sizes()
    _call("qos_engine_mem_sizes", C.byref(cfg), tp_size, C.byref(out))
    return out


def qos_shard_plan(cfg: qos_model_cfg, tp_rank: int, tp_size: int) -> qos_shard:
    out = qos_shard()
    _call("qos_shard_plan", C.byref(cfg), tp_rank, tp_size, C.byref(out))
    return out


def qos_nccl_unique_id() -> bytes:
    buf = C.create_string_buffer(128)
    _call("qos_nccl_unique_id", buf)
    return buf.raw


def qos_op_gemm(A, B, Cout, M: int, N: int, K: int, epi: str = "store_bf16", bias=None, stream=None):
    _call("qos_op_gemm", A, B, Cout, M, N, K, EPI[epi], bias, stream)


def qos_op_gemm_ex(A, B, Cout, M: int, N: int, K: int, epi: str = "store_bf16", bias=None, ksplit: int = 0,
                   stream=None):
    _call("qos_op_gemm_ex", A, B, Cout, M, N, K, EPI[epi], bias, ksplit, stream)


def qos_op_rmsnorm(x, g, out, T: int, d: int, eps: float, stream=None):
    _call("qos_op_rmsnorm", x, g, out, T, d, eps, stream)


def launch_count() -> int:
    n = C.c_int64()
    _call("qos_engine_launch_count", None, C.byref(n))
    return n.value


# ---------------------------------------------------------------------------- batches
@dataclass
class _BatchKeep:
    b: qos_batch
    keep: list


def make_batch(prefill=(), decode=()) -> _BatchKeep:
    """prefill: iterable of (req, kv_start, tokens); decode: iterable of (req, ctx_len, token)."""
    prefill = list(prefill)
    decode = list(decode)
    keep = []
    P = (qos_prefill_chunk * max(1, len(prefill)))()
    for i, (req, kv_start, toks) in enumerate(prefill):
        arr = np.ascontiguousarray(np.asarray(toks, dtype=np.int32))
        keep.append(arr)
        P[i] = qos_prefill_chunk(int(req), int(kv_start), int(len(arr)), arr.ctypes.data_as(C.POINTER(C.c_int32)))
    D = (qos_decode * max(1, len(decode)))()
    for i, (req, ctx, tok) in enumerate(decode):
        D[i] = qos_decode(int(req), int(ctx), int(tok))
    keep += [P, D]
    return _BatchKeep(qos_batch(len(prefill), P, len(decode), D), keep)


def batch_from_synth(b) -> _BatchKeep:
    """synth.Batch -> C descriptor."""
    return make_batch([(c.req, c.kv_start, c.tokens) for c in b.prefill],
                      [(d.req, d.ctx_len, d.token) for d in b.decode])


# ---------------------------------------------------------------------------- engine
def model_cfg(n_layers, d_model, n_heads, n_kv_heads, head_dim, ffn_dim, vocab, rope_theta, rms_eps,
              qkv_bias=False, num_blocks=4096, max_seq_len=8192, max_requests=1024,
              max_batch_tokens=8448, max_batch_rows=264) -> qos_model_cfg:
    return qos_model_cfg(n_layers, d_model, n_heads, n_kv_heads, head_dim, ffn_dim, vocab, rope_theta, rms_eps,
                         int(bool(qkv_bias)), 16, num_blocks, max_seq_len, max_requests, max_batch_tokens,
                         max_batch_rows)


def qos_group_unique_id() -> bytes:
    buf = C.create_string_buffer(64)
    _call("qos_group_unique_id", buf)
    return buf.raw


class Group:
    """Peer group of tp_size ranks: in-process (qos_group_create) or, with `group_id`, this
    process's membership (rank `rank`) of a cross-process group (qos_group_open).  Destroy after
    its engines."""

    def __init__(self, tp_size: int, group_id: bytes | None = None, rank: int = 0):
        self.tp_size = tp_size
        h = _P()
        if group_id is None:
            _call("qos_group_create", tp_size, C.byref(h))
        else:
            _call("qos_group_open", bytes(group_id).ljust(64, b"\0")[:64], tp_size, rank, C.byref(h))
        self.h = h

    def close(self):
        if getattr(self, "h", None):
            _call("qos_group_destroy", self.h)
            self.h = None


def run_ranks(fn, engines):
    """Call fn(rank, engine) on one thread per rank (a peer group's ranks must step concurrently;
    ctypes releases the GIL during the C calls).  Returns the per-rank results; re-raises the
    first failure."""
    import concurrent.futures as cf
    with cf.ThreadPoolExecutor(max_workers=len(engines)) as ex:
        futs = [ex.submit(fn, r, e) for r, e in enumerate(engines)]
        return [f.result() for f in futs]


class Engine:
    """One libqoserve engine on one GPU (one TP rank).  Device arenas are torch tensors."""

    def __init__(self, cfg: qos_model_cfg, device: int = 0, tp_rank: int = 0, tp_size: int = 1,
                 nccl_uid: bytes | None = None, torch_arenas: bool = True, group: "Group | None" = None):
        import torch
        self.cfg = cfg
        self.device = device
        self.tp_rank, self.tp_size = tp_rank, tp_size
        self.sizes = qos_engine_mem_sizes(cfg, tp_size)
        mem = None
        self._arenas = []
        if torch_arenas:
            dev = torch.device("cuda", device)
            arenas = [torch.empty(int(n), dtype=torch.uint8, device=dev)
                      for n in (self.sizes.weight_bytes, self.sizes.kv_bytes, self.sizes.workspace_bytes)]
            self._arenas = arenas
            mem = qos_mem(arenas[0].data_ptr(), arenas[1].data_ptr(), arenas[2].data_ptr())
        h = _P()
        if group is not None:
            assert tp_size == group.tp_size
            _call("qos_engine_create_peer", C.byref(cfg), device, tp_rank, group.h,
                  C.byref(mem) if mem is not None else None, C.byref(h))
        else:
            _call("qos_engine_create", C.byref(cfg), device, tp_rank, tp_size, nccl_uid,
                  C.byref(mem) if mem is not None else None, C.byref(h))
        self.h = h
        self.group = group

    def close(self):
        if getattr(self, "h", None):
            lib.qos_engine_destroy(self.h)
            self.h = None
            self._arenas = []

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # weights
    def qos_engine_load_synthetic(self, seed: int = 0):
        _call("qos_engine_load_synthetic", self.h, seed)

    def qos_engine_read_weight(self, name: str, row0: int, nrows: int, cols: int) -> np.ndarray:
        out = np.empty((nrows, cols), dtype=np.uint16)
        _call("qos_engine_read_weight", self.h, name.encode(), row0, nrows, out.ctypes.data)
        return out

    # KV
    def qos_kv_alloc(self, req: int, n_tokens_total: int):
        _call("qos_kv_alloc", self.h, req, n_tokens_total)

    def qos_kv_free(self, req: int):
        _call("qos_kv_free", self.h, req)

    def qos_kv_table(self, req: int) -> list[int]:
        n = C.c_int32()
        _call("qos_kv_table", self.h, req, None, 0, C.byref(n))
        buf = (C.c_int32 * max(1, n.value))()
        _call("qos_kv_table", self.h, req, buf, n.value, C.byref(n))
        return [buf[i] for i in range(n.value)]

    def qos_kv_table_device(self, req: int) -> list[int]:
        n = C.c_int32()
        _call("qos_kv_table", self.h, req, None, 0, C.byref(n))
        buf = (C.c_int32 * max(1, n.value))()
        _call("qos_kv_table_device", self.h, req, buf, n.value, C.byref(n))
        return [buf[i] for i in range(n.value)]

    def qos_kv_cached_len(self, req: int) -> int:
        n = C.c_int32()
        _call("qos_kv_cached_len", self.h, req, C.byref(n))
        return n.value

    def qos_kv_free_blocks(self) -> int:
        n = C.c_int64()
        _call("qos_kv_free_blocks", self.h, C.byref(n))
        return n.value

    def qos_kv_fill_synthetic(self, req: int, n_tokens: int, seed: int = 2):
        _call("qos_kv_fill_synthetic", self.h, req, n_tokens, seed)

    def qos_kv_write(self, layer: int, req: int, pos0: int, k_bits: np.ndarray, v_bits: np.ndarray):
        k = np.ascontiguousarray(k_bits, dtype=np.uint16)
        v = np.ascontiguousarray(v_bits, dtype=np.uint16)
        _call("qos_kv_write", self.h, layer, req, pos0, k.shape[0], k.ctypes.data, v.ctypes.data)

    def qos_kv_read(self, layer: int, req: int, pos0: int, n: int, hkv: int, hd: int):
        k = np.empty((n, hkv, hd), dtype=np.uint16)
        v = np.empty((n, hkv, hd), dtype=np.uint16)
        _call("qos_kv_read", self.h, layer, req, pos0, n, k.ctypes.data, v.ctypes.data)
        return k, v

    # step
    def qos_hybrid_step(self, batch: _BatchKeep, logits=None, logits_dtype: int = QOS_F32, next_tokens=None,
                        outputs_on_host: bool = False, stream=None):
        _call("qos_hybrid_step", self.h, C.byref(batch.b), logits, logits_dtype, next_tokens,
              int(bool(outputs_on_host)), stream)

    def qos_hybrid_step_ex(self, batch: _BatchKeep, logits=None, logits_dtype: int = QOS_F32, next_tokens=None,
                           outputs_on_host: bool = False, stream=None, decode_tokens_dev=None):
        """qos_hybrid_step with the decodes' tokens read from device memory (int32 pointer)."""
        _call("qos_hybrid_step_ex", self.h, C.byref(batch.b), logits, logits_dtype, next_tokens,
              int(bool(outputs_on_host)), stream, decode_tokens_dev)

    def step_host(self, batch: _BatchKeep, vocab: int):
        """Convenience: run a step with host outputs; returns (logits f32 [R, V], tokens [R])."""
        R = batch.b.n_prefill + batch.b.n_decode
        lg = np.empty((R, vocab), dtype=np.float32)
        tk = np.empty((R,), dtype=np.int32)
        self.qos_hybrid_step(batch, lg.ctypes.data, QOS_F32, tk.ctypes.data, True, None)
        return lg, tk

    def qos_profile_step(self, chunk_len: int, ctx_lens, reps: int = 10, kv_start: int = 0, warmup: int = -1):
        ctx = np.ascontiguousarray(np.asarray(ctx_lens, dtype=np.int32))
        med, p95 = C.c_float(), C.c_float()
        _call("qos_profile_step_ex", self.h, chunk_len, kv_start, len(ctx),
              ctx.ctypes.data_as(C.POINTER(C.c_int32)), warmup, reps, C.byref(med), C.byref(p95))
        return med.value, p95.value

    def qos_engine_set_option(self, name: str, value: int):
        _call("qos_engine_set_option", self.h, name.encode(), int(value))

    def qos_engine_set_timing(self, enable: bool):
        _call("qos_engine_set_timing", self.h, int(bool(enable)))

    def qos_last_step_timing(self):
        ms = (C.c_float * len(TIMING_CLASSES))()
        n = (C.c_int32 * len(TIMING_CLASSES))()
        _call("qos_last_step_timing", self.h, ms, n)
        return {k: (ms[i], n[i]) for i, k in enumerate(TIMING_CLASSES)}

    def qos_last_step_io(self):
        a, b = C.c_int64(), C.c_int64()
        _call("qos_last_step_io", self.h, C.byref(a), C.byref(b))
        return a.value, b.value

    # ops
    def qos_op_qkv_rope_append(self, layer: int, batch: _BatchKeep, h_bits: np.ndarray, q_cols: int):
        hh = np.ascontiguousarray(h_bits, dtype=np.uint16)
        q = np.empty((hh.shape[0], q_cols), dtype=np.uint16)
        _call("qos_op_qkv_rope_append", self.h, layer, C.byref(batch.b), hh.ctypes.data, q.ctypes.data)
        return q

    def qos_op_attention(self, layer: int, batch: _BatchKeep, q_bits: np.ndarray) -> np.ndarray:
        q = np.ascontiguousarray(q_bits, dtype=np.uint16)
        out = np.empty(q.shape, dtype=np.float32)
        _call("qos_op_attention", self.h, layer, C.byref(batch.b), q.ctypes.data, out.ctypes.data)
        return out
