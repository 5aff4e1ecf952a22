// gen.cu — device implementation of the synthetic weight / KV generator.
// The paper serves Hugging Face checkpoints; with no network the engine
// draws bf16 weights from a counter-based generator whose SPEC (not code) is shared with the
// oracle, which has its own numpy implementation:
//   a = ((splitmix64((seed ^ fnv1a64(name)) + i) >> 40) - 2^23) / 2^23
//   linear: bf16(fp32(a * s)), s = fp32(1/sqrt(fan_in));  embed / kvfill: bf16(a);
//   norm: bf16(fp32(1 + fp32(0.1 a)));  bias: bf16(fp32(0.02 a))      (all fp32 ops RNE, no FMA)
#include <cuda_fp16.h>

#include "common.cuh"
#include "internal.h"

namespace qos {

uint64_t fnv1a64(const char* s) {
  uint64_t h = 0xCBF29CE484222325ull;
  for (; *s; ++s) {
    h ^= (uint8_t)*s;
    h *= 0x100000001B3ull;
  }
  return h;
}

QOS_DEV uint64_t splitmix64(uint64_t z) {
  z += 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

QOS_DEV float gen_value(uint64_t base, uint64_t i, int kind, float s) {
  const int k = int(splitmix64(base + i) >> 40);
  const float a = float(k - (1 << 23)) * (1.0f / 8388608.0f);  // exact
  switch (kind) {
    case GEN_LINEAR: return __fmul_rn(a, s);
    case GEN_NORM: return __fadd_rn(1.0f, __fmul_rn(0.1f, a));
    case GEN_BIAS: return __fmul_rn(0.02f, a);
    default: return a;  // embed, kvfill
  }
}

// dst[r * dst_ld + c] for r < rows, c < cols  <-  element (row0 + r, col0 + c) of a source
// tensor with src_cols columns.  interleave >= 0 remaps destination rows for the gate/up
// interleave of QOS_EPI_SILU_GATE: dst row = (r / 64) * 128 + interleave * 64 + r % 64.
__global__ void gen_fill_kernel(__nv_bfloat16* __restrict__ dst, int64_t dst_ld, int64_t rows, int64_t cols,
                                uint64_t base, int64_t row0, int64_t col0, int64_t src_cols, int kind, float s,
                                int interleave) {
  const int64_t n = rows * cols;
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < n; e += int64_t(gridDim.x) * blockDim.x) {
    const int64_t r = e / cols, c = e % cols;
    const uint64_t i = uint64_t((row0 + r) * src_cols + col0 + c);
    const int64_t dr = interleave >= 0 ? (r / 64) * 128 + interleave * 64 + (r % 64) : r;
    dst[dr * dst_ld + c] = __float2bfloat16_rn(gen_value(base, i, kind, s));
  }
}

__global__ void gen_bias_f32_kernel(float* __restrict__ dst, int64_t n, uint64_t base, int64_t off) {
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < n; e += int64_t(gridDim.x) * blockDim.x)
    dst[e] = __bfloat162float(__float2bfloat16_rn(gen_value(base, uint64_t(off + e), GEN_BIAS, 0.f)));
}

// KV fill of one request for one (layer, K|V) plane: positions [0, n), local heads h <
// hkv_local map to global head kv_head0 + h; i = (pos * hkv_global + global head) * hd + j.
__global__ void kvfill_kernel(uint16_t* __restrict__ plane, const int32_t* __restrict__ table, int n,
                              int hkv_local, int hkv_global, int kv_head0, int hd, uint64_t base, int fp16) {
  const int64_t total = int64_t(n) * hkv_local * hd;
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < total; e += int64_t(gridDim.x) * blockDim.x) {
    const int j = int(e % hd);
    const int h = int((e / hd) % hkv_local);
    const int pos = int(e / (int64_t(hd) * hkv_local));
    const uint64_t i = (uint64_t(pos) * hkv_global + kv_head0 + h) * hd + j;
    const int blk = table[pos >> 4];
    const float v = gen_value(base, i, GEN_EMBED, 0.f);  // exact in fp32 (24-bit fraction)
    plane[((int64_t(blk) * hkv_local + h) * 16 + (pos & 15)) * hd + j] =
        fp16 ? __half_as_ushort(__float2half_rn(v)) : __bfloat16_as_ushort(__float2bfloat16_rn(v));
  }
}

static int grid_for(int64_t n) {
  int64_t b = (n + 255) / 256;
  return int(b < 148 * 16 ? (b < 1 ? 1 : b) : 148 * 16);
}

cudaError_t gen_fill_bf16_ex(void* dst, int64_t dst_ld, int64_t rows, int64_t cols, uint64_t seed, uint64_t name_hash,
                             int64_t row0, int64_t col0, int64_t src_cols, int kind, int fan_in, int interleave,
                             cudaStream_t st) {
  const float s = kind == GEN_LINEAR ? float(1.0 / sqrt(double(fan_in))) : 0.f;
  count_launch();
  gen_fill_kernel<<<grid_for(rows * cols), 256, 0, st>>>((__nv_bfloat16*)dst, dst_ld, rows, cols, seed ^ name_hash,
                                                          row0, col0, src_cols, kind, s, interleave);
  return cudaGetLastError();
}

cudaError_t gen_fill_bf16(void* dst, int64_t dst_ld, int64_t rows, int64_t cols, uint64_t seed, uint64_t name_hash,
                          int64_t row0, int64_t col0, int64_t src_cols, int kind, int fan_in, cudaStream_t st) {
  return gen_fill_bf16_ex(dst, dst_ld, rows, cols, seed, name_hash, row0, col0, src_cols, kind, fan_in, -1, st);
}

cudaError_t gen_fill_f32_bias(float* dst, int64_t n, uint64_t seed, uint64_t name_hash, int64_t off, cudaStream_t st) {
  count_launch();
  gen_bias_f32_kernel<<<grid_for(n), 256, 0, st>>>(dst, n, seed ^ name_hash, off);
  return cudaGetLastError();
}

cudaError_t kvfill_launch(void* plane, const int32_t* d_table, int n_tokens, int hkv_local, int hkv_global,
                          int kv_head0, int hd, uint64_t seed, uint64_t name_hash, int fp16, cudaStream_t st) {
  if (n_tokens == 0) return cudaSuccess;
  count_launch();
  kvfill_kernel<<<grid_for(int64_t(n_tokens) * hkv_local * hd), 256, 0, st>>>(
      (uint16_t*)plane, d_table, n_tokens, hkv_local, hkv_global, kv_head0, hd, seed ^ name_hash, fp16);
  return cudaGetLastError();
}

}  // namespace qos
