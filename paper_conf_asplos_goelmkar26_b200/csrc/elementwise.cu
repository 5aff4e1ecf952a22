// elementwise.cu — HBM-bound per-token kernels of the hybrid step (SURVEY.md §8(a) rows a2, a3,
// a5+a6, a13 gather, a14):
//   embed_rmsnorm   x = E[tok] (fp32 residual init) and h = RMSNorm(x)·g1 of layer 0   (a2+a3)
//   rmsnorm         h = RMSNorm(r)·g from the fp32 residual stream                       (a3)
//   gather_rmsnorm  the R logit rows (last token of each chunk, every decode) + final norm (a13)
//   (RoPE + the paged KV append (a5+a6) run in the QKV GEMM epilogue, gemm.cu)
//   argmax          greedy token, lowest index on ties                                    (a14)
// One CTA per token row; 16-byte vector loads/stores; fp32 statistics.
#include <cfloat>

#include "common.cuh"
#include "internal.h"

namespace qos {

constexpr int kRowThreads = 256;

QOS_DEV float block_sum(float v, float* red) {
  v = warp_sum(v);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  __syncthreads();
  if (l == 0) red[w] = v;
  __syncthreads();
  float s = 0.f;
  for (int i = 0; i < (int)(blockDim.x >> 5); ++i) s += red[i];
  return s;
}

// d is a multiple of 8; each thread handles 8 contiguous elements per chunk.  Rows up to
// kRowThreads * 8 * kMaxChunks elements (8192 at 256 threads: Llama-3-70B) are held in
// registers: one HBM read of the row, all loads issued before the reduction.
constexpr int kMaxChunks = 4;
QOS_DEV void norm_row(const float* x, const __nv_bfloat16* g, __nv_bfloat16* out, int d, float eps, float* red) {
  if (d <= int(blockDim.x) * 8 * kMaxChunks) {
    float4 a[kMaxChunks], b[kMaxChunks];
    float ss = 0.f;
#pragma unroll
    for (int k = 0; k < kMaxChunks; ++k) {
      const int c = (threadIdx.x + k * blockDim.x) * 8;
      if (c < d) {
        a[k] = __ldcs(reinterpret_cast<const float4*>(x + c));
        b[k] = __ldcs(reinterpret_cast<const float4*>(x + c + 4));
      } else {
        a[k] = b[k] = make_float4(0.f, 0.f, 0.f, 0.f);
      }
    }
#pragma unroll
    for (int k = 0; k < kMaxChunks; ++k)
      ss += a[k].x * a[k].x + a[k].y * a[k].y + a[k].z * a[k].z + a[k].w * a[k].w + b[k].x * b[k].x +
            b[k].y * b[k].y + b[k].z * b[k].z + b[k].w * b[k].w;
    const float inv = rsqrtf(block_sum(ss, red) / float(d) + eps);
#pragma unroll
    for (int k = 0; k < kMaxChunks; ++k) {
      const int c = (threadIdx.x + k * blockDim.x) * 8;
      if (c < d) {
        const float v[8] = {a[k].x, a[k].y, a[k].z, a[k].w, b[k].x, b[k].y, b[k].z, b[k].w};
        const uint4 gw = __ldg(reinterpret_cast<const uint4*>(g + c));
        const uint32_t gg[4] = {gw.x, gw.y, gw.z, gw.w};
        uint32_t pk[4];
#pragma unroll
        for (int i = 0; i < 4; ++i)
          pk[i] = pack_bf16(v[2 * i] * inv * bf16_lo(gg[i]), v[2 * i + 1] * inv * bf16_hi(gg[i]));
        *reinterpret_cast<uint4*>(out + c) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
      }
    }
    return;
  }
  // longer rows: two passes (the second read hits L1/L2)
  float ss = 0.f;
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    const float4 a = *reinterpret_cast<const float4*>(x + c);
    const float4 b = *reinterpret_cast<const float4*>(x + c + 4);
    ss += a.x * a.x + a.y * a.y + a.z * a.z + a.w * a.w + b.x * b.x + b.y * b.y + b.z * b.z + b.w * b.w;
  }
  const float tot = block_sum(ss, red);
  const float inv = rsqrtf(tot / float(d) + eps);
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    const float4 a = *reinterpret_cast<const float4*>(x + c);
    const float4 b = *reinterpret_cast<const float4*>(x + c + 4);
    const float v[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
    const uint4 gw = *reinterpret_cast<const uint4*>(g + c);
    const uint32_t gg[4] = {gw.x, gw.y, gw.z, gw.w};
    uint32_t pk[4];
#pragma unroll
    for (int i = 0; i < 4; ++i)
      pk[i] = pack_bf16(v[2 * i] * inv * bf16_lo(gg[i]), v[2 * i + 1] * inv * bf16_hi(gg[i]));
    *reinterpret_cast<uint4*>(out + c) = make_uint4(pk[0], pk[1], pk[2], pk[3]);
  }
}

__global__ void __launch_bounds__(kRowThreads) embed_rmsnorm_kernel(const int32_t* __restrict__ tokens,
                                                                    const __nv_bfloat16* __restrict__ emb,
                                                                    const __nv_bfloat16* __restrict__ g,
                                                                    float* __restrict__ resid,
                                                                    __nv_bfloat16* __restrict__ out, int d, float eps) {
  griddep_wait();
  griddep_launch_dependents();
  __shared__ float red[32];
  const int t = blockIdx.x;
  const __nv_bfloat16* e = emb + size_t(tokens[t]) * d;
  float* r = resid + size_t(t) * d;
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    const uint4 w = *reinterpret_cast<const uint4*>(e + c);
    *reinterpret_cast<float4*>(r + c) = make_float4(bf16_lo(w.x), bf16_hi(w.x), bf16_lo(w.y), bf16_hi(w.y));
    *reinterpret_cast<float4*>(r + c + 4) = make_float4(bf16_lo(w.z), bf16_hi(w.z), bf16_lo(w.w), bf16_hi(w.w));
  }
  // each thread re-reads only the elements it wrote: no barrier needed before norm_row
  norm_row(r, g, out + size_t(t) * d, d, eps, red);
}

__global__ void __launch_bounds__(kRowThreads) rmsnorm_kernel(const float* __restrict__ x,
                                                              const __nv_bfloat16* __restrict__ g,
                                                              __nv_bfloat16* __restrict__ out, int d, float eps) {
  griddep_wait();
  griddep_launch_dependents();
  __shared__ float red[32];
  const int t = blockIdx.x;
  norm_row(x + size_t(t) * d, g, out + size_t(t) * d, d, eps, red);
}

__global__ void __launch_bounds__(kRowThreads) gather_rmsnorm_kernel(const float* __restrict__ x,
                                                                     const int32_t* __restrict__ rows,
                                                                     const __nv_bfloat16* __restrict__ g,
                                                                     __nv_bfloat16* __restrict__ out, int d,
                                                                     float eps) {
  griddep_wait();
  griddep_launch_dependents();
  __shared__ float red[32];
  const int r = blockIdx.x;
  norm_row(x + size_t(rows[r]) * d, g, out + size_t(r) * d, d, eps, red);
}

// resid[t] += add[t] (bf16); out[t] = RMSNorm(resid[t]) * g.  `out` may alias `add`: every
// thread reads add[c] in pass 1 before it writes out[c] in pass 2 (same indices, same thread).
__global__ void __launch_bounds__(kRowThreads) add_rmsnorm_kernel(float* __restrict__ resid, const __nv_bfloat16* add,
                                                                  const __nv_bfloat16* __restrict__ g,
                                                                  __nv_bfloat16* out, int d, float eps) {
  griddep_wait();
  griddep_launch_dependents();
  __shared__ float red[32];
  const int t = blockIdx.x;
  float* r = resid + size_t(t) * d;
  const __nv_bfloat16* a = add + size_t(t) * d;
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    const uint4 w = *reinterpret_cast<const uint4*>(a + c);
    float4 x0 = *reinterpret_cast<float4*>(r + c), x1 = *reinterpret_cast<float4*>(r + c + 4);
    x0.x += bf16_lo(w.x); x0.y += bf16_hi(w.x); x0.z += bf16_lo(w.y); x0.w += bf16_hi(w.y);
    x1.x += bf16_lo(w.z); x1.y += bf16_hi(w.z); x1.z += bf16_lo(w.w); x1.w += bf16_hi(w.w);
    *reinterpret_cast<float4*>(r + c) = x0;
    *reinterpret_cast<float4*>(r + c + 4) = x1;
  }
  norm_row(r, g, out + size_t(t) * d, d, eps, red);
}

// Peer-memory TP reduction (in-process peer group, qos_engine_create_peer): row t of every
// rank's bf16 partial (O or down projection output of its head / FFN slice) is
// read straight from that rank's workspace (same device, or a peer GPU over NVLink), summed in
// fp32 in rank order — so every rank computes the bit-identical sum — and added to the fp32
// residual; with g != nullptr the row is then RMS-normalised into `out` (the next GEMM's A
// operand).  One kernel replaces all-reduce + add + RMSNorm.  Ordering against the producers'
// GEMMs is by stream events (engine.cu: peer_sync); loads bypass L1 (__ldcg).
__global__ void __launch_bounds__(kRowThreads) peer_add_rmsnorm_kernel(PeerPtrs parts, int tp, float* __restrict__ resid,
                                                                       const __nv_bfloat16* __restrict__ g,
                                                                       __nv_bfloat16* __restrict__ out, int d,
                                                                       float eps) {
  griddep_wait();
  griddep_launch_dependents();
  __shared__ float red[32];
  const int t = blockIdx.x;
  float* r = resid + size_t(t) * d;
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    float s[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
    for (int k = 0; k < tp; ++k) {
      const uint4 w = __ldcg(reinterpret_cast<const uint4*>(
          reinterpret_cast<const __nv_bfloat16*>(parts.p[k]) + size_t(t) * d + c));
      s[0] += bf16_lo(w.x); s[1] += bf16_hi(w.x); s[2] += bf16_lo(w.y); s[3] += bf16_hi(w.y);
      s[4] += bf16_lo(w.z); s[5] += bf16_hi(w.z); s[6] += bf16_lo(w.w); s[7] += bf16_hi(w.w);
    }
    float4 x0 = *reinterpret_cast<float4*>(r + c), x1 = *reinterpret_cast<float4*>(r + c + 4);
    x0.x += s[0]; x0.y += s[1]; x0.z += s[2]; x0.w += s[3];
    x1.x += s[4]; x1.y += s[5]; x1.z += s[6]; x1.w += s[7];
    *reinterpret_cast<float4*>(r + c) = x0;
    *reinterpret_cast<float4*>(r + c + 4) = x1;
  }
  if (g) norm_row(r, g, out + size_t(t) * d, d, eps, red);  // same thread -> element map: no barrier
}

// Two-shot form of the same reduction for larger groups (tp >= 4): rank `rank` reduces only the
// rows [row0, row0 + gridDim.x) it owns (reduce-scatter by row slices: reads (tp-1)/tp of one
// partial instead of tp-1 partials), adds them to its residual rows, normalises them into its own
// h and stores the normalised bf16 rows into every peer's h (the all-gather, by peer stores).
// store_resid (last layer, g == nullptr): the updated fp32 residual rows are stored into every
// peer's residual instead, so the final gather + norm of the logit rows sees fresh rows.
__global__ void __launch_bounds__(kRowThreads) peer_rs_norm_ag_kernel(PeerPtrs parts, PeerPtrs hs, PeerPtrs resids,
                                                                      int tp, int rank, int row0,
                                                                      const __nv_bfloat16* __restrict__ g, int d,
                                                                      float eps) {
  griddep_wait();
  griddep_launch_dependents();
  __shared__ float red[32];
  const int t = row0 + blockIdx.x;
  float* r = reinterpret_cast<float*>(const_cast<void*>(resids.p[rank])) + size_t(t) * d;
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    float s[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
    for (int k = 0; k < tp; ++k) {
      const uint4 w = __ldcg(reinterpret_cast<const uint4*>(
          reinterpret_cast<const __nv_bfloat16*>(parts.p[k]) + size_t(t) * d + c));
      s[0] += bf16_lo(w.x); s[1] += bf16_hi(w.x); s[2] += bf16_lo(w.y); s[3] += bf16_hi(w.y);
      s[4] += bf16_lo(w.z); s[5] += bf16_hi(w.z); s[6] += bf16_lo(w.w); s[7] += bf16_hi(w.w);
    }
    float4 x0 = *reinterpret_cast<float4*>(r + c), x1 = *reinterpret_cast<float4*>(r + c + 4);
    x0.x += s[0]; x0.y += s[1]; x0.z += s[2]; x0.w += s[3];
    x1.x += s[4]; x1.y += s[5]; x1.z += s[6]; x1.w += s[7];
    *reinterpret_cast<float4*>(r + c) = x0;
    *reinterpret_cast<float4*>(r + c + 4) = x1;
    if (!g) {
      for (int k = 0; k < tp; ++k) {
        if (k == rank) continue;
        float* pr = reinterpret_cast<float*>(const_cast<void*>(resids.p[k])) + size_t(t) * d + c;
        *reinterpret_cast<float4*>(pr) = x0;
        *reinterpret_cast<float4*>(pr + 4) = x1;
      }
    }
  }
  if (!g) return;
  __nv_bfloat16* own = reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(hs.p[rank])) + size_t(t) * d;
  norm_row(r, g, own, d, eps, red);
  // the thread re-reads only the h elements it wrote and forwards them to the peers
  for (int c = threadIdx.x * 8; c < d; c += blockDim.x * 8) {
    const uint4 v = *reinterpret_cast<const uint4*>(own + c);
    for (int k = 0; k < tp; ++k)
      if (k != rank)
        *reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(const_cast<void*>(hs.p[k])) + size_t(t) * d + c) = v;
  }
}

// Vocab-parallel LM head gather over peer memory: rank k's [R][Vl] f32 logits slice -> columns
// [k*Vl, (k+1)*Vl) of out [R][tp*Vl].
__global__ void peer_gather_logits_kernel(PeerPtrs loc, int tp, int R, int Vl, float* __restrict__ out) {
  griddep_wait();
  griddep_launch_dependents();
  const int64_t per = int64_t(R) * Vl, n = per * tp;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const int k = int(i / per);
    const int64_t rem = i - int64_t(k) * per;
    const int r = int(rem / Vl), j = int(rem - int64_t(r) * Vl);
    out[int64_t(r) * Vl * tp + int64_t(k) * Vl + j] = __ldcg(reinterpret_cast<const float*>(loc.p[k]) + rem);
  }
}

__global__ void add_f32_kernel(float* __restrict__ resid, const __nv_bfloat16* __restrict__ add, int64_t n) {
  griddep_wait();
  griddep_launch_dependents();
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
    resid[i] += __bfloat162float(add[i]);
}

__global__ void unshard_logits_kernel(const float* __restrict__ in, float* __restrict__ out, int R, int Vl, int tp) {
  griddep_wait();
  griddep_launch_dependents();
  const int64_t n = int64_t(R) * Vl * tp;
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x) {
    const int j = int(i % Vl);
    const int r = int((i / Vl) % R);
    const int k = int(i / (int64_t(Vl) * R));
    out[int64_t(r) * Vl * tp + int64_t(k) * Vl + j] = in[i];
  }
}

// argmax per row; ties -> lowest index.  logits f32 or bf16 [R][V].
// argmax per row; ties -> lowest index.  logits f32 or bf16 [R][V].  Grid (R, S): CTA (r, s)
// scans the s-th of S contiguous slices of row r (16-byte loads on the f32 path), parks its
// (value, index) in part[r][s]; the last of the row's S CTAs to arrive merges the slices in
// slice order (arrival counter, reset for the next launch).  S = 1 writes out directly.
QOS_DEV void amax_merge(float& best, int& bi, float v, int i) {
  if (v > best || (v == best && i < bi)) {
    best = v;
    bi = i;
  }
}
__global__ void argmax_kernel(const void* __restrict__ logits, int is_f32, int V, int32_t* __restrict__ out,
                              float2* __restrict__ part, int* __restrict__ cnt) {
  griddep_wait();
  griddep_launch_dependents();
  const int r = blockIdx.x, S = gridDim.y, sl = blockIdx.y;
  const int per = ((V + S - 1) / S + 3) & ~3;  // slice length, a multiple of 4
  const int i0 = sl * per, i1 = min(V, i0 + per);
  float best = -INFINITY;
  int bi = 0x7fffffff;
  if (is_f32 && (V & 3) == 0) {
    const float4* row = reinterpret_cast<const float4*>(reinterpret_cast<const float*>(logits) + size_t(r) * V);
    for (int q = (i0 >> 2) + threadIdx.x; q < (i1 >> 2); q += blockDim.x) {  // this thread's indices increase
      const float4 x = __ldcs(row + q);
      const int i = q << 2;
      if (x.x > best) { best = x.x; bi = i; }
      if (x.y > best) { best = x.y; bi = i + 1; }
      if (x.z > best) { best = x.z; bi = i + 2; }
      if (x.w > best) { best = x.w; bi = i + 3; }
    }
  } else {
    for (int i = i0 + threadIdx.x; i < i1; i += blockDim.x) {
      const float v = is_f32 ? reinterpret_cast<const float*>(logits)[size_t(r) * V + i]
                             : __bfloat162float(reinterpret_cast<const __nv_bfloat16*>(logits)[size_t(r) * V + i]);
      if (v > best) { best = v; bi = i; }
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1)
    amax_merge(best, bi, __shfl_xor_sync(0xffffffffu, best, o), __shfl_xor_sync(0xffffffffu, bi, o));
  __shared__ float sv[32];
  __shared__ int si[32];
  __shared__ int s_last;
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) {
    sv[w] = best;
    si[w] = bi;
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  for (int k = 1; k < (int)(blockDim.x >> 5); ++k) amax_merge(best, bi, sv[k], si[k]);
  if (S == 1) {
    out[r] = bi;
    return;
  }
  part[size_t(r) * S + sl] = make_float2(best, __int_as_float(bi));
  __threadfence();
  s_last = atomicAdd(cnt + r, 1) == S - 1;
  if (!s_last) return;
  __threadfence();
  float b2 = -INFINITY;
  int i2 = 0x7fffffff;
  for (int k = 0; k < S; ++k) {
    const float2 pk = __ldcg(part + size_t(r) * S + k);
    amax_merge(b2, i2, pk.x, __float_as_int(pk.y));
  }
  out[r] = i2;
  cnt[r] = 0;
}

__global__ void f32_to_bf16_kernel(const float* __restrict__ x, __nv_bfloat16* __restrict__ y, int64_t n) {
  griddep_wait();
  griddep_launch_dependents();
  for (int64_t i = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; i < n; i += int64_t(gridDim.x) * blockDim.x)
    y[i] = __float2bfloat16_rn(x[i]);
}

__global__ void kv_scatter_kernel(__nv_bfloat16* __restrict__ plane, const int32_t* __restrict__ trow, int pos0, int n,
                                  int Hkv, int hd, const __nv_bfloat16* __restrict__ src) {
  const int64_t total = int64_t(n) * Hkv * hd;
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < total; e += int64_t(gridDim.x) * blockDim.x) {
    const int j = int(e % hd), h = int((e / hd) % Hkv), i = int(e / (int64_t(hd) * Hkv));
    const int p = pos0 + i;
    plane[((int64_t(trow[p >> 4]) * Hkv + h) * 16 + (p & 15)) * hd + j] = src[e];
  }
}
__global__ void kv_gather_kernel(const __nv_bfloat16* __restrict__ plane, const int32_t* __restrict__ trow, int pos0,
                                 int n, int Hkv, int hd, __nv_bfloat16* __restrict__ dst) {
  const int64_t total = int64_t(n) * Hkv * hd;
  for (int64_t e = blockIdx.x * int64_t(blockDim.x) + threadIdx.x; e < total; e += int64_t(gridDim.x) * blockDim.x) {
    const int j = int(e % hd), h = int((e / hd) % Hkv), i = int(e / (int64_t(hd) * Hkv));
    const int p = pos0 + i;
    dst[e] = plane[((int64_t(trow[p >> 4]) * Hkv + h) * 16 + (p & 15)) * hd + j];
  }
}
__global__ void table_update_kernel(int32_t* __restrict__ tables, int table_w, const int32_t* __restrict__ tr, int n) {
  griddep_wait();
  griddep_launch_dependents();
  const int i = blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) tables[size_t(tr[3 * i]) * table_w + tr[3 * i + 1]] = tr[3 * i + 2];
}

// ------------------------------------------------------------------------------ host
static int grid_of(int64_t n) {
  const int64_t b = (n + 255) / 256;
  return int(b < 1 ? 1 : (b > 4096 ? 4096 : b));
}
cudaError_t launch_kv_scatter(void* plane, const int32_t* d_table_row, int pos0, int n, int Hkv, int hd,
                              const void* src, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  count_launch();
  kv_scatter_kernel<<<grid_of(int64_t(n) * Hkv * hd), 256, 0, st>>>((__nv_bfloat16*)plane, d_table_row, pos0, n, Hkv,
                                                                     hd, (const __nv_bfloat16*)src);
  return cudaGetLastError();
}
cudaError_t launch_kv_gather(const void* plane, const int32_t* d_table_row, int pos0, int n, int Hkv, int hd, void* dst,
                             cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  count_launch();
  kv_gather_kernel<<<grid_of(int64_t(n) * Hkv * hd), 256, 0, st>>>((const __nv_bfloat16*)plane, d_table_row, pos0, n,
                                                                    Hkv, hd, (__nv_bfloat16*)dst);
  return cudaGetLastError();
}
cudaError_t launch_table_update(int32_t* tables, int table_w, const int32_t* triples, int n, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(table_update_kernel, dim3((n + 255) / 256), dim3(256), 0, st, tables, table_w, triples, n);
}
// decode tokens taken from device memory (qos_hybrid_step_ex): the step's token array gets
// src[0..n) at the decode rows, clamped to [0, vocab) (the engine's own argmax outputs always are)
__global__ void token_patch_kernel(int32_t* __restrict__ dst, const int32_t* __restrict__ src, int n, int vocab) {
  griddep_wait();
  griddep_launch_dependents();
  for (int i = blockIdx.x * blockDim.x + threadIdx.x; i < n; i += gridDim.x * blockDim.x)
    dst[i] = min(max(src[i], 0), vocab - 1);
}
cudaError_t launch_token_patch(int32_t* dst, const int32_t* src, int n, int vocab, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(token_patch_kernel, dim3((n + 255) / 256), dim3(256), 0, st, dst, src, n, vocab);
}
cudaError_t launch_embed_rmsnorm(const int32_t* tokens, const void* emb, const void* g, float* resid, void* out,
                                 int T, int d, float eps, cudaStream_t st) {
  if (T == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(embed_rmsnorm_kernel, dim3(T), dim3(kRowThreads), 0, st, tokens, (const __nv_bfloat16*)emb, (const __nv_bfloat16*)g, resid,
                                                  (__nv_bfloat16*)out, d, eps);
}
cudaError_t launch_rmsnorm(const float* x, const void* g, void* out, int T, int d, float eps, cudaStream_t st) {
  if (T == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(rmsnorm_kernel, dim3(T), dim3(kRowThreads), 0, st, x, (const __nv_bfloat16*)g, (__nv_bfloat16*)out, d, eps);
}
cudaError_t launch_gather_rmsnorm(const float* x, const int32_t* rows, const void* g, void* out, int R, int d,
                                  float eps, cudaStream_t st) {
  if (R == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(gather_rmsnorm_kernel, dim3(R), dim3(kRowThreads), 0, st, x, rows, (const __nv_bfloat16*)g, (__nv_bfloat16*)out, d, eps);
}
cudaError_t launch_add_rmsnorm(float* resid, const void* add, const void* g, void* out, int T, int d, float eps,
                               cudaStream_t st) {
  if (T == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(add_rmsnorm_kernel, dim3(T), dim3(kRowThreads), 0, st, resid, (const __nv_bfloat16*)add, (const __nv_bfloat16*)g,
                                                (__nv_bfloat16*)out, d, eps);
}
cudaError_t launch_add_f32(float* resid, const void* add_bf16, size_t n, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(add_f32_kernel, dim3(grid_of(int64_t(n))), dim3(256), 0, st, resid, (const __nv_bfloat16*)add_bf16, int64_t(n));
}
cudaError_t launch_peer_add_rmsnorm(const PeerPtrs& parts, int tp, float* resid, const void* g, void* out, int T, int d,
                                    float eps, cudaStream_t st) {
  if (T == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(peer_add_rmsnorm_kernel, dim3(T), dim3(kRowThreads), 0, st, parts, tp, resid,
                    (const __nv_bfloat16*)g, (__nv_bfloat16*)out, d, eps);
}
cudaError_t launch_peer_rs_norm_ag(const PeerPtrs& parts, const PeerPtrs& hs, const PeerPtrs& resids, int tp, int rank,
                                   int row0, int nrows, const void* g, int d, float eps, cudaStream_t st) {
  if (nrows <= 0) return cudaSuccess;
  count_launch();
  return launch_pdl(peer_rs_norm_ag_kernel, dim3(nrows), dim3(kRowThreads), 0, st, parts, hs, resids, tp, rank, row0,
                    (const __nv_bfloat16*)g, d, eps);
}
cudaError_t launch_peer_gather_logits(const PeerPtrs& loc, int tp, int R, int Vl, float* out, cudaStream_t st) {
  if (R == 0) return cudaSuccess;
  count_launch();
  return launch_pdl(peer_gather_logits_kernel, dim3(grid_of(int64_t(R) * Vl * tp)), dim3(256), 0, st, loc, tp, R, Vl,
                    out);
}
cudaError_t launch_unshard_logits(const float* in, float* out, int R, int Vl, int tp, cudaStream_t st) {
  count_launch();
  return launch_pdl(unshard_logits_kernel, dim3(grid_of(int64_t(R) * Vl * tp)), dim3(256), 0, st, in, out, R, Vl, tp);
}
cudaError_t launch_argmax(const void* logits, int logits_f32, int R, int V, int32_t* out, cudaStream_t st,
                          float2* part, int* cnt) {
  if (R == 0) return cudaSuccess;
  count_launch();
  // slices per row: fill about two CTAs per SM (R = 129 logit rows -> 3 slices of ~43k entries)
  int S = part && cnt ? std::max(1, std::min(kArgmaxMaxSlices, (2 * 148 + R - 1) / R)) : 1;
  return launch_pdl(argmax_kernel, dim3(R, S), dim3(512), 0, st, logits, logits_f32, V, out, part, cnt);
}
cudaError_t launch_f32_to_bf16(const float* x, void* y, int64_t n, cudaStream_t st) {
  if (n == 0) return cudaSuccess;
  count_launch();
  const int blocks = int((n + 1023) / 1024 < 4096 ? (n + 1023) / 1024 : 4096);
  return launch_pdl(f32_to_bf16_kernel, dim3(blocks), dim3(1024), 0, st, x, (__nv_bfloat16*)y, n);
}

}  // namespace qos
