// attention.cu — paged attention of the hybrid batch.
//
// Both kernels read K/V straight from the paged cache (layout [L][K|V][block][Hkv][16][hd],
// one 16-token block of one kv head = 16 x hd bf16 contiguous) with TMA: a 3-D tensor map over
// the whole pool (dims {hd, blocks*Hkv*16, L*2}, box {64, 16, 1}, 128-B swizzle), so every
// (block, head) tile lands bank-conflict-free for ldmatrix.  A producer warp keeps a ring of
// 8 block-stages in flight (full/empty mbarriers); consumer warps run flash-attention style
// online softmax (fp32, exp2) with m16n8k16 tensor-core MMAs (Q K^T in bf16; P V in fp16:
// V is cached in fp16, P rounded to fp16).
//
//  * decode (a8): split-K.  Work item = (decode row, kv head, key range).  The MMAs are
//    transposed so the 16 keys of a paged block are the M rows and the GQA group (<= 8 query
//    heads) is the N = 8 columns: S^T = K Q^T, O^T += V^T P^T (P^T moved into B-fragment
//    layout with movmatrix).  The 4 consumer warps take interleaved blocks of the item and are
//    merged in smem; the last split of a (row, kv head) merges the splits (LSE merge).
//    decode_attn_persist_kernel (option decode_persist, measured slower at small steps) runs the
//    same item body in persistent CTAs.
//  (prefill attention (a7) lives in attention_tc.cu on tcgen05/TMEM.)
// HBM bytes per decode key = 2 * hd * 2 (K + V) per kv head: the kernel is bandwidth-bound.
#include <algorithm>
#include <cfloat>

#include "common.cuh"
#include "internal.h"

namespace qos {

constexpr int kConsumerWarps = 4;
constexpr int kAttnThreads = (kConsumerWarps + 1) * 32;
// Block i goes to consumer warp i % kConsumerWarps and ring stage i % NS (NS = ring depth, 8 or
// 4).  With a multiple, stage s is always consumed by the same warp, in order, so no waiter can
// run a full phase ahead of an mbarrier (parity waits would then alias).

template <int HD, int NS>
struct AttnCfg {
  static_assert(NS % kConsumerWarps == 0, "ring depth must be a multiple of the consumer warps");
  static constexpr int kBlockBytes = 16 * HD * 2;     // one (block, head) tile
  static constexpr int kStageBytes = 2 * kBlockBytes; // K + V
  static constexpr int kHalves = HD / 64;
  static constexpr int kNT = HD / 8;                  // n-tiles of the output (8 dims each)
  static constexpr int kKS = HD / 16;                 // k-steps of Q K^T
  static constexpr int kSmemBytes = NS * kStageBytes + 1024 + 2 * NS * 8 + 64;
};

struct AttnParams {
  const __nv_bfloat16* q;
  int q_ld;
  void* out;
  int out_ld;
  int out_f32;
  int layer, H, Hkv;
  const int32_t* tables;
  int table_w;
  float scale_log2;
};

// byte offset of 16-B chunk `ch` of key row `kr` inside a swizzled (block, head) tile
QOS_DEV uint32_t tile_off(int kr, int ch) {
  return uint32_t((ch >> 3) * 2048 + kr * 128 + (((ch & 7) ^ (kr & 7)) << 4));
}

template <int HD>
QOS_DEV void issue_block_load(const CUtensorMap* map, uint8_t* stage, uint64_t* bar, int layer, int row) {
  using C = AttnCfg<HD, 4>;
#pragma unroll
  for (int h = 0; h < C::kHalves; ++h) {
    tma_load_3d(stage + h * 2048, map, bar, h * 64, row, layer * 2 + 0);
    tma_load_3d(stage + C::kBlockBytes + h * 2048, map, bar, h * 64, row, layer * 2 + 1);
  }
}


QOS_DEV uint32_t movmatrix_trans(uint32_t x) {
  uint32_t y;
  asm volatile("movmatrix.sync.aligned.m8n8.trans.b16 %0, %1;" : "=r"(y) : "r"(x));
  return y;
}

// S^T[16 keys][8 heads] = K[16][HD] · Q^T[HD][8]   (A = K from smem, B = Q^T from registers)
template <int HD>
QOS_DEV void qk_block_t(const uint32_t (&qb)[HD / 16][2], uint32_t ktile, int lane, float (&s)[4]) {
  s[0] = s[1] = s[2] = s[3] = 0.f;
  const int kr = (lane & 7) + ((lane >> 3) & 1) * 8;
  const int csel = lane >> 4;
#pragma unroll
  for (int ks = 0; ks < HD / 16; ++ks) {
    uint32_t a[4];
    ldmatrix_x4(ktile + tile_off(kr, 2 * ks + csel), a[0], a[1], a[2], a[3]);
    mma_bf16_16816(s, a, qb[ks][0], qb[ks][1]);
  }
}

// O^T[HD][8] += V^T[HD][16 keys] · P^T[16 keys][8]   (A = V^T via ldmatrix.trans, B = P^T;
// fp16 operands: V is cached in fp16 and P is rounded to fp16, 2^-11 relative)
template <int HD>
QOS_DEV void pv_block_t(uint32_t b0, uint32_t b1, uint32_t vtile, int lane, float (&o)[HD / 16][4]) {
  const int kr = (lane & 7) + (lane >> 4) * 8;
  const int csel = (lane >> 3) & 1;
#pragma unroll
  for (int md = 0; md < HD / 16; ++md) {
    uint32_t a[4];
    ldmatrix_x4_trans(vtile + tile_off(kr, 2 * md + csel), a[0], a[1], a[2], a[3]);
    mma_f16_16816(o[md], a, b0, b1);
  }
}

// ------------------------------------------------------------------------------ decode
template <int HD, int NS>
__global__ void __launch_bounds__(kAttnThreads, 3)
    decode_attn_kernel(const __grid_constant__ CUtensorMap kvmap, const AttnParams p, const DecodeItem* __restrict__ items,
                       float* __restrict__ partials, int* __restrict__ counters) {
  using C = AttnCfg<HD, NS>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * C::kStageBytes);
  uint64_t* empty = full + NS;

  griddep_wait();  // q and the appended K/V come from the previous kernel
  griddep_launch_dependents();
  const DecodeItem it = items[blockIdx.x];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int group = p.H / p.Hkv;
  const int blk0 = it.key0 >> 4;
  const int nblk = ((it.key1 + 15) >> 4) - blk0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    fence_mbar_init();
  }
  __syncthreads();

  if (warp == kConsumerWarps) {
    if (elect_one()) {
      tma_prefetch_desc(&kvmap);
      const int32_t* trow = p.tables + size_t(it.table) * p.table_w;
      for (int i = 0; i < nblk; ++i) {
        const int s = i % NS;
        const uint32_t ph = (i / NS) & 1;
        mbar_wait(&empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&full[s], C::kStageBytes);
        const int block = __ldg(trow + blk0 + i);
        issue_block_load<HD>(&kvmap, smem + s * C::kStageBytes, &full[s], p.layer,
                             (block * p.Hkv + it.kv_head) * 16);
      }
    }
  }

  // per-warp state: thread (g, t) owns keys g, g+8 of each block and heads 2t, 2t+1
  const int g = lane >> 2, t = lane & 3;
  float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
  float o[HD / 16][4];
  if (warp < kConsumerWarps) {
#pragma unroll
    for (int md = 0; md < HD / 16; ++md) o[md][0] = o[md][1] = o[md][2] = o[md][3] = 0.f;
    // B fragments of Q^T: (dims 2t.., head g) — zero for heads >= group
    uint32_t qb[HD / 16][2];
    const __nv_bfloat16* qh = p.q + size_t(it.row) * p.q_ld + size_t(it.kv_head * group + g) * HD;
#pragma unroll
    for (int ks = 0; ks < HD / 16; ++ks) {
      qb[ks][0] = g < group ? *reinterpret_cast<const uint32_t*>(qh + ks * 16 + 2 * t) : 0u;
      qb[ks][1] = g < group ? *reinterpret_cast<const uint32_t*>(qh + ks * 16 + 2 * t + 8) : 0u;
    }
    for (int i = warp; i < nblk; i += kConsumerWarps) {
      const int s = i % NS;
      const uint32_t ph = (i / NS) & 1;
      mbar_wait(&full[s], ph);
      const uint32_t kt = smem_u32(smem + s * C::kStageBytes);
      float sc[4];
      qk_block_t<HD>(qb, kt, lane, sc);
      const int kbase = (blk0 + i) * 16;
      const bool v0 = kbase + g < it.key1, v1 = kbase + g + 8 < it.key1;
      // scores (log2 units); c0,c2 -> head 2t (keys g, g+8); c1,c3 -> head 2t+1
      const float s0 = v0 ? sc[0] * p.scale_log2 : -INFINITY, s1 = v0 ? sc[1] * p.scale_log2 : -INFINITY;
      const float s2 = v1 ? sc[2] * p.scale_log2 : -INFINITY, s3 = v1 ? sc[3] * p.scale_log2 : -INFINITY;
      float mx0 = fmaxf(m[0], fmaxf(s0, s2)), mx1 = fmaxf(m[1], fmaxf(s1, s3));
#pragma unroll
      for (int off = 4; off < 32; off <<= 1) {
        mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, off));
        mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, off));
      }
      const float b0 = (mx0 == -INFINITY) ? 0.f : mx0, b1 = (mx1 == -INFINITY) ? 0.f : mx1;
      const float a0 = exp2f(m[0] - b0), a1 = exp2f(m[1] - b1);
      m[0] = mx0;
      m[1] = mx1;
      const float p0 = exp2f(s0 - b0), p1 = exp2f(s1 - b1), p2 = exp2f(s2 - b0), p3 = exp2f(s3 - b1);
      l[0] = l[0] * a0 + p0 + p2;
      l[1] = l[1] * a1 + p1 + p3;
#pragma unroll
      for (int md = 0; md < HD / 16; ++md) {
        o[md][0] *= a0;
        o[md][1] *= a1;
        o[md][2] *= a0;
        o[md][3] *= a1;
      }
      // P^T as B fragments: transpose the two 8x8 (keys x heads) halves of fp16 P
      pv_block_t<HD>(movmatrix_trans(pack_f16(p0, p1)), movmatrix_trans(pack_f16(p2, p3)), kt + C::kBlockBytes, lane, o);
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
    }
#pragma unroll
    for (int off = 4; off < 32; off <<= 1) {
      l[0] += __shfl_xor_sync(0xffffffffu, l[0], off);
      l[1] += __shfl_xor_sync(0xffffffffu, l[1], off);
    }
  }
  __syncthreads();  // every stage consumed; the ring is free for the merge
  // merge area: o [warp][head 8][HD], m [warp][8], l [warp][8]
  float* so = reinterpret_cast<float*>(smem);
  float* sm = so + kConsumerWarps * 8 * HD;
  float* sl = sm + kConsumerWarps * 8;
  if (warp < kConsumerWarps) {
#pragma unroll
    for (int md = 0; md < HD / 16; ++md) {
      so[(warp * 8 + 2 * t) * HD + md * 16 + g] = o[md][0];
      so[(warp * 8 + 2 * t + 1) * HD + md * 16 + g] = o[md][1];
      so[(warp * 8 + 2 * t) * HD + md * 16 + g + 8] = o[md][2];
      so[(warp * 8 + 2 * t + 1) * HD + md * 16 + g + 8] = o[md][3];
    }
    if (g == 0) {
      sm[warp * 8 + 2 * t] = m[0];
      sm[warp * 8 + 2 * t + 1] = m[1];
      sl[warp * 8 + 2 * t] = l[0];
      sl[warp * 8 + 2 * t + 1] = l[1];
    }
  }
  __syncthreads();
  auto merged = [&](int r, int d, float& M, float& L) {
    M = -INFINITY;
#pragma unroll
    for (int w = 0; w < kConsumerWarps; ++w) M = fmaxf(M, sm[w * 8 + r]);
    float acc = 0.f;
    L = 0.f;
#pragma unroll
    for (int w = 0; w < kConsumerWarps; ++w) {
      const float mw = sm[w * 8 + r];
      const float f = (mw == -INFINITY) ? 0.f : exp2f(mw - M);
      acc += f * so[(w * 8 + r) * HD + d];
      L += f * sl[w * 8 + r];
    }
    return acc;
  };
  auto store_out = [&](int r, int d, float v) {
    const size_t off = size_t(it.row) * p.out_ld + size_t(it.kv_head * group + r) * HD + d;
    if (p.out_f32)
      reinterpret_cast<float*>(p.out)[off] = v;
    else
      reinterpret_cast<__nv_bfloat16*>(p.out)[off] = __float2bfloat16_rn(v);
  };
  if (it.nsplit == 1) {  // the whole key range in one item: normalise and store
    for (int idx = threadIdx.x; idx < group * HD; idx += blockDim.x) {
      float M, L;
      const float acc = merged(idx / HD, idx % HD, M, L);
      store_out(idx / HD, idx % HD, acc / L);
    }
    return;
  }
  float* part = partials + size_t(it.part) * group * (HD + 2);
  for (int idx = threadIdx.x; idx < group * HD; idx += blockDim.x) {
    const int r = idx / HD, d = idx % HD;
    float M, L;
    const float acc = merged(r, d, M, L);
    part[r * (HD + 2) + d] = acc;
    if (d == 0) {
      part[r * (HD + 2) + HD] = M;
      part[r * (HD + 2) + HD + 1] = L;
    }
  }
  // split-K combine fused into the last finishing item of this (decode row, kv head):
  // out = sum_s 2^(m_s - M) o_s / sum_s 2^(m_s - M) l_s   (LSE merge)
  __syncthreads();
  __shared__ int s_last;
  if (threadIdx.x == 0) {
    // release: this CTA's partial (ordered before by the barrier) is visible before the count;
    // acquire: the last arriver sees every other split's partial
    int prev;
    asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], 1;" : "=r"(prev) : "l"(counters + it.counter) : "memory");
    s_last = (prev == it.nsplit - 1);
  }
  __syncthreads();
  if (!s_last) return;
  const size_t stride = size_t(group) * (HD + 2);
  const float* pb = partials + size_t(it.part_base) * stride;
  for (int idx = threadIdx.x; idx < group * HD; idx += blockDim.x) {
    const int r = idx / HD, d = idx % HD;
    float M = -INFINITY;
    for (int s2 = 0; s2 < it.nsplit; ++s2) M = fmaxf(M, __ldcg(pb + s2 * stride + r * (HD + 2) + HD));
    float L = 0.f, acc = 0.f;
    for (int s2 = 0; s2 < it.nsplit; ++s2) {
      const float* ps = pb + s2 * stride + r * (HD + 2);
      const float f = exp2f(__ldcg(ps + HD) - M);
      L += f * __ldcg(ps + HD + 1);
      acc += f * __ldcg(ps + d);
    }
    store_out(r, d, acc / L);
  }
  if (threadIdx.x == 0) counters[it.counter] = 0;  // ready for the next layer
}

// ------------------------------------------------------------------------------ decode, persistent
// The kernel above as persistent CTAs (option decode_persist): CTA c runs items c, c + G,
// c + 2G, ... of the longest-first list (round-robin over a descending list: LPT-like).  The
// ring's stage / phase and the block -> consumer-warp assignment run on a per-CTA cumulative
// block count, so the producer streams the next item's blocks while the consumer warps merge
// and store the current one (their merge area is separate from the ring), and an item costs no
// CTA launch, barrier setup or pipeline fill.  Aimed at decode-heavy small steps, whose short
// key ranges (a 16-decode step at ctx 1k: 1024 items of 8 blocks) are latency-bound, not
// HBM-bound.
constexpr int kPersistMergeBytes = kConsumerWarps * 8 * 128 * 4 + 2 * kConsumerWarps * 8 * 4;

template <int HD, int NS>
__global__ void __launch_bounds__(kAttnThreads, 2)
    decode_attn_persist_kernel(const __grid_constant__ CUtensorMap kvmap, const AttnParams p,
                               const DecodeItem* __restrict__ items, int n_items, float* __restrict__ partials,
                               int* __restrict__ counters) {
  using C = AttnCfg<HD, NS>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + NS * C::kStageBytes);
  uint64_t* empty = full + NS;
  float* so = reinterpret_cast<float*>(smem + NS * C::kStageBytes + 2 * NS * 8 + 64);  // merge area
  float* sm = so + kConsumerWarps * 8 * HD;
  float* sl = sm + kConsumerWarps * 8;
  __shared__ int s_last;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int group = p.H / p.Hkv;
  if (threadIdx.x == 0) {
    for (int s = 0; s < NS; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    fence_mbar_init();
  }
  if (warp == kConsumerWarps && lane == 0) tma_prefetch_desc(&kvmap);
  __syncthreads();
  griddep_wait();  // q and the appended K/V come from the previous kernel
  griddep_launch_dependents();

  if (warp == kConsumerWarps) {
    // ------------------------------------------------------------ producer: every item's blocks
    if (elect_one()) {
      uint32_t gb = 0;  // cumulative block count of this CTA
      for (int ii = blockIdx.x; ii < n_items; ii += gridDim.x) {
        const DecodeItem it = items[ii];
        const int blk0 = it.key0 >> 4, nblk = ((it.key1 + 15) >> 4) - blk0;
        const int32_t* trow = p.tables + size_t(it.table) * p.table_w + blk0;
        for (int i = 0; i < nblk; ++i, ++gb) {
          const int s = int(gb % NS);
          const uint32_t ph = (gb / NS) & 1;
          const int block = __ldg(trow + i);
          mbar_wait(&empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&full[s], C::kStageBytes);
          issue_block_load<HD>(&kvmap, smem + s * C::kStageBytes, &full[s], p.layer, (block * p.Hkv + it.kv_head) * 16);
        }
      }
    }
    return;
  }
  // ---------------------------------------------------------------- consumers (4 warps, 128 threads)
  auto cbar = []() { asm volatile("bar.sync 1, 128;" ::: "memory"); };
  const int g = lane >> 2, t = lane & 3;
  uint32_t gb = 0;
  for (int ii = blockIdx.x; ii < n_items; ii += gridDim.x) {
    const DecodeItem it = items[ii];
    const int blk0 = it.key0 >> 4, nblk = ((it.key1 + 15) >> 4) - blk0;
    float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
    float o[HD / 16][4];
#pragma unroll
    for (int md = 0; md < HD / 16; ++md) o[md][0] = o[md][1] = o[md][2] = o[md][3] = 0.f;
    uint32_t qb[HD / 16][2];
    const __nv_bfloat16* qh = p.q + size_t(it.row) * p.q_ld + size_t(it.kv_head * group + g) * HD;
#pragma unroll
    for (int ks = 0; ks < HD / 16; ++ks) {
      qb[ks][0] = g < group ? *reinterpret_cast<const uint32_t*>(qh + ks * 16 + 2 * t) : 0u;
      qb[ks][1] = g < group ? *reinterpret_cast<const uint32_t*>(qh + ks * 16 + 2 * t + 8) : 0u;
    }
    // block i of the item is cumulative block gb + i: stage (gb + i) % NS, warp (gb + i) % 4
    for (int i = int((uint32_t(warp) - gb) & (kConsumerWarps - 1)); i < nblk; i += kConsumerWarps) {
      const uint32_t gi = gb + uint32_t(i);
      const int s = int(gi % NS);
      const uint32_t ph = (gi / NS) & 1;
      mbar_wait(&full[s], ph);
      const uint32_t kt = smem_u32(smem + s * C::kStageBytes);
      float sc[4];
      qk_block_t<HD>(qb, kt, lane, sc);
      const int kbase = (blk0 + i) * 16;
      const bool v0 = kbase + g < it.key1, v1 = kbase + g + 8 < it.key1;
      const float s0 = v0 ? sc[0] * p.scale_log2 : -INFINITY, s1 = v0 ? sc[1] * p.scale_log2 : -INFINITY;
      const float s2 = v1 ? sc[2] * p.scale_log2 : -INFINITY, s3 = v1 ? sc[3] * p.scale_log2 : -INFINITY;
      float mx0 = fmaxf(m[0], fmaxf(s0, s2)), mx1 = fmaxf(m[1], fmaxf(s1, s3));
#pragma unroll
      for (int off = 4; off < 32; off <<= 1) {
        mx0 = fmaxf(mx0, __shfl_xor_sync(0xffffffffu, mx0, off));
        mx1 = fmaxf(mx1, __shfl_xor_sync(0xffffffffu, mx1, off));
      }
      const float b0 = (mx0 == -INFINITY) ? 0.f : mx0, b1 = (mx1 == -INFINITY) ? 0.f : mx1;
      const float a0 = exp2f(m[0] - b0), a1 = exp2f(m[1] - b1);
      m[0] = mx0;
      m[1] = mx1;
      const float p0 = exp2f(s0 - b0), p1 = exp2f(s1 - b1), p2 = exp2f(s2 - b0), p3 = exp2f(s3 - b1);
      l[0] = l[0] * a0 + p0 + p2;
      l[1] = l[1] * a1 + p1 + p3;
#pragma unroll
      for (int md = 0; md < HD / 16; ++md) {
        o[md][0] *= a0;
        o[md][1] *= a1;
        o[md][2] *= a0;
        o[md][3] *= a1;
      }
      pv_block_t<HD>(movmatrix_trans(pack_f16(p0, p1)), movmatrix_trans(pack_f16(p2, p3)), kt + C::kBlockBytes, lane, o);
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
    }
    gb += uint32_t(nblk);
#pragma unroll
    for (int off = 4; off < 32; off <<= 1) {
      l[0] += __shfl_xor_sync(0xffffffffu, l[0], off);
      l[1] += __shfl_xor_sync(0xffffffffu, l[1], off);
    }
    cbar();  // the previous item's merge has read the merge area
#pragma unroll
    for (int md = 0; md < HD / 16; ++md) {
      so[(warp * 8 + 2 * t) * HD + md * 16 + g] = o[md][0];
      so[(warp * 8 + 2 * t + 1) * HD + md * 16 + g] = o[md][1];
      so[(warp * 8 + 2 * t) * HD + md * 16 + g + 8] = o[md][2];
      so[(warp * 8 + 2 * t + 1) * HD + md * 16 + g + 8] = o[md][3];
    }
    if (g == 0) {
      sm[warp * 8 + 2 * t] = m[0];
      sm[warp * 8 + 2 * t + 1] = m[1];
      sl[warp * 8 + 2 * t] = l[0];
      sl[warp * 8 + 2 * t + 1] = l[1];
    }
    cbar();
    auto merged = [&](int r, int d, float& M, float& L) {
      M = -INFINITY;
#pragma unroll
      for (int w = 0; w < kConsumerWarps; ++w) M = fmaxf(M, sm[w * 8 + r]);
      float acc = 0.f;
      L = 0.f;
#pragma unroll
      for (int w = 0; w < kConsumerWarps; ++w) {
        const float mw = sm[w * 8 + r];
        const float f = (mw == -INFINITY) ? 0.f : exp2f(mw - M);
        acc += f * so[(w * 8 + r) * HD + d];
        L += f * sl[w * 8 + r];
      }
      return acc;
    };
    auto store_out = [&](int r, int d, float v) {
      const size_t off = size_t(it.row) * p.out_ld + size_t(it.kv_head * group + r) * HD + d;
      if (p.out_f32)
        reinterpret_cast<float*>(p.out)[off] = v;
      else
        reinterpret_cast<__nv_bfloat16*>(p.out)[off] = __float2bfloat16_rn(v);
    };
    if (it.nsplit == 1) {
      for (int idx = threadIdx.x; idx < group * HD; idx += kConsumerWarps * 32) {
        float M, L;
        const float acc = merged(idx / HD, idx % HD, M, L);
        store_out(idx / HD, idx % HD, acc / L);
      }
      continue;
    }
    float* part = partials + size_t(it.part) * group * (HD + 2);
    for (int idx = threadIdx.x; idx < group * HD; idx += kConsumerWarps * 32) {
      const int r = idx / HD, d = idx % HD;
      float M, L;
      const float acc = merged(r, d, M, L);
      part[r * (HD + 2) + d] = acc;
      if (d == 0) {
        part[r * (HD + 2) + HD] = M;
        part[r * (HD + 2) + HD + 1] = L;
      }
    }
    cbar();
    if (threadIdx.x == 0) {
      int prev;
      asm volatile("atom.acq_rel.gpu.global.add.s32 %0, [%1], 1;" : "=r"(prev) : "l"(counters + it.counter) : "memory");
      s_last = (prev == it.nsplit - 1);
    }
    cbar();
    if (!s_last) continue;
    const size_t stride = size_t(group) * (HD + 2);
    const float* pb = partials + size_t(it.part_base) * stride;
    for (int idx = threadIdx.x; idx < group * HD; idx += kConsumerWarps * 32) {
      const int r = idx / HD, d = idx % HD;
      float M = -INFINITY;
      for (int s2 = 0; s2 < it.nsplit; ++s2) M = fmaxf(M, __ldcg(pb + s2 * stride + r * (HD + 2) + HD));
      float L = 0.f, acc = 0.f;
      for (int s2 = 0; s2 < it.nsplit; ++s2) {
        const float* ps = pb + s2 * stride + r * (HD + 2);
        const float f = exp2f(__ldcg(ps + HD) - M);
        L += f * __ldcg(ps + HD + 1);
        acc += f * __ldcg(ps + d);
      }
      store_out(r, d, acc / L);
    }
    if (threadIdx.x == 0) counters[it.counter] = 0;  // ready for the next layer
  }
}

// ------------------------------------------------------------------------------ host
static AttnParams to_params(const AttnLaunch& a) {
  AttnParams p;
  p.q = reinterpret_cast<const __nv_bfloat16*>(a.q);
  p.q_ld = a.q_ld;
  p.out = a.out;
  p.out_ld = a.out_ld;
  p.out_f32 = a.out_f32;
  p.layer = a.layer;
  p.H = a.H;
  p.Hkv = a.Hkv;
  p.tables = a.tables;
  p.table_w = a.table_w;
  p.scale_log2 = a.scale_log2;
  return p;
}

template <int HD, int NS>
static cudaError_t decode_t(const AttnLaunch& a, const DecodeItem* items, int n_items, float* partials, int* counters,
                            cudaStream_t st) {
  static std::atomic<uint64_t> set{0};
  if (cudaError_t e = smem_attr_once(decode_attn_kernel<HD, NS>, int(AttnCfg<HD, NS>::kSmemBytes), set); e != cudaSuccess) return e;
  return launch_pdl(decode_attn_kernel<HD, NS>, dim3(n_items), dim3(kAttnThreads), AttnCfg<HD, NS>::kSmemBytes, st,
                    *a.kv_tmap, to_params(a), items, partials, counters);
}

template <int HD, int NS>
static cudaError_t decode_persist_t(const AttnLaunch& a, const DecodeItem* items, int n_items, float* partials,
                                    int* counters, cudaStream_t st) {
  constexpr int smem = AttnCfg<HD, NS>::kSmemBytes + kPersistMergeBytes;
  auto kern = decode_attn_persist_kernel<HD, NS>;
  static std::atomic<uint64_t> set{0};
  if (cudaError_t e = smem_attr_once(kern, smem, set); e != cudaSuccess) return e;
  int dev = 0, sms = 0, per_sm = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  if (cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kern, kAttnThreads, smem); e != cudaSuccess)
    return e;
  const int grid = std::min(n_items, std::max(1, per_sm) * sms);
  return launch_pdl(kern, dim3(grid), dim3(kAttnThreads), smem, st, *a.kv_tmap, to_params(a), items, n_items, partials,
                    counters);
}

cudaError_t launch_decode_attention(const AttnLaunch& a, const DecodeItem* items, int n_items, float* partials,
                                    int* counters, cudaStream_t st) {
  if (n_items == 0) return cudaSuccess;
  count_launch(1);
  if (a.decode_persist) {
    if (a.hd == 128) return decode_persist_t<128, 8>(a, items, n_items, partials, counters, st);
    if (a.hd == 64) return decode_persist_t<64, 8>(a, items, n_items, partials, counters, st);
    return cudaErrorInvalidValue;
  }
  if (a.hd == 128)
    return a.decode_stages == 4 ? decode_t<128, 4>(a, items, n_items, partials, counters, st)
                                : decode_t<128, 8>(a, items, n_items, partials, counters, st);
  if (a.hd == 64)
    return a.decode_stages == 4 ? decode_t<64, 4>(a, items, n_items, partials, counters, st)
                                : decode_t<64, 8>(a, items, n_items, partials, counters, st);
  return cudaErrorInvalidValue;
}

}  // namespace qos
