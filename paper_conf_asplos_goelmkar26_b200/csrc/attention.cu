// attention.cu — paged attention of the hybrid batch.
//
// Both kernels read K/V straight from the paged cache (layout [L][K|V][block][Hkv][16][hd],
// one 16-token block of one kv head = 16 x hd bf16 contiguous) with TMA: a 3-D tensor map over
// the whole pool (dims {hd, blocks*Hkv*16, L*2}, box {64, 16, 1}, 128-B swizzle), so every
// (block, head) tile lands bank-conflict-free for ldmatrix.  A producer warp keeps a ring of
// 8 block-stages in flight (full/empty mbarriers); consumer warps run flash-attention style
// online softmax (fp32, exp2) with m16n8k16 bf16 tensor-core MMAs.
//
//  * decode (a8): split-K.  Work item = (decode row, kv head, key range).  The GQA group of
//    H/Hkv query heads forms the M=16 rows of the MMA (rows >= group are zero); the 4
//    consumer warps take interleaved key blocks of the item and are merged in smem; each item
//    writes an (o, m, l) partial and decode_combine merges the splits (LSE merge).
//  * prefill (a7): work item = (chunk, tile of positions, kv head); rows = (position, head in
//    group) pairs (16 per warp), every warp walks the causal key range [0, last pos] and skips
//    blocks that lie entirely in its future.
// HBM bytes per decode key = 2 * hd * 2 (K + V) per kv head: the kernel is bandwidth-bound.
#include <cfloat>

#include "common.cuh"
#include "internal.h"

namespace qos {

constexpr int kAttnStages = 8;
constexpr int kConsumerWarps = 4;
constexpr int kAttnThreads = (kConsumerWarps + 1) * 32;

template <int HD>
struct AttnCfg {
  static constexpr int kBlockBytes = 16 * HD * 2;     // one (block, head) tile
  static constexpr int kStageBytes = 2 * kBlockBytes; // K + V
  static constexpr int kHalves = HD / 64;
  static constexpr int kNT = HD / 8;                  // n-tiles of the output (8 dims each)
  static constexpr int kKS = HD / 16;                 // k-steps of Q K^T
  static constexpr int kSmemBytes = kAttnStages * kStageBytes + 1024 + 2 * kAttnStages * 8 + 64;
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
  using C = AttnCfg<HD>;
#pragma unroll
  for (int h = 0; h < C::kHalves; ++h) {
    tma_load_3d(stage + h * 2048, map, bar, h * 64, row, layer * 2 + 0);
    tma_load_3d(stage + C::kBlockBytes + h * 2048, map, bar, h * 64, row, layer * 2 + 1);
  }
}

// S[16 rows][16 keys] = Q · K^T for one key block (two n-tiles of 8 keys)
template <int HD>
QOS_DEV void qk_block(const uint32_t (&qa)[HD / 16][4], uint32_t ktile, int lane, float (&s)[2][4]) {
#pragma unroll
  for (int j = 0; j < 2; ++j)
#pragma unroll
    for (int e = 0; e < 4; ++e) s[j][e] = 0.f;
  const int kr = ((lane >> 4) << 3) + (lane & 7);
  const int csel = (lane >> 3) & 1;
#pragma unroll
  for (int ks = 0; ks < HD / 16; ++ks) {
    uint32_t b0, b1, b2, b3;
    ldmatrix_x4(ktile + tile_off(kr, 2 * ks + csel), b0, b1, b2, b3);
    mma_bf16_16816(s[0], qa[ks], b0, b1);
    mma_bf16_16816(s[1], qa[ks], b2, b3);
  }
}

// O[16 rows][HD] += P[16][16 keys] · V[16 keys][HD], with P carried as two bf16 terms
// (P = P_hi + P_lo): the products with the bf16 V are then exact to ~2^-16, so the fp32 output
// meets the 2e-3 attention tolerance (a single bf16 P alone leaves a 2^-9 rounding floor).
template <int HD>
QOS_DEV void pv_block(const uint32_t (&pa)[4], const uint32_t (&pl)[4], uint32_t vtile, int lane, float (&o)[HD / 8][4]) {
  const int kr = (((lane >> 3) & 1) << 3) + (lane & 7);
  const int csel = lane >> 4;
#pragma unroll
  for (int nd = 0; nd < HD / 16; ++nd) {
    uint32_t b0, b1, b2, b3;
    ldmatrix_x4_trans(vtile + tile_off(kr, 2 * nd + csel), b0, b1, b2, b3);
    mma_bf16_16816(o[2 * nd], pa, b0, b1);
    mma_bf16_16816(o[2 * nd + 1], pa, b2, b3);
    mma_bf16_16816(o[2 * nd], pl, b0, b1);
    mma_bf16_16816(o[2 * nd + 1], pl, b2, b3);
  }
}

// Load A fragments of Q for rows (ra, rb) of a 16-row MMA tile; null pointer = zero row.
template <int HD>
QOS_DEV void load_q_frags(const __nv_bfloat16* qa_row, const __nv_bfloat16* qb_row, int t, uint32_t (&qa)[HD / 16][4]) {
#pragma unroll
  for (int ks = 0; ks < HD / 16; ++ks) {
    const int c0 = ks * 16 + 2 * t;
    qa[ks][0] = qa_row ? *reinterpret_cast<const uint32_t*>(qa_row + c0) : 0u;
    qa[ks][1] = qb_row ? *reinterpret_cast<const uint32_t*>(qb_row + c0) : 0u;
    qa[ks][2] = qa_row ? *reinterpret_cast<const uint32_t*>(qa_row + c0 + 8) : 0u;
    qa[ks][3] = qb_row ? *reinterpret_cast<const uint32_t*>(qb_row + c0 + 8) : 0u;
  }
}

// One online-softmax step for the two rows a thread owns. s: raw scores (scaled inside).
// valid(j, e) decides masking. Updates m, l (per-thread partial), rescales o, returns P frags.
QOS_DEV void split_bf16(float a, float b, uint32_t& hi, uint32_t& lo) {
  hi = pack_bf16(a, b);
  lo = pack_bf16(a - bf16_lo(hi), b - bf16_hi(hi));
}

template <int HD, typename Valid>
QOS_DEV void softmax_step(float (&s)[2][4], float (&m)[2], float (&l)[2], float (&o)[HD / 8][4], float scale_log2,
                          Valid valid, uint32_t (&pa)[4], uint32_t (&pl)[4]) {
  float mx[2] = {m[0], m[1]};
#pragma unroll
  for (int j = 0; j < 2; ++j)
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float v = valid(j, e) ? s[j][e] * scale_log2 : -INFINITY;
      s[j][e] = v;
      mx[e >> 1] = fmaxf(mx[e >> 1], v);
    }
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 1));
    mx[r] = fmaxf(mx[r], __shfl_xor_sync(0xffffffffu, mx[r], 2));
  }
  float base[2], alpha[2];
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    base[r] = (mx[r] == -INFINITY) ? 0.f : mx[r];
    alpha[r] = exp2f(m[r] - base[r]);  // m = -inf -> 0
    m[r] = mx[r];
    l[r] *= alpha[r];
  }
#pragma unroll
  for (int j = 0; j < 2; ++j)
#pragma unroll
    for (int e = 0; e < 4; ++e) {
      const float p = exp2f(s[j][e] - base[e >> 1]);
      s[j][e] = p;
      l[e >> 1] += p;
    }
#pragma unroll
  for (int nt = 0; nt < HD / 8; ++nt) {
    o[nt][0] *= alpha[0];
    o[nt][1] *= alpha[0];
    o[nt][2] *= alpha[1];
    o[nt][3] *= alpha[1];
  }
  split_bf16(s[0][0], s[0][1], pa[0], pl[0]);
  split_bf16(s[0][2], s[0][3], pa[1], pl[1]);
  split_bf16(s[1][0], s[1][1], pa[2], pl[2]);
  split_bf16(s[1][2], s[1][3], pa[3], pl[3]);
}

// ------------------------------------------------------------------------------ decode
template <int HD>
__global__ void __launch_bounds__(kAttnThreads, 3)
    decode_attn_kernel(const __grid_constant__ CUtensorMap kvmap, const AttnParams p, const DecodeItem* __restrict__ items,
                       float* __restrict__ partials, int* __restrict__ counters) {
  using C = AttnCfg<HD>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kAttnStages * C::kStageBytes);
  uint64_t* empty = full + kAttnStages;

  const DecodeItem it = items[blockIdx.x];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int group = p.H / p.Hkv;
  const int blk0 = it.key0 >> 4;
  const int nblk = ((it.key1 + 15) >> 4) - blk0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < kAttnStages; ++s) {
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
        const int s = i % kAttnStages;
        const uint32_t ph = (i / kAttnStages) & 1;
        mbar_wait(&empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&full[s], C::kStageBytes);
        const int block = __ldg(trow + blk0 + i);
        issue_block_load<HD>(&kvmap, smem + s * C::kStageBytes, &full[s], p.layer,
                             (block * p.Hkv + it.kv_head) * 16);
      }
    }
  }

  // per-warp state, merged through smem at the end (region reuses the stage ring)
  float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
  float o[HD / 8][4];
  const int g = lane >> 2, t = lane & 3;
  if (warp < kConsumerWarps) {
#pragma unroll
    for (int nt = 0; nt < HD / 8; ++nt) o[nt][0] = o[nt][1] = o[nt][2] = o[nt][3] = 0.f;
    uint32_t qa[HD / 16][4];
    const __nv_bfloat16* qrow = p.q + size_t(it.row) * p.q_ld + size_t(it.kv_head * group) * HD;
    load_q_frags<HD>(g < group ? qrow + g * HD : nullptr, (g + 8) < group ? qrow + (g + 8) * HD : nullptr, t, qa);
    for (int i = warp; i < nblk; i += kConsumerWarps) {
      const int s = i % kAttnStages;
      const uint32_t ph = (i / kAttnStages) & 1;
      mbar_wait(&full[s], ph);
      const uint32_t kt = smem_u32(smem + s * C::kStageBytes);
      float sc[2][4];
      qk_block<HD>(qa, kt, lane, sc);
      const int kbase = (blk0 + i) * 16;
      uint32_t pa[4], pl[4];
      softmax_step<HD>(sc, m, l, o, p.scale_log2,
                       [&](int j, int e) { return kbase + 8 * j + 2 * t + (e & 1) < it.key1; }, pa, pl);
      pv_block<HD>(pa, pl, kt + C::kBlockBytes, lane, o);
      __syncwarp();
      if (lane == 0) mbar_arrive(&empty[s]);
    }
    l[0] += __shfl_xor_sync(0xffffffffu, l[0], 1);
    l[0] += __shfl_xor_sync(0xffffffffu, l[0], 2);
    l[1] += __shfl_xor_sync(0xffffffffu, l[1], 1);
    l[1] += __shfl_xor_sync(0xffffffffu, l[1], 2);
  }
  __syncthreads();  // every stage consumed; the ring is free for the merge
  // merge area: [warp][row<16][HD] o, then [warp][16] m, [warp][16] l
  float* so = reinterpret_cast<float*>(smem);
  float* sm = so + kConsumerWarps * 16 * HD;
  float* sl = sm + kConsumerWarps * 16;
  if (warp < kConsumerWarps) {
    if (g < group) {
#pragma unroll
      for (int nt = 0; nt < HD / 8; ++nt) {
        so[(warp * 16 + g) * HD + nt * 8 + 2 * t] = o[nt][0];
        so[(warp * 16 + g) * HD + nt * 8 + 2 * t + 1] = o[nt][1];
      }
      if (t == 0) {
        sm[warp * 16 + g] = m[0];
        sl[warp * 16 + g] = l[0];
      }
    }
    if (g + 8 < group) {
#pragma unroll
      for (int nt = 0; nt < HD / 8; ++nt) {
        so[(warp * 16 + g + 8) * HD + nt * 8 + 2 * t] = o[nt][2];
        so[(warp * 16 + g + 8) * HD + nt * 8 + 2 * t + 1] = o[nt][3];
      }
      if (t == 0) {
        sm[warp * 16 + g + 8] = m[1];
        sl[warp * 16 + g + 8] = l[1];
      }
    }
  }
  __syncthreads();
  // merge the 4 warps: (M, L, acc) per (row r < group, dim d)
  auto merged = [&](int r, int d, float& M, float& L) {
    M = -INFINITY;
#pragma unroll
    for (int w = 0; w < kConsumerWarps; ++w) M = fmaxf(M, sm[w * 16 + r]);
    float acc = 0.f;
    L = 0.f;
#pragma unroll
    for (int w = 0; w < kConsumerWarps; ++w) {
      const float mw = sm[w * 16 + r];
      const float f = (mw == -INFINITY) ? 0.f : exp2f(mw - M);
      acc += f * so[(w * 16 + r) * HD + d];
      L += f * sl[w * 16 + r];
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
  __threadfence();
  __syncthreads();
  __shared__ int s_last;
  if (threadIdx.x == 0) s_last = (atomicAdd(counters + it.counter, 1) == it.nsplit - 1);
  __syncthreads();
  if (!s_last) return;
  __threadfence();
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

// ------------------------------------------------------------------------------ prefill
template <int HD>
__global__ void __launch_bounds__(kAttnThreads)
    prefill_attn_kernel(const __grid_constant__ CUtensorMap kvmap, const AttnParams p,
                        const PrefillItem* __restrict__ items) {
  using C = AttnCfg<HD>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + kAttnStages * C::kStageBytes);
  uint64_t* empty = full + kAttnStages;

  const PrefillItem it = items[blockIdx.x];
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int group = p.H / p.Hkv;
  const int ppw = 16 / group;  // positions per warp
  const int last_pos = it.pos0 + it.npos - 1;
  const int nblk = (last_pos >> 4) + 1;

  if (threadIdx.x == 0) {
    for (int s = 0; s < kAttnStages; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], kConsumerWarps);
    }
    fence_mbar_init();
  }
  __syncthreads();

  if (warp == kConsumerWarps) {
    if (elect_one()) {
      tma_prefetch_desc(&kvmap);
      const int32_t* trow = p.tables + size_t(it.table) * p.table_w;
      for (int i = 0; i < nblk; ++i) {
        const int s = i % kAttnStages;
        const uint32_t ph = (i / kAttnStages) & 1;
        mbar_wait(&empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&full[s], C::kStageBytes);
        const int block = __ldg(trow + i);
        issue_block_load<HD>(&kvmap, smem + s * C::kStageBytes, &full[s], p.layer,
                             (block * p.Hkv + it.kv_head) * 16);
      }
    }
    return;
  }

  const int g = lane >> 2, t = lane & 3;
  // rows of this thread: (warp*ppw + g/group ...) mapped as row = warp*16 + g (+8)
  int pos_r[2], tok_r[2], head_r[2];
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    const int rr = g + 8 * r;
    const int pi = warp * ppw + rr / group;
    const bool ok = (rr < ppw * group) && (pi < it.npos);
    pos_r[r] = ok ? it.pos0 + pi : -1;
    tok_r[r] = it.row0 + pi;
    head_r[r] = it.kv_head * group + rr % group;
  }
  const int warp_max_pos = it.pos0 + min(it.npos, (warp + 1) * ppw) - 1;
  const bool warp_active = warp * ppw < it.npos;

  uint32_t qa[HD / 16][4];
  load_q_frags<HD>(pos_r[0] >= 0 ? p.q + size_t(tok_r[0]) * p.q_ld + size_t(head_r[0]) * HD : nullptr,
                   pos_r[1] >= 0 ? p.q + size_t(tok_r[1]) * p.q_ld + size_t(head_r[1]) * HD : nullptr, t, qa);
  float m[2] = {-INFINITY, -INFINITY}, l[2] = {0.f, 0.f};
  float o[HD / 8][4];
#pragma unroll
  for (int nt = 0; nt < HD / 8; ++nt) o[nt][0] = o[nt][1] = o[nt][2] = o[nt][3] = 0.f;

  for (int i = 0; i < nblk; ++i) {
    const int s = i % kAttnStages;
    const uint32_t ph = (i / kAttnStages) & 1;
    const int kbase = i * 16;
    if (warp_active && kbase <= warp_max_pos) {
      mbar_wait(&full[s], ph);
      const uint32_t kt = smem_u32(smem + s * C::kStageBytes);
      float sc[2][4];
      qk_block<HD>(qa, kt, lane, sc);
      uint32_t pa[4], pl[4];
      softmax_step<HD>(sc, m, l, o, p.scale_log2,
                       [&](int j, int e) { return kbase + 8 * j + 2 * t + (e & 1) <= pos_r[e >> 1]; }, pa, pl);
      pv_block<HD>(pa, pl, kt + C::kBlockBytes, lane, o);
    } else {
      mbar_wait(&full[s], ph);  // keep the ring phase consistent
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&empty[s]);
  }
  l[0] += __shfl_xor_sync(0xffffffffu, l[0], 1);
  l[0] += __shfl_xor_sync(0xffffffffu, l[0], 2);
  l[1] += __shfl_xor_sync(0xffffffffu, l[1], 1);
  l[1] += __shfl_xor_sync(0xffffffffu, l[1], 2);
#pragma unroll
  for (int r = 0; r < 2; ++r) {
    if (pos_r[r] < 0) continue;
    const float inv = 1.f / l[r];
    const size_t off = size_t(tok_r[r]) * p.out_ld + size_t(head_r[r]) * HD;
#pragma unroll
    for (int nt = 0; nt < HD / 8; ++nt) {
      const float v0 = o[nt][2 * r] * inv, v1 = o[nt][2 * r + 1] * inv;
      const int d = nt * 8 + 2 * t;
      if (p.out_f32) {
        *reinterpret_cast<float2*>(reinterpret_cast<float*>(p.out) + off + d) = make_float2(v0, v1);
      } else {
        *reinterpret_cast<uint32_t*>(reinterpret_cast<__nv_bfloat16*>(p.out) + off + d) = pack_bf16(v0, v1);
      }
    }
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

int prefill_positions_per_tile(int group) { return kConsumerWarps * (16 / group); }

template <int HD>
static cudaError_t decode_t(const AttnLaunch& a, const DecodeItem* items, int n_items, float* partials, int* counters,
                            cudaStream_t st) {
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(decode_attn_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         AttnCfg<HD>::kSmemBytes);
    if (e != cudaSuccess) return e;
    set = true;
  }
  AttnParams p = to_params(a);
  decode_attn_kernel<HD><<<n_items, kAttnThreads, AttnCfg<HD>::kSmemBytes, st>>>(*a.kv_tmap, p, items, partials,
                                                                                  counters);
  return cudaGetLastError();
}

cudaError_t launch_decode_attention(const AttnLaunch& a, const DecodeItem* items, int n_items, float* partials,
                                    int* counters, cudaStream_t st) {
  if (n_items == 0) return cudaSuccess;
  count_launch(1);
  if (a.hd == 128) return decode_t<128>(a, items, n_items, partials, counters, st);
  if (a.hd == 64) return decode_t<64>(a, items, n_items, partials, counters, st);
  return cudaErrorInvalidValue;
}

template <int HD>
static cudaError_t prefill_t(const AttnLaunch& a, const PrefillItem* items, int n_items, cudaStream_t st) {
  static bool set = false;
  if (!set) {
    cudaError_t e = cudaFuncSetAttribute(prefill_attn_kernel<HD>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         AttnCfg<HD>::kSmemBytes);
    if (e != cudaSuccess) return e;
    set = true;
  }
  prefill_attn_kernel<HD><<<n_items, kAttnThreads, AttnCfg<HD>::kSmemBytes, st>>>(*a.kv_tmap, to_params(a), items);
  return cudaGetLastError();
}

cudaError_t launch_prefill_attention(const AttnLaunch& a, const PrefillItem* items, int n_items, cudaStream_t st) {
  if (n_items == 0) return cudaSuccess;
  count_launch(1);
  if (a.hd == 128) return prefill_t<128>(a, items, n_items, st);
  if (a.hd == 64) return prefill_t<64>(a, items, n_items, st);
  return cudaErrorInvalidValue;
}

}  // namespace qos
