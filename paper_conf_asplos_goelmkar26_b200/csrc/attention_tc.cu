// attention_tc.cu — varlen causal prefill attention over the paged KV cache on tcgen05 tensor
// cores with TMEM accumulators ("prefill chunk attends to its own
// earlier KV blocks plus itself", BASELINE.json:north_star; chunked prefill).
//
// Work item = (chunk, 128-row Q tile, kv head).  The 128 rows pack (position, head-in-group)
// pairs, so one K/V tile serves the whole GQA group: 128/g positions x g heads.
//   warp 0      TMA producer: K and V tiles of 64 keys (4 paged blocks x 2 halves of 64 dims,
//               128-B swizzle; one 5-D box per half when the 4 block ids are consecutive)
//   warp 1      MMA issuer (one lane): S_j = Q K_j^T  (UMMA 128x64x16, A,B from smem) into
//               TMEM;  O += P_j V_j  (UMMA 128xHDx16, A = P from TMEM, B = V MN-major)
//   warps 2..5  softmax, one TMEM lane (= one row) per thread: masked fp32 online softmax with
//               exp2, P written back over S in TMEM in fp16 (V is cached in fp16, so P.V is
//               one kind::f16 MMA with f16 operands) and released in two 32-key halves; O is
//               rescaled in TMEM only when the running max grows by more than 2^8 (P <= 2^8
//               otherwise); epilogue O / l -> global.
// Two CTAs share an SM (96 KB smem, 256 TMEM columns each) so one CTA's softmax overlaps the
// other's MMAs.  Kernels: prefill_attn_persist_kernel (default: persistent CTAs over host-dealt
// LPT item lists), prefill_attn_tc_kernel (one item per CTA, option fa_persist=0),
// prefill_attn_pair_kernel (cta_group::2 CTA pairs, option fa_pair; measured slower) and
// prefill_attn_pp_kernel (two q tiles ping-ponged in one CTA, option fa_qtiles=2; slower).
#include <cfloat>
#include <climits>
#include <cstdlib>

#include "common.cuh"
#include "internal.h"

#ifndef QOS_FA_LAZY
#define QOS_FA_LAZY 8.f   // rescale O only when the running max grows by more than this (log2)
#endif

namespace qos {

// NQ = q tiles per CTA.  Both share every K/V tile.
//   NQ = 1: 2 CTAs per SM: Q + 2-stage K and V rings (96 KB at HD 128) and 256 TMEM columns
//           each (two 64-column S/P buffers + the O accumulator).
//   NQ = 2: 1 CTA per SM, 8 softmax warps (one group of 4 per q tile): Q0, Q1 + 4-stage K and
//           V rings (192 KB), 512 TMEM columns (S/P double buffer and O per q tile).  Each K/V
//           tile feeds 256 query rows, halving the L2 -> SM traffic per FLOP, and the deeper
//           ring covers the L2 latency (with NQ = 1 the MMA-only and QK-only variants run as
//           long as the full kernel: the 2-deep K/V feed, not the tensor core, bounds it).
// With two S buffers per q tile the MMA warp issues QK of tile j+1 before PV of tile j, so a
// softmax group never waits on its own PV.
template <int HD, int NQ>
struct FaCfg {
  static constexpr int kRows = 128;                  // Q-tile rows (UMMA M)
  static constexpr int kKeys = 64;                   // keys per K/V tile (4 paged blocks)
  static constexpr int kHalves = HD / 64;
  static constexpr int kQBytes = kRows * HD * 2;     // 32 KB at HD 128
  static constexpr int kTileBytes = kKeys * HD * 2;  // one K or V tile
  static constexpr int kStages = NQ == 1 ? 2 : 4;
  static constexpr int kSmem = NQ * kQBytes + 2 * kStages * kTileBytes + 1024 + 512;
  static constexpr int kThreads = 64 + NQ * 128;
  static constexpr int kMinBlocks = NQ == 1 ? 2 : 1;
  // TMEM columns: S/P buffer b of q tile g at g*128 + b*64, O of q tile g at NQ*128 + g*128
  static constexpr uint32_t kTmemCols = NQ * 256;
  static constexpr uint32_t col_s(int g, int b) { return uint32_t(g * 128 + b * 64); }
  static constexpr uint32_t col_o(int g) { return uint32_t(NQ * 128 + g * 128); }
};

QOS_DEV void tmem_st32x32b_x16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
QOS_DEV void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
QOS_DEV float ex2(float x) {  // MUFU.EX2 (flush-to-zero; arguments are <= 8 here)
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}

QOS_DEV float fmax3(float a, float b, float c) {  // FMNMX3
  float d;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(d) : "f"(a), "f"(b), "f"(c));
  return d;
}

// packed fp32 pair arithmetic (sm_100: FFMA2 / FADD2)
QOS_DEV float2 fma2(float2 a, float2 b, float2 c) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rc, rd;\n\t"
      "mov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\tmov.b64 rc, {%6, %7};\n\t"
      "fma.rn.f32x2 rd, ra, rb, rc;\n\tmov.b64 {%0, %1}, rd;\n\t}"
      : "=f"(d.x), "=f"(d.y)
      : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y), "f"(c.x), "f"(c.y));
  return d;
}
QOS_DEV float2 add2(float2 a, float2 b) {
  float2 d;
  asm("{\n\t.reg .b64 ra, rb, rd;\n\t"
      "mov.b64 ra, {%2, %3};\n\tmov.b64 rb, {%4, %5};\n\t"
      "add.rn.f32x2 rd, ra, rb;\n\tmov.b64 {%0, %1}, rd;\n\t}"
      : "=f"(d.x), "=f"(d.y)
      : "f"(a.x), "f"(a.y), "f"(b.x), "f"(b.y));
  return d;
}

// 2^x for a pair on the FMA pipe (relieves MUFU, which at 16 ex2/clk/SM is as slow as the
// tensor core on a 128x64 S tile): x = j + f with j = rint(x) (1.5*2^23 round trick), f in
// [-0.5, 0.5]; 2^f by a degree-3 minimax polynomial (max relative error 7.5e-5, below the
// fp16 rounding of P, 2^-11); 2^j is added into the exponent field.  x is clamped at -125 so
// the biased exponent of the result stays >= 1 (2^-125 rounds to 0 in fp16, like MUFU's
// flush-to-zero; masked scores arrive here as -inf).
QOS_DEV float2 ex2_poly2(float2 x) {
  x.x = fmaxf(x.x, -125.f);
  x.y = fmaxf(x.y, -125.f);
  const float2 magic = make_float2(12582912.f, 12582912.f), nmagic = make_float2(-12582912.f, -12582912.f);
  const float2 t = add2(x, magic);
  const float2 f = fma2(add2(t, nmagic), make_float2(-1.f, -1.f), x);  // x - rint(x), exact
  float2 p = fma2(make_float2(0.05517150089144707f, 0.05517150089144707f), f,
                  make_float2(0.24261096119880676f, 0.24261096119880676f));
  p = fma2(p, f, make_float2(0.6932609677314758f, 0.6932609677314758f));
  p = fma2(p, f, make_float2(0.9999280571937561f, 0.9999280571937561f));
  return make_float2(__uint_as_float(__float_as_uint(p.x) + (__float_as_uint(t.x) << 23)),
                     __uint_as_float(__float_as_uint(p.y) + (__float_as_uint(t.y) << 23)));
}

// D[tmem] (+)= A[tmem] · B[smem desc]   (kind::f16, A = 16-bit pairs packed in 32-bit columns)
QOS_DEV void umma_bf16_ts(uint32_t d_tmem, uint32_t a_tmem, uint64_t b_desc, uint32_t idesc, uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n\t}" ::"r"(d_tmem),
      "r"(a_tmem), "l"(b_desc), "r"(idesc), "r"(accumulate)
      : "memory");
}

// MN-major 128-B swizzled operand (V: key rows of 64 contiguous dims): atoms of 8 K-rows x
// 64 MN elements (1 KB); K atoms stacked at SBO = 1024 B, MN atoms (the second 64 dims) at
// LBO = one 64-dim half of the tile.
QOS_DEV uint64_t umma_desc_sw128_mn(uint32_t smem_addr, uint32_t lbo_bytes) {
  uint64_t d = 0;
  d |= (uint64_t)((smem_addr & 0x3FFFF) >> 4);
  d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}

struct FaParams {
  const __nv_bfloat16* q;
  int q_ld;
  void* out;
  int out_ld;
  int out_f32;
  int layer, H, Hkv;
  const int32_t* tables;
  int table_w;
  float scale_log2;
  int kv_first = 0;  // persistent kernel: issue an item's first K/V tile before its Q (option fa_kvfirst)
  int tma5 = 0;      // persistent kernel: a tile's 4 blocks in one 5-D box when their ids are consecutive
  int psplit = 0;    // persistent kernel: release P to the P.V MMAs in two halves of 32 keys
};

// Work item = NQ consecutive entries of `items`: q tiles of one (chunk, kv head) that share
// grp_last (the host pads a short group with a duplicate that stores nothing).
template <int HD, int POLY, int NQ>
__global__ void __launch_bounds__(FaCfg<HD, NQ>::kThreads, FaCfg<HD, NQ>::kMinBlocks)
    prefill_attn_tc_kernel(const __grid_constant__ CUtensorMap kvmap, const FaParams p,
                           const PrefillItem* __restrict__ items) {
  using C = FaCfg<HD, NQ>;
  constexpr int S = C::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                          // NQ x kQBytes
  uint8_t* sK = smem + NQ * C::kQBytes;
  uint8_t* sV = sK + S * C::kTileBytes;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sV + S * C::kTileBytes);
  uint64_t* k_full = bar;
  uint64_t* k_empty = k_full + S;
  uint64_t* v_full = k_empty + S;
  uint64_t* v_empty = v_full + S;
  uint64_t* s_full = v_empty + S;        // [NQ][2]
  uint64_t* p_full = s_full + 2 * NQ;    // [NQ][2]
  uint64_t* o_full = p_full + 2 * NQ;    // [NQ]
  uint64_t* o_final = o_full + NQ;       // [NQ] completes once, when the last PV has landed
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(o_final + NQ);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const PrefillItem it0 = items[blockIdx.x * NQ];
  const int group = p.H / p.Hkv;
  const int ppt = C::kRows / group;  // positions per tile
  const int last_pos = it0.grp_last;  // over the NQ q tiles
  const int ntiles = last_pos / C::kKeys + 1;
  const int last_blk = last_pos >> 4;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_empty[i], 1);
      mbar_init(&v_full[i], 1);
      mbar_init(&v_empty[i], 1);
    }
    for (int g = 0; g < NQ; ++g) {
      for (int b = 0; b < 2; ++b) {
        mbar_init(&s_full[g * 2 + b], 1);
        mbar_init(&p_full[g * 2 + b], 128);
      }
      mbar_init(&o_full[g], 1);
      mbar_init(&o_final[g], 1);
    }
    fence_mbar_init();
  }
  if (warp == 1) tmem_alloc<C::kTmemCols>(tmem_slot);
  griddep_wait();  // q and the appended K/V come from the previous kernel
  griddep_launch_dependents();

  // ---- Q tiles -> smem (softmax group g = (warp - 2) / 4; one row per thread), K-major 128-B swizzle
  const int qg = warp >= 2 ? (warp - 2) >> 2 : 0;
  const PrefillItem it = items[blockIdx.x * NQ + qg];
  int row = 0, pos_r = -1;
  size_t tok_off = 0;
  if (warp >= 2) {
    row = (warp & 3) * 32 + lane;  // the TMEM lane quarter this warp may access
    const int pi = row / group, hh = row % group;
    const bool ok = row < ppt * group && pi < it.npos;
    pos_r = ok ? it.pos0 + pi : -1;
    tok_off = size_t(it.row0 + pi) * p.out_ld + size_t(it.kv_head * group + hh) * HD;
    const __nv_bfloat16* src = p.q + size_t(it.row0 + pi) * p.q_ld + size_t(it.kv_head * group + hh) * HD;
    uint8_t* q_dst = sQ + qg * C::kQBytes;
    uint4 v[HD / 8];
#pragma unroll
    for (int ch = 0; ch < HD / 8; ++ch) v[ch] = ok ? *reinterpret_cast<const uint4*>(src + ch * 8) : make_uint4(0, 0, 0, 0);
#pragma unroll
    for (int ch = 0; ch < HD / 8; ++ch) {
      const int hf = ch >> 3, c = ch & 7;
      *reinterpret_cast<uint4*>(q_dst + hf * (C::kRows * 128) + row * 128 + ((c ^ (row & 7)) << 4)) = v[ch];
    }
    fence_proxy_async_smem();
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer
    if (elect_one()) {
      tma_prefetch_desc(&kvmap);
      const int32_t* trow = p.tables + size_t(it0.table) * p.table_w;
      auto load_tile = [&](uint8_t* dst, uint64_t* full, int j, int plane) {
        for (int b = 0; b < C::kKeys / 16; ++b) {
          const int blk = min(j * (C::kKeys / 16) + b, last_blk);  // past the causal end: a valid block (P = 0)
          const int r = (__ldg(trow + blk) * p.Hkv + it0.kv_head) * 16;
#pragma unroll
          for (int hf = 0; hf < C::kHalves; ++hf)
            tma_load_3d(dst + hf * (C::kKeys * 128) + b * 2048, &kvmap, full, hf * 64, r, p.layer * 2 + plane);
        }
      };
      for (int j = 0; j < ntiles; ++j) {
        const int s = j % S;
        const uint32_t ph = (j / S) & 1;
        mbar_wait(&k_empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&k_full[s], C::kTileBytes);
        load_tile(sK + s * C::kTileBytes, &k_full[s], j, 0);
        mbar_wait(&v_empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&v_full[s], C::kTileBytes);
        load_tile(sV + s * C::kTileBytes, &v_full[s], j, 1);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer
    if (elect_one()) {
      constexpr uint32_t idesc_qk = umma_idesc_bf16(128, C::kKeys);
      // P.V in fp16 (A = P in TMEM, B = V cached in fp16, MN-major): formats a/b = f16 (0)
      constexpr uint32_t idesc_pv = (1u << 4) | (1u << 16) | ((uint32_t(HD) >> 3) << 17) | ((128u >> 4) << 24);
      auto issue_pv = [&](int t) {
        const int s = t % S;
        mbar_wait(&v_full[s], (t / S) & 1);
        const uint32_t v_base = smem_u32(sV + s * C::kTileBytes);
        for (int g = 0; g < NQ; ++g) {
          mbar_wait(&p_full[g * 2 + (t & 1)], (t >> 1) & 1);
          tc_fence_after();
          const uint32_t p_tmem = tmem + C::col_s(g, t & 1);
#pragma unroll
          for (int kk = 0; kk < C::kKeys / 16; ++kk) {
            const uint64_t vd = umma_desc_sw128_mn(v_base + kk * 2048, C::kKeys * 128);
            const uint32_t pc = p_tmem + (kk >> 1) * 32 + (kk & 1) * 8;
            if (POLY != -2) umma_bf16_ts(tmem + C::col_o(g), pc, vd, idesc_pv, (t | kk) != 0);
          }
          umma_commit(&o_full[g]);
        }
        umma_commit(&v_empty[s]);
      };
      for (int j = 0; j < ntiles; ++j) {
        // S_g(j) = Q_g K_j^T into S buffer j%2 of q tile g; its previous tenant P_g(j-2) was
        // consumed by PV(j-2), issued before this point (tcgen05 ops execute in issue order)
        const int s = j % S;
        mbar_wait(&k_full[s], (j / S) & 1);
        tc_fence_after();
        const uint32_t k_base = smem_u32(sK + s * C::kTileBytes);
        for (int g = 0; g < NQ; ++g) {
          const uint32_t q_base = smem_u32(sQ + g * C::kQBytes);
          const uint32_t s_tmem = tmem + C::col_s(g, j & 1);
#pragma unroll
          for (int ks = 0; ks < HD / 16; ++ks) {
            const uint32_t qoff = (ks >> 2) * (C::kRows * 128) + (ks & 3) * 32;
            const uint32_t koff = (ks >> 2) * (C::kKeys * 128) + (ks & 3) * 32;
            if (POLY != -3) umma_bf16(s_tmem, umma_desc_sw128(q_base + qoff), umma_desc_sw128(k_base + koff), idesc_qk, ks != 0);
          }
          umma_commit(&s_full[g * 2 + (j & 1)]);
        }
        umma_commit(&k_empty[s]);
        if (j >= 1) issue_pv(j - 1);   // O += P(j-1) V(j-1) while the softmax works on S(j)
      }
      issue_pv(ntiles - 1);
      for (int g = 0; g < NQ; ++g) umma_commit(&o_final[g]);
    }
  } else {
    // ------------------------------------------------------------------ softmax (group qg)
    const uint32_t lane_base = tmem + (uint32_t((warp & 3) * 32) << 16);
    const uint32_t o_addr = lane_base + C::col_o(qg);
    uint64_t* my_s_full = s_full + qg * 2;
    uint64_t* my_p_full = p_full + qg * 2;
    const int warp_min_pos = __shfl_sync(0xffffffffu, pos_r < 0 ? INT_MAX : pos_r, 0);  // row 0 of the warp
    float m_used = -INFINITY, l = 0.f;
    for (int j = 0; j < ntiles; ++j) {
      const int sb = j & 1;
      mbar_wait(&my_s_full[sb], (j >> 1) & 1);
      tc_fence_after();
      if (POLY < 0) {  // measurement-only variants: MMA + TMA pipeline without the softmax
        tc_fence_before();
        mbar_arrive(&my_p_full[sb]);
        continue;
      }
      const uint32_t s_addr = lane_base + C::col_s(qg, sb);
      const int key0 = j * C::kKeys;
      // masking only where a key of this tile can exceed a row's position
      const bool masked = __any_sync(0xffffffffu, key0 + C::kKeys - 1 > (pos_r < 0 ? -1 : pos_r)) ||
                          warp_min_pos == INT_MAX;
      // the whole S row (64 fp32) in one batch of TMEM loads and a single wait
      uint32_t r[C::kKeys];
#pragma unroll
      for (int c = 0; c < C::kKeys / 16; ++c)
        tmem_ld32x32b_x16(s_addr + c * 16, *reinterpret_cast<uint32_t(*)[16]>(&r[c * 16]));
      tmem_ld_wait();
      // causal mask (only the tiles that reach past a row's position): masked scores become
      // -inf, so the max and exp passes below are the same for every tile (2^-inf = 0).  Kept a
      // real branch so unmasked tiles do not execute predicated selects.
      if (masked) {
        const int lim = (pos_r < 0 ? -1 : pos_r) - key0;  // key i is visible iff i <= lim
#pragma unroll
        for (int i = 0; i < C::kKeys; ++i)
          if (i > lim) r[i] = 0xff800000u;  // -inf
      }
      // row max of the raw scores (scaled afterwards; the scale is positive)
      // (four independent 3-input max chains: a short dependency chain)
      float mq[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
      for (int i = 0; i < C::kKeys; i += 2)
        mq[(i >> 1) & 3] = fmax3(mq[(i >> 1) & 3], __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
      float mx = fmax3(mq[0], mq[1], fmaxf(mq[2], mq[3]));
      mx *= p.scale_log2;
      // lazy rescale: keep the previous max unless the new one exceeds it by > 8 (P <= 2^8)
      const bool rescale = mx > m_used + QOS_FA_LAZY;
      const float m_new = rescale ? mx : m_used;
      const float alpha = (rescale && m_used != -INFINITY) ? ex2(m_used - m_new) : 1.f;
      const float mb = (m_new == -INFINITY) ? 0.f : m_new;
      // pass 2: P = 2^(s*scale - m) and the row sum; P written in fp16 (2^-11 relative, so the
      // fp32 P.V meets the 2e-3 attention bar; bf16 P alone measured 2.3-3.6e-3) over the S
      // columns each chunk has just read: [32c, 32c+16) hold the fp16 pairs of keys 32c..32c+31.
      float2 sum2[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
      const float2 scale2 = make_float2(p.scale_log2, p.scale_log2), nmb2 = make_float2(-mb, -mb);
#pragma unroll
      for (int c = 0; c < C::kKeys / 32; ++c) {
        uint32_t hi[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          // paired fp32 ops (FFMA2 / FADD2) halve the softmax's FMA-pipe instructions
          const float2 x = fma2(make_float2(__uint_as_float(r[c * 32 + 2 * i]), __uint_as_float(r[c * 32 + 2 * i + 1])),
                                scale2, nmb2);
          // every POLY-th pair on the FMA pipe (POLY = 0: none), the rest on MUFU
          float2 pp = (POLY > 0 && i % (POLY > 0 ? POLY : 1) == (POLY > 0 ? POLY : 1) - 1) ? ex2_poly2(x) : make_float2(ex2(x.x), ex2(x.y));
          hi[i] = pack_f16(pp.x, pp.y);
          sum2[i & 3] = add2(sum2[i & 3], pp);
        }
        tmem_st32x32b_x16(s_addr + c * 32, hi);
      }
      const float2 s01 = add2(sum2[0], sum2[1]), s23 = add2(sum2[2], sum2[3]);
      const float sum = (s01.x + s23.x) + (s01.y + s23.y);
      tmem_st_wait();
      l = l * alpha + sum;
      if (j >= 1 && __any_sync(0xffffffffu, alpha != 1.f)) {
        // rescale O (tiles < j) before PV(j) accumulates into it.  Wait for PV(j-1) only here:
        // PV(j-2) was issued before QK(j), whose completion was awaited above, so o_full is at
        // phase j-1 or j and this parity wait cannot alias.
        mbar_wait(&o_full[qg], (j - 1) & 1);
        tc_fence_after();
#pragma unroll 1
        for (int c = 0; c < HD / 16; ++c) {
          uint32_t r2[16];
          tmem_ld32x32b_x16(o_addr + c * 16, r2);
          tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 16; ++i) r2[i] = __float_as_uint(__uint_as_float(r2[i]) * alpha);
          tmem_st32x32b_x16(o_addr + c * 16, r2);
        }
        tmem_st_wait();
      }
      m_used = m_new;
      tc_fence_before();
      mbar_arrive(&my_p_full[sb]);
    }
    // epilogue: O / l
    // o_full may be anywhere in phases n-2..n here (its waits are skipped when no rescale is
    // needed), so a parity wait on it could alias; the dedicated o_final barrier completes once
    mbar_wait(&o_final[qg], 0);
    tc_fence_after();
    const float inv = (l > 0.f) ? 1.f / l : 0.f;
#pragma unroll 1
    for (int c = 0; c < HD / 32; ++c) {
      uint32_t r2[32];
      tmem_ld32x32b_x16(o_addr + c * 32, *reinterpret_cast<uint32_t(*)[16]>(&r2[0]));
      tmem_ld32x32b_x16(o_addr + c * 32 + 16, *reinterpret_cast<uint32_t(*)[16]>(&r2[16]));
      tmem_ld_wait();
      if (pos_r >= 0 && !it.pad) {
        if (p.out_f32) {
          float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(p.out) + tok_off + c * 32);
#pragma unroll
          for (int i = 0; i < 8; ++i)
            dst[i] = make_float4(__uint_as_float(r2[4 * i]) * inv, __uint_as_float(r2[4 * i + 1]) * inv,
                                 __uint_as_float(r2[4 * i + 2]) * inv, __uint_as_float(r2[4 * i + 3]) * inv);
        } else {
          uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.out) + tok_off + c * 32);
#pragma unroll
          for (int i = 0; i < 4; ++i)
            dst[i] = make_uint4(pack_bf16(__uint_as_float(r2[8 * i]) * inv, __uint_as_float(r2[8 * i + 1]) * inv),
                                pack_bf16(__uint_as_float(r2[8 * i + 2]) * inv, __uint_as_float(r2[8 * i + 3]) * inv),
                                pack_bf16(__uint_as_float(r2[8 * i + 4]) * inv, __uint_as_float(r2[8 * i + 5]) * inv),
                                pack_bf16(__uint_as_float(r2[8 * i + 6]) * inv, __uint_as_float(r2[8 * i + 7]) * inv));
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<C::kTmemCols>(tmem);
  }
}


// ---------------------------------------------------------------- persistent variant (fa_persist=1)
// The single-q-tile kernel above as a persistent CTA (2 per SM): CTA c runs the work items
// items[cta_off[c] .. cta_off[c+1]) back to back (the host assigns the LPT-sorted items to CTAs
// greedily by key tiles, like the hardware block scheduler would).  Barrier phases and the
// K/V ring run on per-CTA cumulative tile counts, TMEM and barriers are set up once, and the
// next item's Q is staged while the current item's epilogue drains O, so the MMA warp starts
// the next item's QK(0) under that epilogue and the producer streams its K/V tiles under the
// current item's tail.  With short causal chunks (2048 tokens from position 0: 16 key tiles
// per item on average) the per-CTA prologue/epilogue was a third of the launch.
template <int HD, int POLY>
__global__ void __launch_bounds__(FaCfg<HD, 1>::kThreads, 2)
    prefill_attn_persist_kernel(const __grid_constant__ CUtensorMap kvmap, const __grid_constant__ CUtensorMap qmap,
                                const __grid_constant__ CUtensorMap kvmap5, const FaParams p,
                                const PrefillItem* __restrict__ items, const int32_t* __restrict__ cta_off) {
  using C = FaCfg<HD, 1>;
  constexpr int S = C::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = smem + C::kQBytes;
  uint8_t* sV = sK + S * C::kTileBytes;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sV + S * C::kTileBytes);
  uint64_t* k_full = bar;
  uint64_t* k_empty = k_full + S;
  uint64_t* v_full = k_empty + S;
  uint64_t* v_empty = v_full + S;
  uint64_t* s_full = v_empty + S;   // [2]
  uint64_t* p_full = s_full + 2;    // [2 buffers][2 key halves]
  uint64_t* o_full = p_full + 4;    // completes once per P.V
  uint64_t* o_final = o_full + 1;   // completes once per item
  uint64_t* q_full = o_final + 1;   // completes once per item (Q tile landed, TMA)
  uint64_t* q_empty = q_full + 1;   // completes once per item (its last QK done: sQ free)
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(q_empty + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int i_begin = cta_off[blockIdx.x], i_end = cta_off[blockIdx.x + 1];
  const int group = p.H / p.Hkv;
  const int ppt = C::kRows / group;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_empty[i], 1);
      mbar_init(&v_full[i], 1);
      mbar_init(&v_empty[i], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&s_full[b], 1);
      mbar_init(&p_full[2 * b], 128);
      mbar_init(&p_full[2 * b + 1], 128);
    }
    mbar_init(o_full, 1);
    mbar_init(o_final, 1);
    mbar_init(q_full, 1);
    mbar_init(q_empty, 1);
    fence_mbar_init();
  }
  if (warp == 1) tmem_alloc<C::kTmemCols>(tmem_slot);
  griddep_wait();  // q and the appended K/V come from the previous kernel
  griddep_launch_dependents();
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer
    if (elect_one()) {
      tma_prefetch_desc(&kvmap);
      tma_prefetch_desc(&qmap);
      uint32_t jg = 0;
      for (int ii = i_begin, n = 0; ii < i_end; ++ii, ++n) {
        const PrefillItem it = items[ii];
        const int nt = it.grp_last / C::kKeys + 1, last_blk = it.grp_last >> 4;
        const int32_t* trow = p.tables + size_t(it.table) * p.table_w;
        // tile j of the item into ring slot jg % S; the tile's 4 block-table entries are read
        // once (independent loads) for its K and V halves; past the causal end a valid block (P = 0)
        auto load_kv = [&](int j) {
          const int s = int(jg % S);
          const uint32_t ph = (jg / S) & 1;
          constexpr int NB = C::kKeys / 16;
          int id[NB];
#pragma unroll
          for (int b = 0; b < NB; ++b) id[b] = __ldg(trow + min(j * NB + b, last_blk));
          // the tile's blocks are one run of consecutive ids (the allocator hands out the lowest
          // free ids, so a fresh request's blocks usually are): one 5-D box per 64-dim half
          bool run = p.tma5 != 0 && j * NB + NB - 1 <= last_blk;
#pragma unroll
          for (int b = 1; b < NB; ++b) run = run && id[b] == id[0] + b;
          auto load = [&](uint8_t* dst, uint64_t* full, int plane) {
            if (run) {
#pragma unroll
              for (int hf = 0; hf < C::kHalves; ++hf)
                tma_load_5d(dst + hf * (C::kKeys * 128), &kvmap5, full, hf * 64, 0, it.kv_head, id[0], p.layer * 2 + plane);
            } else {
#pragma unroll
              for (int b = 0; b < NB; ++b)
#pragma unroll
                for (int hf = 0; hf < C::kHalves; ++hf)
                  tma_load_3d(dst + hf * (C::kKeys * 128) + b * 2048, &kvmap, full, hf * 64,
                              (id[b] * p.Hkv + it.kv_head) * 16, p.layer * 2 + plane);
            }
          };
          mbar_wait(&k_empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&k_full[s], C::kTileBytes);
          load(sK + s * C::kTileBytes, &k_full[s], 0);
          mbar_wait(&v_empty[s], ph ^ 1);
          mbar_arrive_expect_tx(&v_full[s], C::kTileBytes);
          load(sV + s * C::kTileBytes, &v_full[s], 1);
          ++jg;
        };
        // with kv_first the item's first K/V tile goes out before its Q, which has to wait for
        // the previous item's last QK to release sQ
        if (p.kv_first) load_kv(0);
        // Q tile of the item: rows (position, head-in-group) = a {64 dims, group heads, ppt rows}
        // box per 64-dim half; issued as soon as the previous item's last QK has read sQ
        // (group * ppt rows: 125 when the GQA group is 5 — the remaining rows of sQ are never
        //  valid rows (pos_r < 0: fully masked, nothing stored) and the box fills only the others)
        if (n > 0) mbar_wait(q_empty, uint32_t(n - 1) & 1);
        mbar_arrive_expect_tx(q_full, uint32_t(C::kHalves) * 128u * uint32_t(group * ppt));
#pragma unroll
        for (int hf = 0; hf < C::kHalves; ++hf)
          tma_load_3d(sQ + hf * (C::kRows * 128), &qmap, q_full, hf * 64, it.kv_head * group, it.row0);
        for (int j = p.kv_first ? 1 : 0; j < nt; ++j) load_kv(j);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer
    if (elect_one()) {
      constexpr uint32_t idesc_qk = umma_idesc_bf16(128, C::kKeys);
      constexpr uint32_t idesc_pv = (1u << 4) | (1u << 16) | ((uint32_t(HD) >> 3) << 17) | ((128u >> 4) << 24);
      // O += P(tg) V(tg); `first`: the item's first tile (overwrites O)
      auto issue_pv = [&](uint32_t tg, bool first) {
        const int s = int(tg % S);
        mbar_wait(&v_full[s], (tg / S) & 1);
        const uint32_t v_base = smem_u32(sV + s * C::kTileBytes);
        const uint32_t p_tmem = tmem + C::col_s(0, int(tg & 1));
        // P arrives in two halves of 32 keys (fa_psplit: the first half's MMAs run while the
        // softmax computes the second half; without it only the second barrier is used)
        auto pv_mmas = [&](int kk0, int kk1) {
          for (int kk = kk0; kk < kk1; ++kk) {
            const uint64_t vd = umma_desc_sw128_mn(v_base + kk * 2048, C::kKeys * 128);
            const uint32_t pc = p_tmem + (kk >> 1) * 32 + (kk & 1) * 8;
            umma_bf16_ts(tmem + C::col_o(0), pc, vd, idesc_pv, (!first || kk != 0) ? 1u : 0u);
          }
        };
        constexpr int KK = C::kKeys / 16;
        if (p.psplit) {
          mbar_wait(&p_full[(tg & 1) * 2], (tg >> 1) & 1);
          tc_fence_after();
          pv_mmas(0, KK / 2);
          mbar_wait(&p_full[(tg & 1) * 2 + 1], (tg >> 1) & 1);
          tc_fence_after();
          pv_mmas(KK / 2, KK);
        } else {
          mbar_wait(&p_full[(tg & 1) * 2 + 1], (tg >> 1) & 1);
          tc_fence_after();
          pv_mmas(0, KK);
        }
        umma_commit(o_full);
        umma_commit(&v_empty[s]);
      };
      uint32_t jg = 0;
      for (int ii = i_begin, n = 0; ii < i_end; ++ii, ++n) {
        const int nt = items[ii].grp_last / C::kKeys + 1;
        mbar_wait(q_full, uint32_t(n) & 1);  // this item's Q is in smem
        tc_fence_after();
        const uint32_t q_base = smem_u32(sQ);
        for (int j = 0; j < nt; ++j) {
          const uint32_t tg = jg + uint32_t(j);
          const int s = int(tg % S);
          mbar_wait(&k_full[s], (tg / S) & 1);
          tc_fence_after();
          const uint32_t k_base = smem_u32(sK + s * C::kTileBytes);
          const uint32_t s_tmem = tmem + C::col_s(0, int(tg & 1));
#pragma unroll
          for (int ks = 0; ks < HD / 16; ++ks) {
            const uint32_t qoff = (ks >> 2) * (C::kRows * 128) + (ks & 3) * 32;
            const uint32_t koff = (ks >> 2) * (C::kKeys * 128) + (ks & 3) * 32;
            umma_bf16(s_tmem, umma_desc_sw128(q_base + qoff), umma_desc_sw128(k_base + koff), idesc_qk, ks != 0);
          }
          umma_commit(&s_full[tg & 1]);
          umma_commit(&k_empty[s]);
          if (j >= 1) issue_pv(tg - 1, j == 1);   // O += P(j-1) V(j-1) while the softmax works on S(j)
        }
        umma_commit(q_empty);  // every QK of this item has been issued: sQ is free once they complete
        issue_pv(jg + uint32_t(nt) - 1, nt == 1);
        umma_commit(o_final);
        jg += uint32_t(nt);
      }
    }
  } else {
    // ------------------------------------------------------------------ softmax + Q staging + epilogue
    const int row = (warp & 3) * 32 + lane;  // the TMEM lane quarter this warp may access
    const uint32_t lane_base = tmem + (uint32_t((warp & 3) * 32) << 16);
    const uint32_t o_addr = lane_base + C::col_o(0);
    const int pi = row / group, hh = row % group;
    uint32_t jg = 0;
    for (int ii = i_begin, n = 0; ii < i_end; ++ii, ++n) {
      const PrefillItem it = items[ii];
      const int nt = it.grp_last / C::kKeys + 1;
      const bool ok = row < ppt * group && pi < it.npos;
      const int pos_r = ok ? it.pos0 + pi : -1;
      const size_t tok_off = size_t(it.row0 + pi) * p.out_ld + size_t(it.kv_head * group + hh) * HD;
      const int warp_min_pos = __shfl_sync(0xffffffffu, pos_r < 0 ? INT_MAX : pos_r, 0);  // row 0 of the warp
      float m_used = -INFINITY, l = 0.f;
      for (int j = 0; j < nt; ++j) {
        const uint32_t tg = jg + uint32_t(j);
        const int sb = int(tg & 1);
        mbar_wait(&s_full[sb], (tg >> 1) & 1);
        tc_fence_after();
        const uint32_t s_addr = lane_base + C::col_s(0, sb);
        const int key0 = j * C::kKeys;
        const bool masked = __any_sync(0xffffffffu, key0 + C::kKeys - 1 > (pos_r < 0 ? -1 : pos_r)) ||
                            warp_min_pos == INT_MAX;
        uint32_t r[C::kKeys];
#pragma unroll
        for (int c = 0; c < C::kKeys / 16; ++c)
          tmem_ld32x32b_x16(s_addr + c * 16, *reinterpret_cast<uint32_t(*)[16]>(&r[c * 16]));
        tmem_ld_wait();
        if (masked) {
          const int lim = (pos_r < 0 ? -1 : pos_r) - key0;
#pragma unroll
          for (int i = 0; i < C::kKeys; ++i)
            if (i > lim) r[i] = 0xff800000u;  // -inf
        }
        float mq[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
        for (int i = 0; i < C::kKeys; i += 2)
          mq[(i >> 1) & 3] = fmax3(mq[(i >> 1) & 3], __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
        float mx = fmax3(mq[0], mq[1], fmaxf(mq[2], mq[3]));
        mx *= p.scale_log2;
        const bool rescale = mx > m_used + QOS_FA_LAZY;
        const float m_new = rescale ? mx : m_used;
        const float alpha = (rescale && m_used != -INFINITY) ? ex2(m_used - m_new) : 1.f;
        const float mb = (m_new == -INFINITY) ? 0.f : m_new;
        // rescale O (tiles < j) before PV(j) accumulates into it; PV(tg-2) completed before
        // QK(tg) (awaited above), so o_full has completed tg-1 or tg times and this parity wait
        // cannot alias.  With fa_psplit it happens before the first half of P is released.
        auto rescale_o = [&]() {
          if (j >= 1 && __any_sync(0xffffffffu, alpha != 1.f)) {
            mbar_wait(o_full, (tg - 1) & 1);
            tc_fence_after();
#pragma unroll 1
            for (int c = 0; c < HD / 16; ++c) {
              uint32_t r2[16];
              tmem_ld32x32b_x16(o_addr + c * 16, r2);
              tmem_ld_wait();
#pragma unroll
              for (int i = 0; i < 16; ++i) r2[i] = __float_as_uint(__uint_as_float(r2[i]) * alpha);
              tmem_st32x32b_x16(o_addr + c * 16, r2);
            }
            tmem_st_wait();
          }
        };
        if (p.psplit) rescale_o();
        float2 sum2[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        const float2 scale2 = make_float2(p.scale_log2, p.scale_log2), nmb2 = make_float2(-mb, -mb);
#pragma unroll
        for (int c = 0; c < C::kKeys / 32; ++c) {
          uint32_t hi[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const float2 x = fma2(make_float2(__uint_as_float(r[c * 32 + 2 * i]), __uint_as_float(r[c * 32 + 2 * i + 1])),
                                  scale2, nmb2);
            float2 pp = (POLY > 0 && i % (POLY > 0 ? POLY : 1) == (POLY > 0 ? POLY : 1) - 1) ? ex2_poly2(x) : make_float2(ex2(x.x), ex2(x.y));
            hi[i] = pack_f16(pp.x, pp.y);
            sum2[i & 3] = add2(sum2[i & 3], pp);
          }
          tmem_st32x32b_x16(s_addr + c * 32, hi);
          if (p.psplit) {
            tmem_st_wait();
            tc_fence_before();
            mbar_arrive(&p_full[sb * 2 + c]);
          }
        }
        const float2 s01 = add2(sum2[0], sum2[1]), s23 = add2(sum2[2], sum2[3]);
        const float sum = (s01.x + s23.x) + (s01.y + s23.y);
        l = l * alpha + sum;
        if (!p.psplit) {
          tmem_st_wait();
          rescale_o();
          tc_fence_before();
          mbar_arrive(&p_full[sb * 2 + 1]);
        }
        m_used = m_new;
      }
      mbar_wait(o_final, uint32_t(n) & 1);
      tc_fence_after();
      const float inv = (l > 0.f) ? 1.f / l : 0.f;
#pragma unroll 1
      for (int c = 0; c < HD / 32; ++c) {
        uint32_t r2[32];
        tmem_ld32x32b_x16(o_addr + c * 32, *reinterpret_cast<uint32_t(*)[16]>(&r2[0]));
        tmem_ld32x32b_x16(o_addr + c * 32 + 16, *reinterpret_cast<uint32_t(*)[16]>(&r2[16]));
        tmem_ld_wait();
        if (pos_r >= 0 && !it.pad) {
          if (p.out_f32) {
            float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(p.out) + tok_off + c * 32);
#pragma unroll
            for (int i = 0; i < 8; ++i)
              dst[i] = make_float4(__uint_as_float(r2[4 * i]) * inv, __uint_as_float(r2[4 * i + 1]) * inv,
                                   __uint_as_float(r2[4 * i + 2]) * inv, __uint_as_float(r2[4 * i + 3]) * inv);
          } else {
            uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.out) + tok_off + c * 32);
#pragma unroll
            for (int i = 0; i < 4; ++i)
              dst[i] = make_uint4(pack_bf16(__uint_as_float(r2[8 * i]) * inv, __uint_as_float(r2[8 * i + 1]) * inv),
                                  pack_bf16(__uint_as_float(r2[8 * i + 2]) * inv, __uint_as_float(r2[8 * i + 3]) * inv),
                                  pack_bf16(__uint_as_float(r2[8 * i + 4]) * inv, __uint_as_float(r2[8 * i + 5]) * inv),
                                  pack_bf16(__uint_as_float(r2[8 * i + 6]) * inv, __uint_as_float(r2[8 * i + 7]) * inv));
          }
        }
      }
      jg += uint32_t(nt);
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<C::kTmemCols>(tmem);
  }
}

// ---------------------------------------------------------------- CTA-pair variant (fa_pair=1)
// The persistent kernel above on a thread-block cluster of 2 CTAs (2 SMs of one TPC) issuing
// tcgen05.mma.cta_group::2: one work item = two consecutive 128-row q tiles of one (chunk, kv
// head), CTA r holding q tile r in its smem and its 128 rows of S / P / O in its own TMEM.
//   S = Q K^T  (UMMA M = 256, N = 64 keys): B is split by N, so CTA r stages only keys
//              [32r, 32r + 32) of each 64-key tile;
//   O += P V   (UMMA M = 256, N = HD = 128, A = P from each CTA's TMEM): B = V is split by N,
//              so CTA r stages only dims [64r, 64r + 64) of the tile's 64 keys.
// Each K/V tile therefore costs every SM 16 KB of L2 -> SM traffic for 128 rows instead of
// 32 KB: the single-CTA kernel moves 128 FLOP per L2 byte (4.2 MFLOP of QK + PV per 32 KB),
// which at ~42 B/cycle/SM of L2 throughput caps it near 66% of the tensor peak — the measured
// ceiling of its MMA + TMA pipeline (profiles/prefill_attn_caps_ncu_r2a.jsonl).  (TMA
// multicast does not help at cluster size 2: the L2 de-duplicates only within ~4 requests.)
// Both CTAs' TMA loads complete on the leader's full barriers; the leader's commits arrive
// on both CTAs' barriers (multicast); the softmax warps of both CTAs release a P buffer on the
// leader's barrier (one remote arrive per warp).  2 pairs share an SM pair (96 KB smem and 256
// TMEM columns per CTA), so one pair's softmax overlaps the other's MMAs, as in the
// single-CTA kernel.  HD = 128 only (a 64-dim half of V is exactly one 128-B swizzle atom).
struct PairCfg {
  static constexpr int HD = 128;
  static constexpr int kRows = 128;                  // rows per CTA (UMMA M = 256 over the pair)
  static constexpr int kKeys = 64;                   // keys per K/V tile of the pair
  static constexpr int kQBytes = kRows * HD * 2;     // 32 KB
  static constexpr int kKBytes = (kKeys / 2) * HD * 2;  // this CTA's 32 keys x 128 dims: 8 KB
  static constexpr int kVBytes = kKeys * (HD / 2) * 2;  // 64 keys x this CTA's 64 dims: 8 KB
  static constexpr int kStages = 4;
  static constexpr int kSmem = kQBytes + kStages * (kKBytes + kVBytes) + 1024 + 512;
  static constexpr int kThreads = 192;
  static constexpr uint32_t kTmemCols = 256;         // S/P buffers at 0 and 64, O at 128
};

template <int POLY>
__global__ void __launch_bounds__(PairCfg::kThreads, 2)
    prefill_attn_pair_kernel(const __grid_constant__ CUtensorMap kvmap, const __grid_constant__ CUtensorMap qmap,
                             const FaParams p, const PrefillItem* __restrict__ items,
                             const int32_t* __restrict__ cta_off) {
  using C = PairCfg;
  constexpr int S = C::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;
  uint8_t* sK = smem + C::kQBytes;
  uint8_t* sV = sK + S * C::kKBytes;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sV + S * C::kVBytes);
  uint64_t* k_full = bar;            // leader's: both CTAs' K halves landed
  uint64_t* k_empty = k_full + S;    // each CTA's: QK of the slot's tile done
  uint64_t* v_full = k_empty + S;    // leader's
  uint64_t* v_empty = v_full + S;    // each CTA's
  uint64_t* s_full = v_empty + S;    // [2] each CTA's
  uint64_t* p_full = s_full + 2;     // [2] leader's: 4 softmax warps of each CTA
  uint64_t* o_full = p_full + 2;     // each CTA's: completes once per P.V
  uint64_t* o_final = o_full + 1;    // each CTA's: completes once per item
  uint64_t* q_full = o_final + 1;    // leader's: both Q tiles landed
  uint64_t* q_empty = q_full + 1;    // each CTA's: the item's last QK done
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(q_empty + 1);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;
  const int pair = int(blockIdx.x >> 1);
  const int g_begin = cta_off[pair], g_end = cta_off[pair + 1];
  const int group = p.H / p.Hkv;
  const int ppt = C::kRows / group;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_empty[i], 1);
      mbar_init(&v_full[i], 1);
      mbar_init(&v_empty[i], 1);
    }
    for (int b = 0; b < 2; ++b) {
      mbar_init(&s_full[b], 1);
      mbar_init(&p_full[b], 8);
    }
    mbar_init(o_full, 1);
    mbar_init(o_final, 1);
    mbar_init(q_full, 1);
    mbar_init(q_empty, 1);
    fence_mbar_init();
  }
  cluster_sync();  // both CTAs resident before the pair-wide TMEM allocation
  if (warp == 1) tmem_alloc2<C::kTmemCols>(tmem_slot);
  tc_fence_before();
  cluster_sync();  // barrier inits and the TMEM address visible pair-wide
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  griddep_wait();  // q and the appended K/V come from the previous kernel
  griddep_launch_dependents();

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer (both CTAs)
    if (elect_one()) {
      tma_prefetch_desc(&kvmap);
      tma_prefetch_desc(&qmap);
      const uint32_t kf0 = mapa_shared(smem_u32(k_full), 0), vf0 = mapa_shared(smem_u32(v_full), 0);
      const uint32_t qf0 = mapa_shared(smem_u32(q_full), 0);
      uint32_t jg = 0;
      for (int gi = g_begin, n = 0; gi < g_end; ++gi, ++n) {
        const PrefillItem it = items[2 * gi + int(rank)];
        const int nt = it.grp_last / C::kKeys + 1, last_blk = it.grp_last >> 4;
        const int32_t* trow = p.tables + size_t(it.table) * p.table_w;
        // tile j of this item into ring slot jg % S: K blocks 2r, 2r+1 (both 64-dim halves),
        // V dims [64r, 64r+64) of all 4 blocks; past the causal end a valid block (P = 0)
        auto load_kv = [&](int j) {
          const int s = int(jg % S);
          const uint32_t ph = (jg / S) & 1;
          mbar_wait(&k_empty[s], ph ^ 1);
          if (leader) mbar_arrive_expect_tx(&k_full[s], 2 * C::kKBytes);
#pragma unroll
          for (int bb = 0; bb < 2; ++bb) {
            const int blk = min(j * 4 + int(rank) * 2 + bb, last_blk);
            const int r = (__ldg(trow + blk) * p.Hkv + it.kv_head) * 16;
#pragma unroll
            for (int hf = 0; hf < 2; ++hf)
              tma_load_3d_2cta(sK + s * C::kKBytes + hf * 4096 + bb * 2048, &kvmap, kf0 + uint32_t(s) * 8, hf * 64, r,
                               p.layer * 2);
          }
          mbar_wait(&v_empty[s], ph ^ 1);
          if (leader) mbar_arrive_expect_tx(&v_full[s], 2 * C::kVBytes);
#pragma unroll
          for (int b = 0; b < 4; ++b) {
            const int blk = min(j * 4 + b, last_blk);
            const int r = (__ldg(trow + blk) * p.Hkv + it.kv_head) * 16;
            tma_load_3d_2cta(sV + s * C::kVBytes + b * 2048, &kvmap, vf0 + uint32_t(s) * 8, int(rank) * 64, r,
                             p.layer * 2 + 1);
          }
          ++jg;
        };
        // the item's first K/V tile goes out before its Q, which waits for the previous item's
        // last QK to release sQ
        load_kv(0);
        if (n > 0) mbar_wait(q_empty, uint32_t(n - 1) & 1);
        if (leader) mbar_arrive_expect_tx(q_full, 2u * 2u * 128u * uint32_t(group * ppt));
#pragma unroll
        for (int hf = 0; hf < 2; ++hf)
          tma_load_3d_2cta(sQ + hf * (C::kRows * 128), &qmap, qf0, hf * 64, it.kv_head * group, it.row0);
        for (int j = 1; j < nt; ++j) load_kv(j);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer (leader)
    if (leader && elect_one()) {
      constexpr uint32_t idesc_qk = umma_idesc_bf16(256, C::kKeys);
      constexpr uint32_t idesc_pv = (1u << 4) | (1u << 16) | ((uint32_t(C::HD) >> 3) << 17) | ((256u >> 4) << 24);
      auto issue_pv = [&](uint32_t tg, bool first) {
        const int s = int(tg % S);
        mbar_wait(&v_full[s], (tg / S) & 1);
        mbar_wait(&p_full[tg & 1], (tg >> 1) & 1);
        tc_fence_after();
        const uint32_t v_base = smem_u32(sV + s * C::kVBytes);
        const uint32_t p_tmem = tmem + (tg & 1) * 64;
#pragma unroll
        for (int kk = 0; kk < C::kKeys / 16; ++kk)
          umma_ts_2cta(tmem + 128, p_tmem + (kk >> 1) * 32 + (kk & 1) * 8, umma_desc_sw128_mn(v_base + kk * 2048, 8192),
                       idesc_pv, (!first || kk != 0) ? 1u : 0u);
        umma_commit_2cta(o_full);
        umma_commit_2cta(&v_empty[s]);
      };
      const uint32_t q_base = smem_u32(sQ);
      uint32_t jg = 0;
      for (int gi = g_begin, n = 0; gi < g_end; ++gi, ++n) {
        const int nt = items[2 * gi].grp_last / C::kKeys + 1;
        mbar_wait(q_full, uint32_t(n) & 1);
        tc_fence_after();
        for (int j = 0; j < nt; ++j) {
          const uint32_t tg = jg + uint32_t(j);
          const int s = int(tg % S);
          mbar_wait(&k_full[s], (tg / S) & 1);
          tc_fence_after();
          const uint32_t k_base = smem_u32(sK + s * C::kKBytes);
#pragma unroll
          for (int ks = 0; ks < C::HD / 16; ++ks)
            umma_bf16_2cta(tmem + (tg & 1) * 64, umma_desc_sw128(q_base + (ks >> 2) * (C::kRows * 128) + (ks & 3) * 32),
                           umma_desc_sw128(k_base + (ks >> 2) * 4096 + (ks & 3) * 32), idesc_qk, ks != 0);
          umma_commit_2cta(&s_full[tg & 1]);
          umma_commit_2cta(&k_empty[s]);
          if (j >= 1) issue_pv(tg - 1, j == 1);  // O += P(j-1) V(j-1) while the softmax works on S(j)
        }
        umma_commit_2cta(q_empty);  // every QK of this item issued: both sQ free once they complete
        issue_pv(jg + uint32_t(nt) - 1, nt == 1);
        umma_commit_2cta(o_final);
        jg += uint32_t(nt);
      }
    }
  } else {
    // ------------------------------------------------------------------ softmax + epilogue (both CTAs)
    const int row = (warp & 3) * 32 + lane;
    const uint32_t lane_base = tmem + (uint32_t((warp & 3) * 32) << 16);
    const uint32_t o_addr = lane_base + 128;
    const uint32_t pf0 = mapa_shared(smem_u32(p_full), 0);
    const int pi = row / group, hh = row % group;
    uint32_t jg = 0;
    for (int gi = g_begin, n = 0; gi < g_end; ++gi, ++n) {
      const PrefillItem it = items[2 * gi + int(rank)];
      const int nt = it.grp_last / C::kKeys + 1;
      const bool ok = row < ppt * group && pi < it.npos;
      const int pos_r = ok ? it.pos0 + pi : -1;
      const size_t tok_off = size_t(it.row0 + pi) * p.out_ld + size_t(it.kv_head * group + hh) * C::HD;
      const int warp_min_pos = __shfl_sync(0xffffffffu, pos_r < 0 ? INT_MAX : pos_r, 0);
      float m_used = -INFINITY, l = 0.f;
      for (int j = 0; j < nt; ++j) {
        const uint32_t tg = jg + uint32_t(j);
        const int sb = int(tg & 1);
        mbar_wait(&s_full[sb], (tg >> 1) & 1);
        tc_fence_after();
        const uint32_t s_addr = lane_base + uint32_t(sb) * 64;
        const int key0 = j * C::kKeys;
        const bool masked = __any_sync(0xffffffffu, key0 + C::kKeys - 1 > (pos_r < 0 ? -1 : pos_r)) ||
                            warp_min_pos == INT_MAX;
        uint32_t r[C::kKeys];
#pragma unroll
        for (int c = 0; c < C::kKeys / 16; ++c)
          tmem_ld32x32b_x16(s_addr + c * 16, *reinterpret_cast<uint32_t(*)[16]>(&r[c * 16]));
        tmem_ld_wait();
        if (masked) {
          const int lim = (pos_r < 0 ? -1 : pos_r) - key0;
#pragma unroll
          for (int i = 0; i < C::kKeys; ++i)
            if (i > lim) r[i] = 0xff800000u;  // -inf
        }
        float mq[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
        for (int i = 0; i < C::kKeys; i += 2)
          mq[(i >> 1) & 3] = fmax3(mq[(i >> 1) & 3], __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
        float mx = fmax3(mq[0], mq[1], fmaxf(mq[2], mq[3]));
        mx *= p.scale_log2;
        const bool rescale = mx > m_used + QOS_FA_LAZY;
        const float m_new = rescale ? mx : m_used;
        const float alpha = (rescale && m_used != -INFINITY) ? ex2(m_used - m_new) : 1.f;
        const float mb = (m_new == -INFINITY) ? 0.f : m_new;
        float2 sum2[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
        const float2 scale2 = make_float2(p.scale_log2, p.scale_log2), nmb2 = make_float2(-mb, -mb);
#pragma unroll
        for (int c = 0; c < C::kKeys / 32; ++c) {
          uint32_t hi[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            const float2 x = fma2(make_float2(__uint_as_float(r[c * 32 + 2 * i]), __uint_as_float(r[c * 32 + 2 * i + 1])),
                                  scale2, nmb2);
            float2 pp = (POLY > 0 && i % (POLY > 0 ? POLY : 1) == (POLY > 0 ? POLY : 1) - 1) ? ex2_poly2(x) : make_float2(ex2(x.x), ex2(x.y));
            hi[i] = pack_f16(pp.x, pp.y);
            sum2[i & 3] = add2(sum2[i & 3], pp);
          }
          tmem_st32x32b_x16(s_addr + c * 32, hi);
        }
        const float2 s01 = add2(sum2[0], sum2[1]), s23 = add2(sum2[2], sum2[3]);
        const float sum = (s01.x + s23.x) + (s01.y + s23.y);
        tmem_st_wait();
        l = l * alpha + sum;
        if (j >= 1 && __any_sync(0xffffffffu, alpha != 1.f)) {
          // PV(tg-2) completed before QK(tg) (awaited above): o_full has completed tg-1 or tg times
          mbar_wait(o_full, (tg - 1) & 1);
          tc_fence_after();
#pragma unroll 1
          for (int c = 0; c < C::HD / 16; ++c) {
            uint32_t r2[16];
            tmem_ld32x32b_x16(o_addr + c * 16, r2);
            tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 16; ++i) r2[i] = __float_as_uint(__uint_as_float(r2[i]) * alpha);
            tmem_st32x32b_x16(o_addr + c * 16, r2);
          }
          tmem_st_wait();
        }
        m_used = m_new;
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive_remote(pf0 + uint32_t(sb) * 8);
      }
      mbar_wait(o_final, uint32_t(n) & 1);
      tc_fence_after();
      const float inv = (l > 0.f) ? 1.f / l : 0.f;
#pragma unroll 1
      for (int c = 0; c < C::HD / 32; ++c) {
        uint32_t r2[32];
        tmem_ld32x32b_x16(o_addr + c * 32, *reinterpret_cast<uint32_t(*)[16]>(&r2[0]));
        tmem_ld32x32b_x16(o_addr + c * 32 + 16, *reinterpret_cast<uint32_t(*)[16]>(&r2[16]));
        tmem_ld_wait();
        if (pos_r >= 0 && !it.pad) {
          if (p.out_f32) {
            float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(p.out) + tok_off + c * 32);
#pragma unroll
            for (int i = 0; i < 8; ++i)
              dst[i] = make_float4(__uint_as_float(r2[4 * i]) * inv, __uint_as_float(r2[4 * i + 1]) * inv,
                                   __uint_as_float(r2[4 * i + 2]) * inv, __uint_as_float(r2[4 * i + 3]) * inv);
          } else {
            uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.out) + tok_off + c * 32);
#pragma unroll
            for (int i = 0; i < 4; ++i)
              dst[i] = make_uint4(pack_bf16(__uint_as_float(r2[8 * i]) * inv, __uint_as_float(r2[8 * i + 1]) * inv),
                                  pack_bf16(__uint_as_float(r2[8 * i + 2]) * inv, __uint_as_float(r2[8 * i + 3]) * inv),
                                  pack_bf16(__uint_as_float(r2[8 * i + 4]) * inv, __uint_as_float(r2[8 * i + 5]) * inv),
                                  pack_bf16(__uint_as_float(r2[8 * i + 6]) * inv, __uint_as_float(r2[8 * i + 7]) * inv));
          }
        }
      }
      jg += uint32_t(nt);
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();  // the leader's MMAs / commits into this CTA and the peer's remote arrivals are done
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc2<C::kTmemCols>(tmem);
  }
}

// ---------------------------------------------------------------- ping-pong variant (fa_qtiles=2)
// Two q tiles per CTA (one CTA per SM), 128-key K/V tiles, one S/P buffer per q tile (TMEM:
// S0 [0,128) S1 [128,256) O0 [256,384) O1 [384,512)).  QKᵀ runs as UMMA N = 128 (twice the
// work per instruction of the 64-key kernel) and the tensor core alternates between the two
// q tiles: while softmax group 1 works on S1(j) it executes PV0(j) and QK0(j+1), while group
// 0 works on S0(j+1) it executes PV1(j) and QK1(j+1).  QK_g(j+1) is issued after PV_g(j)
// (same TMEM columns; tcgen05 ops run in issue order), so when a softmax group sees S_g(j+1)
// its PV_g(j) has landed and it may rescale O_g without a wait.
template <int HD>
struct PpCfg {
  static constexpr int kRows = 128, kKeys = 128, kHalves = HD / 64;
  static constexpr int kQBytes = kRows * HD * 2;      // 32 KB at HD 128
  static constexpr int kTileBytes = kKeys * HD * 2;   // 32 KB: one K or V tile
  static constexpr int kStages = 2;
  static constexpr int kSmem = 2 * kQBytes + 2 * kStages * kTileBytes + 1024 + 512 + 2 * 2 * 128 * 4;
  // 2 TMA/MMA warps + per q tile 8 softmax warps: two threads per row, each owning 64 of the
  // tile's 128 keys (and 64 of the row's HD/... output columns for rescale and epilogue)
  static constexpr int kThreads = 64 + 2 * 256;
  static constexpr uint32_t col_s(int g) { return uint32_t(g * 128); }
  static constexpr uint32_t col_o(int g) { return uint32_t(256 + g * HD); }
};

template <int HD, int POLY>
__global__ void __launch_bounds__(PpCfg<HD>::kThreads, 1)
    prefill_attn_pp_kernel(const __grid_constant__ CUtensorMap kvmap, const FaParams p,
                           const PrefillItem* __restrict__ items) {
  using C = PpCfg<HD>;
  constexpr int S = C::kStages;
  constexpr int KH = C::kKeys / 2;   // keys per softmax thread
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sQ = smem;                          // 2 x kQBytes
  uint8_t* sK = smem + 2 * C::kQBytes;
  uint8_t* sV = sK + S * C::kTileBytes;
  uint64_t* bar = reinterpret_cast<uint64_t*>(sV + S * C::kTileBytes);
  uint64_t* k_full = bar;
  uint64_t* k_empty = k_full + S;
  uint64_t* v_full = k_empty + S;
  uint64_t* v_empty = v_full + S;
  uint64_t* s_full = v_empty + S;   // [2]
  uint64_t* p_full = s_full + 2;    // [2]
  uint64_t* o_final = p_full + 2;   // [2]
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(o_final + 2);
  float* xch = reinterpret_cast<float*>(bar + 64);   // [2 groups][2 halves][128 rows]: row max / sum exchange

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const PrefillItem it0 = items[blockIdx.x * 2];
  const int group = p.H / p.Hkv;
  const int ppt = C::kRows / group;
  const int last_pos = it0.grp_last;
  const int ntiles = last_pos / C::kKeys + 1;
  const int last_blk = last_pos >> 4;

  if (threadIdx.x == 0) {
    for (int i = 0; i < S; ++i) {
      mbar_init(&k_full[i], 1);
      mbar_init(&k_empty[i], 1);
      mbar_init(&v_full[i], 1);
      mbar_init(&v_empty[i], 1);
    }
    for (int g = 0; g < 2; ++g) {
      mbar_init(&s_full[g], 1);
      mbar_init(&p_full[g], 256);
      mbar_init(&o_final[g], 1);
    }
    fence_mbar_init();
  }
  if (warp == 1) tmem_alloc<512>(tmem_slot);
  griddep_wait();
  griddep_launch_dependents();

  // softmax warp w >= 2: q tile qg, key half kh, TMEM lane quarter w & 3
  const int sw = warp - 2;
  const int qg = warp >= 2 ? sw >> 3 : 0;
  const int kh = warp >= 2 ? (sw >> 2) & 1 : 0;
  const PrefillItem it = items[blockIdx.x * 2 + qg];
  int row = 0, pos_r = -1;
  size_t tok_off = 0;
  if (warp >= 2) {
    row = (warp & 3) * 32 + lane;
    const int pi = row / group, hh = row % group;
    const bool ok = row < ppt * group && pi < it.npos;
    pos_r = ok ? it.pos0 + pi : -1;
    tok_off = size_t(it.row0 + pi) * p.out_ld + size_t(it.kv_head * group + hh) * HD;
    if (kh == 0) {  // the first half's threads stage the q row
      const __nv_bfloat16* src = p.q + size_t(it.row0 + pi) * p.q_ld + size_t(it.kv_head * group + hh) * HD;
      uint8_t* q_dst = sQ + qg * C::kQBytes;
      uint4 v[HD / 8];
#pragma unroll
      for (int ch = 0; ch < HD / 8; ++ch) v[ch] = ok ? *reinterpret_cast<const uint4*>(src + ch * 8) : make_uint4(0, 0, 0, 0);
#pragma unroll
      for (int ch = 0; ch < HD / 8; ++ch) {
        const int hf = ch >> 3, c = ch & 7;
        *reinterpret_cast<uint4*>(q_dst + hf * (C::kRows * 128) + row * 128 + ((c ^ (row & 7)) << 4)) = v[ch];
      }
      fence_proxy_async_smem();
    }
  }
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp == 0) {
    // ------------------------------------------------------------------ TMA producer
    if (elect_one()) {
      tma_prefetch_desc(&kvmap);
      const int32_t* trow = p.tables + size_t(it0.table) * p.table_w;
      auto load_tile = [&](uint8_t* dst, uint64_t* full, int j, int plane) {
        for (int b = 0; b < C::kKeys / 16; ++b) {
          const int blk = min(j * (C::kKeys / 16) + b, last_blk);
          const int r = (__ldg(trow + blk) * p.Hkv + it0.kv_head) * 16;
#pragma unroll
          for (int hf = 0; hf < C::kHalves; ++hf)
            tma_load_3d(dst + hf * (C::kKeys * 128) + b * 2048, &kvmap, full, hf * 64, r, p.layer * 2 + plane);
        }
      };
      for (int j = 0; j < ntiles; ++j) {
        const int s = j % S;
        const uint32_t ph = (j / S) & 1;
        mbar_wait(&k_empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&k_full[s], C::kTileBytes);
        load_tile(sK + s * C::kTileBytes, &k_full[s], j, 0);
        mbar_wait(&v_empty[s], ph ^ 1);
        mbar_arrive_expect_tx(&v_full[s], C::kTileBytes);
        load_tile(sV + s * C::kTileBytes, &v_full[s], j, 1);
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------------ MMA issuer
    if (elect_one()) {
      constexpr uint32_t idesc_qk = umma_idesc_bf16(128, C::kKeys);
      constexpr uint32_t idesc_pv = (1u << 4) | (1u << 16) | ((uint32_t(HD) >> 3) << 17) | ((128u >> 4) << 24);
      auto issue_qk = [&](int g, int j) {
        const int s = j % S;
        const uint32_t k_base = smem_u32(sK + s * C::kTileBytes);
        const uint32_t q_base = smem_u32(sQ + g * C::kQBytes);
#pragma unroll
        for (int ks = 0; ks < HD / 16; ++ks) {
          const uint32_t qoff = (ks >> 2) * (C::kRows * 128) + (ks & 3) * 32;
          const uint32_t koff = (ks >> 2) * (C::kKeys * 128) + (ks & 3) * 32;
          if (POLY != -3)
            umma_bf16(tmem + C::col_s(g), umma_desc_sw128(q_base + qoff), umma_desc_sw128(k_base + koff), idesc_qk, ks != 0);
        }
        umma_commit(&s_full[g]);
      };
      auto issue_pv = [&](int g, int j) {
        const int s = j % S;
        mbar_wait(&p_full[g], j & 1);
        tc_fence_after();
        const uint32_t v_base = smem_u32(sV + s * C::kTileBytes);
#pragma unroll
        for (int kk = 0; kk < C::kKeys / 16; ++kk) {
          const uint64_t vd = umma_desc_sw128_mn(v_base + kk * 2048, C::kKeys * 128);
          const uint32_t pc = tmem + C::col_s(g) + (kk >> 1) * 32 + (kk & 1) * 8;
          if (POLY != -2) umma_bf16_ts(tmem + C::col_o(g), pc, vd, idesc_pv, (j | kk) != 0);
        }
      };
      mbar_wait(&k_full[0], 0);
      tc_fence_after();
      issue_qk(0, 0);
      issue_qk(1, 0);
      umma_commit(&k_empty[0]);
      for (int j = 0; j < ntiles; ++j) {
        const int s = j % S, s1 = (j + 1) % S;
        const bool more = j + 1 < ntiles;
        mbar_wait(&v_full[s], (j / S) & 1);
        issue_pv(0, j);                       // O0 += P0(j) V(j)
        if (more) {                           // S0(j+1) = Q0 K(j+1)^T (after PV0(j): same columns)
          mbar_wait(&k_full[s1], ((j + 1) / S) & 1);
          tc_fence_after();
          issue_qk(0, j + 1);
        }
        issue_pv(1, j);                       // O1 += P1(j) V(j)
        umma_commit(&v_empty[s]);
        if (more) {
          issue_qk(1, j + 1);
          umma_commit(&k_empty[s1]);
        }
      }
      umma_commit(&o_final[0]);
      umma_commit(&o_final[1]);
    }
  } else {
    // ------------------------------------------------------------------ softmax (q tile qg, key half kh)
    const uint32_t lane_base = tmem + (uint32_t((warp & 3) * 32) << 16);
    const uint32_t s_addr = lane_base + C::col_s(qg) + kh * (KH / 2);  // this half's 32 fp16-pair columns...
    const uint32_t s_rd = lane_base + C::col_s(qg) + kh * KH;          // ...and its 64 fp32 S columns
    const uint32_t o_addr = lane_base + C::col_o(qg) + kh * (HD / 2);
    const int bar_id = 1 + qg * 4 + (warp & 3);   // the two warps (halves) of one row quarter
    float* my_x = xch + (qg * 2 + kh) * 128;
    const float* pe_x = xch + (qg * 2 + (kh ^ 1)) * 128;
    auto pair_sync = [&]() { asm volatile("bar.sync %0, 64;" ::"r"(bar_id) : "memory"); };
    const int warp_min_pos = __shfl_sync(0xffffffffu, pos_r < 0 ? INT_MAX : pos_r, 0);
    float m_used = -INFINITY, l = 0.f;
    for (int j = 0; j < ntiles; ++j) {
      mbar_wait(&s_full[qg], j & 1);
      tc_fence_after();
      if (POLY < 0) {
        tc_fence_before();
        mbar_arrive(&p_full[qg]);
        continue;
      }
      const int key0 = j * C::kKeys + kh * KH;
      const bool masked = __any_sync(0xffffffffu, key0 + KH - 1 > (pos_r < 0 ? -1 : pos_r)) || warp_min_pos == INT_MAX;
      uint32_t r[KH];
#pragma unroll
      for (int c = 0; c < KH / 16; ++c)
        tmem_ld32x32b_x16(s_rd + c * 16, *reinterpret_cast<uint32_t(*)[16]>(&r[c * 16]));
      tmem_ld_wait();
      if (masked) {
        const int lim = (pos_r < 0 ? -1 : pos_r) - key0;
#pragma unroll
        for (int i = 0; i < KH; ++i)
          if (i > lim) r[i] = 0xff800000u;
      }
      float mq[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
      for (int i = 0; i < KH; i += 2)
        mq[(i >> 1) & 3] = fmax3(mq[(i >> 1) & 3], __uint_as_float(r[i]), __uint_as_float(r[i + 1]));
      float mx = fmax3(mq[0], mq[1], fmaxf(mq[2], mq[3]));
      // row max over both halves (partner thread: same row, other key half)
      my_x[row] = mx;
      pair_sync();
      mx = fmaxf(mx, pe_x[row]) * p.scale_log2;
      const bool rescale = mx > m_used + QOS_FA_LAZY;
      const float m_new = rescale ? mx : m_used;
      const float alpha = (rescale && m_used != -INFINITY) ? ex2(m_used - m_new) : 1.f;
      const float mb = (m_new == -INFINITY) ? 0.f : m_new;
      float2 sum2[4] = {make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f), make_float2(0.f, 0.f)};
      const float2 scale2 = make_float2(p.scale_log2, p.scale_log2), nmb2 = make_float2(-mb, -mb);
#pragma unroll
      for (int c = 0; c < KH / 32; ++c) {
        uint32_t hi[16];
#pragma unroll
        for (int i = 0; i < 16; ++i) {
          const float2 x = fma2(make_float2(__uint_as_float(r[c * 32 + 2 * i]), __uint_as_float(r[c * 32 + 2 * i + 1])),
                                scale2, nmb2);
          float2 pp = (POLY > 0 && i % (POLY > 0 ? POLY : 1) == (POLY > 0 ? POLY : 1) - 1) ? ex2_poly2(x) : make_float2(ex2(x.x), ex2(x.y));
          hi[i] = pack_f16(pp.x, pp.y);
          sum2[i & 3] = add2(sum2[i & 3], pp);
        }
        // keys [32c', 32c'+32) of the tile (c' = kh*2 + c) -> fp16 pairs at columns [32c', 32c'+16)
        tmem_st32x32b_x16(lane_base + C::col_s(qg) + (kh * 2 + c) * 32, hi);
      }
      (void)s_addr;
      const float2 s01 = add2(sum2[0], sum2[1]), s23 = add2(sum2[2], sum2[3]);
      l = l * alpha + ((s01.x + s23.x) + (s01.y + s23.y));   // this half's share of the row sum
      if (j >= 1 && __any_sync(0xffffffffu, alpha != 1.f)) {
        // PV_g(j-1) was issued before QK_g(j), whose completion was awaited above
#pragma unroll 1
        for (int c = 0; c < HD / 32; ++c) {
          uint32_t r2[16];
          tmem_ld32x32b_x16(o_addr + c * 16, r2);
          tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 16; ++i) r2[i] = __float_as_uint(__uint_as_float(r2[i]) * alpha);
          tmem_st32x32b_x16(o_addr + c * 16, r2);
        }
      }
      tmem_st_wait();
      m_used = m_new;
      tc_fence_before();
      mbar_arrive(&p_full[qg]);
    }
    // row sum over both halves
    pair_sync();   // the partner has read my_x of the last tile
    my_x[row] = l;
    pair_sync();
    l += pe_x[row];
    mbar_wait(&o_final[qg], 0);
    tc_fence_after();
    const float inv = (l > 0.f) ? 1.f / l : 0.f;
#pragma unroll 1
    for (int c = 0; c < HD / 64; ++c) {
      uint32_t r2[32];
      tmem_ld32x32b_x16(o_addr + c * 32, *reinterpret_cast<uint32_t(*)[16]>(&r2[0]));
      tmem_ld32x32b_x16(o_addr + c * 32 + 16, *reinterpret_cast<uint32_t(*)[16]>(&r2[16]));
      tmem_ld_wait();
      const size_t off = tok_off + kh * (HD / 2) + c * 32;
      if (pos_r >= 0 && !it.pad) {
        if (p.out_f32) {
          float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(p.out) + off);
#pragma unroll
          for (int i = 0; i < 8; ++i)
            dst[i] = make_float4(__uint_as_float(r2[4 * i]) * inv, __uint_as_float(r2[4 * i + 1]) * inv,
                                 __uint_as_float(r2[4 * i + 2]) * inv, __uint_as_float(r2[4 * i + 3]) * inv);
        } else {
          uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.out) + off);
#pragma unroll
          for (int i = 0; i < 4; ++i)
            dst[i] = make_uint4(pack_bf16(__uint_as_float(r2[8 * i]) * inv, __uint_as_float(r2[8 * i + 1]) * inv),
                                pack_bf16(__uint_as_float(r2[8 * i + 2]) * inv, __uint_as_float(r2[8 * i + 3]) * inv),
                                pack_bf16(__uint_as_float(r2[8 * i + 4]) * inv, __uint_as_float(r2[8 * i + 5]) * inv),
                                pack_bf16(__uint_as_float(r2[8 * i + 6]) * inv, __uint_as_float(r2[8 * i + 7]) * inv));
        }
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<512>(tmem);
  }
}

static int g_fa_poly = getenv("QOS_FA_POLY") ? atoi(getenv("QOS_FA_POLY")) : 4;
static int g_fa_tma5 = 1;
static int g_fa_psplit = 1;
static int g_fa_kvfirst = 0;  // neutral in ncu cycles (profiles/ncu_ab_fa_r2c.jsonl)

template <int HD, int POLY, int NQ>
static cudaError_t prefill_tc_t(const AttnLaunch& a, const PrefillItem* items, int n_items, cudaStream_t st) {
  using C = FaCfg<HD, NQ>;
  static std::atomic<uint64_t> set{0};
  if (cudaError_t e = smem_attr_once(prefill_attn_tc_kernel<HD, POLY, NQ>, int(C::kSmem), set); e != cudaSuccess) return e;
  FaParams p;
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
  if (n_items % NQ) return cudaErrorInvalidValue;  // the item list comes in whole groups
  return launch_pdl(prefill_attn_tc_kernel<HD, POLY, NQ>, dim3(n_items / NQ), dim3(C::kThreads), C::kSmem, st,
                    *a.kv_tmap, p, items);
}

template <int HD, int POLY>
static cudaError_t prefill_pp_t(const AttnLaunch& a, const PrefillItem* items, int n_items, cudaStream_t st) {
  using C = PpCfg<HD>;
  static std::atomic<uint64_t> set{0};
  if (cudaError_t e = smem_attr_once(prefill_attn_pp_kernel<HD, POLY>, int(C::kSmem), set); e != cudaSuccess) return e;
  FaParams p;
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
  if (n_items % 2) return cudaErrorInvalidValue;
  return launch_pdl(prefill_attn_pp_kernel<HD, POLY>, dim3(n_items / 2), dim3(C::kThreads), C::kSmem, st, *a.kv_tmap,
                    p, items);
}

template <int HD, int POLY>
static cudaError_t prefill_persist_t(const AttnLaunch& a, const PrefillItem* items, const int32_t* cta_off, int n_cta,
                                     cudaStream_t st) {
  using C = FaCfg<HD, 1>;
  const int group = a.H / a.Hkv;
  CUtensorMap qm;
  const CUtensorMap* qmp = a.q_tmap;
  if (!qmp) {  // op entry points: a map over this launch's q buffer
    if (make_tmap_3d_bf16_strided(&qm, a.q, uint64_t(HD), uint64_t(a.H), uint64_t(a.q_rows), uint64_t(HD) * 2,
                                  uint64_t(a.q_ld) * 2, 64, uint32_t(group), uint32_t(C::kRows / group)) != QOS_OK)
      return cudaErrorInvalidValue;
    qmp = &qm;
  }
  static std::atomic<uint64_t> set{0};
  if (cudaError_t e = smem_attr_once(prefill_attn_persist_kernel<HD, POLY>, int(C::kSmem), set); e != cudaSuccess)
    return e;
  FaParams p;
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
  p.kv_first = g_fa_kvfirst;
  p.tma5 = (g_fa_tma5 && a.kv_tmap5) ? 1 : 0;
  p.psplit = g_fa_psplit;
  return launch_pdl(prefill_attn_persist_kernel<HD, POLY>, dim3(n_cta), dim3(C::kThreads), C::kSmem, st, *a.kv_tmap,
                    *qmp, a.kv_tmap5 ? *a.kv_tmap5 : *a.kv_tmap, p, items, cta_off);
}

template <int POLY>
static cudaError_t prefill_pair_t(const AttnLaunch& a, const PrefillItem* items, const int32_t* cta_off, int n_pairs,
                                  cudaStream_t st) {
  using C = PairCfg;
  const int group = a.H / a.Hkv;
  CUtensorMap qm;
  const CUtensorMap* qmp = a.q_tmap;
  if (!qmp) {
    if (make_tmap_3d_bf16_strided(&qm, a.q, uint64_t(C::HD), uint64_t(a.H), uint64_t(a.q_rows), uint64_t(C::HD) * 2,
                                  uint64_t(a.q_ld) * 2, 64, uint32_t(group), uint32_t(C::kRows / group)) != QOS_OK)
      return cudaErrorInvalidValue;
    qmp = &qm;
  }
  static std::atomic<uint64_t> set{0};
  if (cudaError_t e = smem_attr_once(prefill_attn_pair_kernel<POLY>, int(C::kSmem), set); e != cudaSuccess) return e;
  FaParams p;
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
  return launch_pdl_cluster(prefill_attn_pair_kernel<POLY>, dim3(2 * n_pairs), dim3(C::kThreads), C::kSmem, 2, st,
                            *a.kv_tmap, *qmp, p, items, cta_off);
}

int prefill_pair_max_clusters() {
  static std::atomic<uint64_t> set{0};
  if (smem_attr_once(prefill_attn_pair_kernel<4>, int(PairCfg::kSmem), set) != cudaSuccess) return 0;
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = dim3(2);
  cfg.blockDim = dim3(PairCfg::kThreads);
  cfg.dynamicSmemBytes = PairCfg::kSmem;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = 2;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  int n = 0;
  if (cudaOccupancyMaxActiveClusters(&n, prefill_attn_pair_kernel<4>, &cfg) != cudaSuccess) {
    cudaGetLastError();
    return 0;
  }
  return n;
}

void set_fa_poly(int n) { g_fa_poly = n; }
void set_fa_kvfirst(int v) { g_fa_kvfirst = v; }
void set_fa_tma5(int v) { g_fa_tma5 = v; }
void set_fa_psplit(int v) { g_fa_psplit = v; }

int prefill_tc_positions_per_tile(int group) { return 128 / group; }

cudaError_t launch_prefill_attention_tc(const AttnLaunch& a, const PrefillItem* items, int n_items, cudaStream_t st) {
  if (n_items == 0) return cudaSuccess;
  count_launch(1);
  const int poly = g_fa_poly;
  if (a.pair) {  // CTA pairs over per-pair lists of q-tile pairs (cta_off in pairs of items)
    if (a.hd != 128 || !a.cta_off || a.q_tiles != 2) return cudaErrorInvalidValue;
    return poly == 0 ? prefill_pair_t<0>(a, items, a.cta_off, a.n_cta, st) : prefill_pair_t<4>(a, items, a.cta_off, a.n_cta, st);
  }
  if (a.cta_off && a.q_tiles == 1 && poly >= 0) {  // persistent CTAs over per-CTA item lists
    if (a.hd == 128) return poly == 0   ? prefill_persist_t<128, 0>(a, items, a.cta_off, a.n_cta, st)
                            : poly == 2 ? prefill_persist_t<128, 2>(a, items, a.cta_off, a.n_cta, st)
                            : poly == 3 ? prefill_persist_t<128, 3>(a, items, a.cta_off, a.n_cta, st)
                                        : prefill_persist_t<128, 4>(a, items, a.cta_off, a.n_cta, st);
    if (a.hd == 64) return poly == 0 ? prefill_persist_t<64, 0>(a, items, a.cta_off, a.n_cta, st)
                                     : prefill_persist_t<64, 4>(a, items, a.cta_off, a.n_cta, st);
    return cudaErrorInvalidValue;
  }
  const int nq = a.q_tiles;
  if (nq != 1 && nq != 2) return cudaErrorInvalidValue;
#define QOS_FA_NQ(HDV, PV) \
  return nq == 1 ? prefill_tc_t<HDV, PV, 1>(a, items, n_items, st) : prefill_pp_t<HDV, PV>(a, items, n_items, st);
  if (a.hd == 128) {
    // measurement-only variants: -1 no softmax, -2 also no P.V MMAs, -3 no softmax and no QK MMAs
    if (poly == -1) { QOS_FA_NQ(128, -1) }
    if (poly == -2) { QOS_FA_NQ(128, -2) }
    if (poly == -3) { QOS_FA_NQ(128, -3) }
    if (poly == 0) { QOS_FA_NQ(128, 0) }
    if (poly == 2) { QOS_FA_NQ(128, 2) }
    QOS_FA_NQ(128, 4)
  }
  if (a.hd == 64) {
    if (poly == 0) { QOS_FA_NQ(64, 0) }
    QOS_FA_NQ(64, 4)
  }
#undef QOS_FA_NQ
  return cudaErrorInvalidValue;
}

}  // namespace qos
