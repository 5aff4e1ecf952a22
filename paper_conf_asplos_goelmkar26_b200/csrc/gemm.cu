// gemm.cu — persistent warp-specialised tcgen05 GEMM for the dense projections of the fused
// token batch (SURVEY.md §8(a) rows a4 QKV, a9 O, a11 gate/up + SiLU-gate, a12 down, a13 LM
// head; the paper's "fused prefill-decode MLP", §3.3).
//
//   C[M][N] = epi( A[M][K] · B[N][K]^T ),  A = activations (tokens x K), B = nn.Linear weight.
//
// Design:
//   * tile 128 x BN x 64 (BN = 128 | 256), UMMA M=128 N=BN K=16 (cta_group::1), bf16 -> fp32;
//   * operands staged by TMA (cp.async.bulk.tensor.2d, 128-B swizzle) into a STAGES-deep
//     smem ring guarded by full/empty mbarriers;
//   * warp 0 = TMA producer, warp 1 = MMA issuer (one elected lane) + TMEM owner,
//     warps 2..5 = epilogue (TMEM -> registers -> global), one accumulator row per thread;
//   * two TMEM accumulators (2 x BN fp32 columns) so the epilogue of tile i overlaps the
//     MMAs of tile i+1;
//   * persistent grid (<= #SMs CTAs), tiles ordered N-major / M-minor so the CTAs working at
//     one time share a weight (B) tile and the activation matrix stays L2-resident.
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>

#include <climits>

#include "common.cuh"
#include "internal.h"

namespace qos {

// Programmatic dependent launch switch for the step-chain kernels (see common.cuh).
static int g_pdl = -1;
bool pdl_enabled() {
  if (g_pdl < 0) {
    const char* v = getenv("QOS_PDL");
    g_pdl = (v && atoi(v) == 0) ? 0 : 1;
  }
  return g_pdl != 0;
}
void set_pdl(bool on) { g_pdl = on ? 1 : 0; }

constexpr int kBM = 128;
constexpr int kBK = 64;
constexpr int kGemmThreads = 192;

template <int BN>
struct GemmCfg {
  static constexpr int kStages = (BN == 256) ? 4 : 6;
  static constexpr int kABytes = kBM * kBK * 2;
  static constexpr int kBBytes = BN * kBK * 2;
  static constexpr int kStageBytes = kABytes + kBBytes;
  static constexpr int kTmemCols = 2 * BN;
  // per epilogue warp: a 32-row staging tile (up to 256 B per row) so that the warp's stores
  // are coalesced row segments instead of one row per thread
  static constexpr int kStageWarpBytes = 32 * 256;
  static constexpr int kSmemBytes = kStages * kStageBytes + 1024 /*align*/ + 256 /*barriers*/ + 4 * kStageWarpBytes;
};

struct GemmArgs {
  int M, N, K;
  int mt, nt;       // tiles along M and N
  int ksplit;       // K slices per tile (split-K for weight-bound small-M GEMMs); 1 = off
  int sk;           // stream-K: the (tile, k-block) space in equal contiguous ranges per CTA
  int coop;         // stream-K: cut tiles reduced by all their CTAs after their ranges
  int ordered;      // split-K of EPI_ADD_F32 (ksplit > 1): every slice red.adds its partial into
                    // C in slice order (slice s waits for counters[tile] == s): no partials,
                    // deterministic; units split-major so a slice never waits on a later unit
  int64_t work;     // stream-K: mt * nt * kblocks
  void* C;
  int ldc;          // elements
  const float* bias;
  float* part;      // split-K partials [unit][128][BN] fp32 (ksplit > 1)
  int* counters;    // split-K arrival counter per tile (ksplit > 1), zero between launches
  int a_row0;       // first row of A (TMA coordinate offset): GEMM over a row range of a buffer
  // EPI_QKV_ROPE: RoPE on q and k at each row's position; q -> C, k / v -> the paged cache
  const int32_t* pos;     // [M] positions of the rows
  const int32_t* slot;    // [M] cache slots (block * 16 + offset)
  const float2* rope;     // [max_pos][hd/2] (cos, sin)
  __nv_bfloat16* kplane;  // [blocks][Hkv][16][hd] of this layer
  __nv_bfloat16* vplane;
  int H, Hkv, hd;
  // folded RMSNorm (NormFold, internal.h)
  const float* rs_in;
  float* ss_out;
  float* rs_out;
  int* fcnt;
  const __nv_bfloat16* g_out;
  __nv_bfloat16* h_out;
  int ss_n;
  float inv_d, rms_eps;
  void* scat[8];  // reduce-scatter destinations (NormFold::scat), scat_rs = 0: plain store to C
  int scat_rs;
  int rel_cluster;  // CTA-pair kernel: accumulator release with .release.cluster (experiment; 0 = .cta)
};

static void set_fold(GemmArgs& a, const NormFold* f) {
  a.rs_in = f ? f->rs_in : nullptr;
  a.ss_out = f ? f->ss_out : nullptr;
  a.rs_out = f ? f->rs_out : nullptr;
  a.fcnt = f ? f->cnt : nullptr;
  a.g_out = f ? reinterpret_cast<const __nv_bfloat16*>(f->g_out) : nullptr;
  a.h_out = f ? reinterpret_cast<__nv_bfloat16*>(f->h_out) : nullptr;
  a.ss_n = f ? f->ss_n : 0;
  a.inv_d = f && f->d ? 1.f / float(f->d) : 0.f;
  a.rms_eps = f ? f->eps : 0.f;
  for (int k = 0; k < 8; ++k) a.scat[k] = f ? f->scat[k] : nullptr;
  a.scat_rs = f ? f->scat_rs : 0;
}

// ---- epilogue stores of one thread's 32 consecutive accumulator columns of one row
template <int EPI>
QOS_DEV void epi_store32(const GemmArgs& p, int row, int col, const float (&v)[32]) {
  if constexpr (EPI == EPI_STORE_BF16 || EPI == EPI_BIAS_BF16) {
    uint32_t pk[16];
#pragma unroll
    for (int i = 0; i < 16; ++i) {
      float a0 = v[2 * i], a1 = v[2 * i + 1];
      if constexpr (EPI == EPI_BIAS_BF16) {
        a0 += __ldg(p.bias + col + 2 * i);
        a1 += __ldg(p.bias + col + 2 * i + 1);
      }
      pk[i] = pack_bf16(a0, a1);
    }
    uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.C) + size_t(row) * p.ldc + col);
#pragma unroll
    for (int i = 0; i < 4; ++i) dst[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
  } else if constexpr (EPI == EPI_STORE_F32) {
    float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(p.C) + size_t(row) * p.ldc + col);
#pragma unroll
    for (int i = 0; i < 8; ++i) dst[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
  } else if constexpr (EPI == EPI_ADD_F32) {
    float4* dst = reinterpret_cast<float4*>(reinterpret_cast<float*>(p.C) + size_t(row) * p.ldc + col);
    float4 old[8];
#pragma unroll
    for (int i = 0; i < 8; ++i) old[i] = dst[i];
#pragma unroll
    for (int i = 0; i < 8; ++i)
      dst[i] = make_float4(old[i].x + v[4 * i], old[i].y + v[4 * i + 1], old[i].z + v[4 * i + 2], old[i].w + v[4 * i + 3]);
  }
}
// SiLU-gate: 32 gate columns + the 32 matching up columns -> 32 output columns
QOS_DEV void epi_silu32(const GemmArgs& p, int row, int outcol, const float (&g)[32], const float (&u)[32]) {
  uint32_t pk[16];
#pragma unroll
  for (int i = 0; i < 16; ++i) pk[i] = pack_bf16(silu(g[2 * i]) * u[2 * i], silu(g[2 * i + 1]) * u[2 * i + 1]);
  uint4* dst = reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.C) + size_t(row) * p.ldc + outcol);
#pragma unroll
  for (int i = 0; i < 4; ++i) dst[i] = make_uint4(pk[4 * i], pk[4 * i + 1], pk[4 * i + 2], pk[4 * i + 3]);
}

// Fused a4+a5+a6 epilogue: for every head of the tile, RoPE (rotate-half, pairs i / i+hd/2)
// on q and k, q written to C (the qkv buffer, read by the attention kernels), k and v written
// straight into the paged cache at the row's slot with 32-byte stores.  `fetch(col, v16)`
// returns 16 accumulator columns of this thread's row (TMEM or summed split-K partials).
template <int BN, typename Fetch>
QOS_DEV void epi_qkv_rope(const GemmArgs& p, int row, bool row_ok, int n_t, Fetch fetch, int h0 = 0, int hstep = 1) {
  const int hd = p.hd, half = hd / 2;
  const int ps = row_ok ? __ldg(p.pos + row) : 0;
  const int sl = row_ok ? __ldg(p.slot + row) : 0;
  const float2* cs = p.rope + size_t(ps) * half;
  for (int hh = h0; hh < BN / hd; hh += hstep) {
    const int col0 = n_t * BN + hh * hd;
    if (col0 >= p.N) break;  // warp-uniform
    const int head = col0 / hd;
    __nv_bfloat16* dst;
    if (head < p.H)
      dst = reinterpret_cast<__nv_bfloat16*>(p.C) + size_t(row) * p.ldc + col0;
    else if (head < p.H + p.Hkv)
      dst = p.kplane + ((size_t(sl >> 4) * p.Hkv + (head - p.H)) * 16 + (sl & 15)) * hd;
    else
      dst = p.vplane + ((size_t(sl >> 4) * p.Hkv + (head - p.H - p.Hkv)) * 16 + (sl & 15)) * hd;
    if (head < p.H + p.Hkv) {
      for (int i0 = 0; i0 < half; i0 += 16) {
        float x[16], y[16];
        fetch(hh * hd + i0, x);
        fetch(hh * hd + half + i0, y);
        if (row_ok) {
          uint32_t a[8], b[8];
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const float2 c0 = __ldg(cs + i0 + 2 * k), c1 = __ldg(cs + i0 + 2 * k + 1);
            a[k] = pack_bf16(x[2 * k] * c0.x - y[2 * k] * c0.y, x[2 * k + 1] * c1.x - y[2 * k + 1] * c1.y);
            b[k] = pack_bf16(y[2 * k] * c0.x + x[2 * k] * c0.y, y[2 * k + 1] * c1.x + x[2 * k + 1] * c1.y);
          }
          uint4* da = reinterpret_cast<uint4*>(dst + i0);
          uint4* db = reinterpret_cast<uint4*>(dst + half + i0);
          da[0] = make_uint4(a[0], a[1], a[2], a[3]);
          da[1] = make_uint4(a[4], a[5], a[6], a[7]);
          db[0] = make_uint4(b[0], b[1], b[2], b[3]);
          db[1] = make_uint4(b[4], b[5], b[6], b[7]);
        }
      }
    } else {
      for (int i0 = 0; i0 < hd; i0 += 16) {
        float x[16];
        fetch(hh * hd + i0, x);
        if (row_ok) {
          uint32_t a[8];  // V is cached in fp16 (it meets fp16 P in P.V)
#pragma unroll
          for (int k = 0; k < 8; ++k) a[k] = pack_f16(x[2 * k], x[2 * k + 1]);
          uint4* da = reinterpret_cast<uint4*>(dst + i0);
          da[0] = make_uint4(a[0], a[1], a[2], a[3]);
          da[1] = make_uint4(a[4], a[5], a[6], a[7]);
        }
      }
    }
  }
}

// ---- staged epilogue: a warp's 32 rows (thread = row, as tcgen05.ld 32x32b delivers them)
// are written to a smem tile of RB bytes per row and leave as coalesced 16-byte chunks
// (RB/16 threads per row segment).  16-byte chunk k of row r sits at chunk k ^ sw(r) so both
// the row-per-thread writes and the chunk-per-thread reads are bank-conflict free.
template <int RB>
QOS_DEV uint32_t stg_off(int r, int k) {
  return uint32_t(r * RB + 16 * (k ^ (RB >= 128 ? (r & 7) : ((r >> 1) & 3))));
}
template <int RB>
QOS_DEV void stg_put(uint8_t* stg, int r, int k, uint4 v) {
  *reinterpret_cast<uint4*>(stg + stg_off<RB>(r, k)) = v;
}
// dst(rr, k, v): store chunk k (16 B) of row rr
template <int RB, typename Dst>
QOS_DEV void stg_flush(const uint8_t* stg, int lane, Dst dst) {
  constexpr int kPer = RB / 16;  // threads per row segment
  __syncwarp();
#pragma unroll
  for (int pass = 0; pass < RB * 32 / 512; ++pass) {
    const int idx = pass * 32 + lane;
    const int rr = idx / kPer, k = idx % kPer;
    dst(rr, k, *reinterpret_cast<const uint4*>(stg + stg_off<RB>(rr, k)));
  }
  __syncwarp();
}
QOS_DEV void red_add_v4(float* addr, uint4 v) {  // fire-and-forget fp32 add at L2
  asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(addr), "f"(__uint_as_float(v.x)),
               "f"(__uint_as_float(v.y)), "f"(__uint_as_float(v.z)), "f"(__uint_as_float(v.w))
               : "memory");
}

// The fused a4+a5+a6 epilogue, staged: per head of the tile, RoPE'd q (or k) and v rows are
// built in smem, then written as coalesced row segments to the qkv buffer (q) or to the paged
// cache at each row's slot (k, v).  row0 = first row of this warp; `sl` = this thread's slot.
template <int BN, typename Fetch>
QOS_DEV void epi_qkv_rope_staged(const GemmArgs& p, uint8_t* stg, int lane, int row0, int n_t, Fetch fetch) {
  const int hd = p.hd, half = hd / 2;
  const int row = row0 + lane;
  const bool row_ok = row < p.M;
  const int ps = row_ok ? __ldg(p.pos + row) : 0;
  const int sl = row_ok ? __ldg(p.slot + row) : 0;
  for (int hh = 0; hh < BN / hd; ++hh) {
    const int col0 = n_t * BN + hh * hd;
    if (col0 >= p.N) break;  // warp-uniform
    const int head = col0 / hd;
    const int kind = head < p.H ? 0 : head < p.H + p.Hkv ? 1 : 2;
    const int kvh = kind == 1 ? head - p.H : head - p.H - p.Hkv;
    auto put = [&](int k, const uint32_t (&a)[8]) {  // 16 bf16/f16 values = chunks k, k+1
      if (hd == 128) {
        stg_put<256>(stg, lane, k, make_uint4(a[0], a[1], a[2], a[3]));
        stg_put<256>(stg, lane, k + 1, make_uint4(a[4], a[5], a[6], a[7]));
      } else {
        stg_put<128>(stg, lane, k, make_uint4(a[0], a[1], a[2], a[3]));
        stg_put<128>(stg, lane, k + 1, make_uint4(a[4], a[5], a[6], a[7]));
      }
    };
    if (kind < 2) {
      // RoPE with coalesced cos/sin reads: the 16 (x, y) pairs of chunk i0 are staged in fp32
      // (x in chunks 0-3, y in 4-7 of a 128-B row), then each lane rotates 2 pairs of one row
      // (8 lanes per row read its 128 B of the table) and stores 2 x 4 B of q (or k).
      for (int i0 = 0; i0 < half; i0 += 16) {
        // this lane's cos/sin for its 8 (row, pair couple) slots, requested before the TMEM
        // loads so their latency overlaps the staging
        float4 c[8];
        int slr[8];
#pragma unroll
        for (int pass = 0; pass < 8; ++pass) {
          const int rr = pass * 4 + (lane >> 3), k = lane & 7;
          const int prr = __shfl_sync(0xffffffffu, ps, rr);
          slr[pass] = __shfl_sync(0xffffffffu, sl, rr);
          c[pass] = __ldg(reinterpret_cast<const float4*>(p.rope + size_t(prr) * half + i0 + 2 * k));
        }
        float x[16], y[16];
        fetch(hh * hd + i0, x);
        fetch(hh * hd + half + i0, y);
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          stg_put<128>(stg, lane, k, make_uint4(__float_as_uint(x[4 * k]), __float_as_uint(x[4 * k + 1]),
                                                __float_as_uint(x[4 * k + 2]), __float_as_uint(x[4 * k + 3])));
          stg_put<128>(stg, lane, 4 + k, make_uint4(__float_as_uint(y[4 * k]), __float_as_uint(y[4 * k + 1]),
                                                    __float_as_uint(y[4 * k + 2]), __float_as_uint(y[4 * k + 3])));
        }
        __syncwarp();
#pragma unroll
        for (int pass = 0; pass < 8; ++pass) {
          const int rr = pass * 4 + (lane >> 3), k = lane & 7;  // row, pair couple (2k, 2k+1)
          const float2 xv = *reinterpret_cast<const float2*>(stg + stg_off<128>(rr, k >> 1) + (k & 1) * 8);
          const float2 yv = *reinterpret_cast<const float2*>(stg + stg_off<128>(rr, 4 + (k >> 1)) + (k & 1) * 8);
          const float4 cc = c[pass];
          const uint32_t lo = pack_bf16(xv.x * cc.x - yv.x * cc.y, xv.y * cc.z - yv.y * cc.w);
          const uint32_t hi = pack_bf16(yv.x * cc.x + xv.x * cc.y, yv.y * cc.z + xv.y * cc.w);
          const int r = row0 + rr;
          if (r < p.M) {
            __nv_bfloat16* d = kind == 0 ? reinterpret_cast<__nv_bfloat16*>(p.C) + size_t(r) * p.ldc + col0
                                         : p.kplane + ((size_t(slr[pass] >> 4) * p.Hkv + kvh) * 16 + (slr[pass] & 15)) * hd;
            *reinterpret_cast<uint32_t*>(d + i0 + 2 * k) = lo;
            *reinterpret_cast<uint32_t*>(d + half + i0 + 2 * k) = hi;
          }
        }
        __syncwarp();
      }
      continue;
    }
    // v head: fp16 rows staged whole, then coalesced row segments into the paged cache
    for (int i0 = 0; i0 < hd; i0 += 16) {
      float x[16];
      fetch(hh * hd + i0, x);
      uint32_t a[8];  // V is cached in fp16 (it meets fp16 P in P.V)
#pragma unroll
      for (int k = 0; k < 8; ++k) a[k] = pack_f16(x[2 * k], x[2 * k + 1]);
      put(i0 / 8, a);
    }
    auto dst = [&](int rr, int k, uint4 v) {
      const int slr = __shfl_sync(0xffffffffu, sl, rr);
      if (row0 + rr >= p.M) return;
      reinterpret_cast<uint4*>(p.vplane + ((size_t(slr >> 4) * p.Hkv + kvh) * 16 + (slr & 15)) * hd)[k] = v;
    };
    if (hd == 128) stg_flush<256>(stg, lane, dst);
    else stg_flush<128>(stg, lane, dst);
  }
}

// Epilogue of one row of a tile from summed fp32 partials, in independent column units
// u0, u0 + ustep, ... (32 columns; SiLU: 32 outputs = 32 gate + 32 up columns; QKV: one head),
// so several CTAs can share the reduction of one tile.  fetch32(col, v) / fetch16(col, v)
// return accumulator columns col.. of this thread's row.
template <int BN, int EPI, typename F32, typename F16>
QOS_DEV void epi_units(const GemmArgs& p, int row, bool row_ok, int n_t, int u0, int ustep, F32 fetch32, F16 fetch16) {
  if constexpr (EPI == EPI_QKV_ROPE) {
    epi_qkv_rope<BN>(p, row, row_ok, n_t, fetch16, u0, ustep);
  } else if constexpr (EPI == EPI_SILU_GATE) {
    for (int u = u0; u < BN / 64; u += ustep) {
      const int g = u >> 1, h = u & 1;
      float gv[32], uv[32];
      fetch32(g * 128 + h * 32, gv);
      fetch32(g * 128 + 64 + h * 32, uv);
      const int col = n_t * (BN / 2) + g * 64 + h * 32;
      if (row_ok && col < p.N / 2) epi_silu32(p, row, col, gv, uv);
    }
  } else {
    for (int u = u0; u < BN / 32; u += ustep) {
      float v[32];
      fetch32(u * 32, v);
      const int col = n_t * BN + u * 32;
      if (row_ok && col < p.N) epi_store32<EPI>(p, row, col, v);
    }
  }
}
template <int BN, int EPI>
QOS_DEV int epi_num_units(const GemmArgs& p) {
  return EPI == EPI_QKV_ROPE ? BN / p.hd : EPI == EPI_SILU_GATE ? BN / 64 : BN / 32;
}

QOS_DEV void tmem_ld32(uint32_t taddr, float (&v)[32]) {
  uint32_t r[32];
  tmem_ld32x32b_x16(taddr, *reinterpret_cast<uint32_t(*)[16]>(&r[0]));
  tmem_ld32x32b_x16(taddr + 16, *reinterpret_cast<uint32_t(*)[16]>(&r[16]));
  tmem_ld_wait();
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}

QOS_DEV void epi_bar_sync() { asm volatile("bar.sync 1, 128;" ::: "memory"); }  // the 4 epilogue warps

// Whole tile straight from TMEM, staged through smem (coalesced stores).  Thread = one
// accumulator row (`row`, the warp's rows start at row - lane); tbase = this warp's TMEM lane
// quarter + the accumulator's first column; n_t = the tile's BN-wide column block.
template <int BN, int EPI>
QOS_DEV void epi_tile_staged(const GemmArgs& p, uint8_t* stg, int lane, int n_t, int row, uint32_t tbase) {
        const int row0 = row - lane;
        // folded RMSNorm, consumer side: this row's 1/rms from the producer's per-block sums
        float rs = 1.f;
        if constexpr (EPI == EPI_QKV_ROPE || EPI == EPI_SILU_GATE) {
          if (p.rs_in != nullptr && row < p.M) rs = __ldcg(p.rs_in + row);
        }
        if constexpr (EPI == EPI_QKV_ROPE) {
          epi_qkv_rope_staged<BN>(p, stg, lane, row0, n_t, [&](int col, float (&v)[16]) {
            uint32_t r[16];
            tmem_ld32x32b_x16(tbase + col, r);
            tmem_ld_wait();
#pragma unroll
            for (int i = 0; i < 16; ++i)
              v[i] = __uint_as_float(r[i]) * rs + (p.bias ? __ldg(p.bias + n_t * BN + col + i) : 0.f);
          });
        } else if constexpr (EPI == EPI_SILU_GATE) {
#pragma unroll 1
          for (int g = 0; g < BN / 128; ++g) {
#pragma unroll 1
            for (int h = 0; h < 2; ++h) {
              float gv[32], uv[32];
              tmem_ld32(tbase + g * 128 + h * 32, gv);
              tmem_ld32(tbase + g * 128 + 64 + h * 32, uv);
              const int col = n_t * (BN / 2) + g * 64 + h * 32;
              if (col >= p.N / 2) continue;  // warp-uniform
#pragma unroll
              for (int i = 0; i < 32; ++i) {
                gv[i] *= rs;
                uv[i] *= rs;
              }
              uint32_t pk[16];
#pragma unroll
              for (int i = 0; i < 16; ++i) pk[i] = pack_bf16(silu(gv[2 * i]) * uv[2 * i], silu(gv[2 * i + 1]) * uv[2 * i + 1]);
#pragma unroll
              for (int k = 0; k < 4; ++k) stg_put<64>(stg, lane, k, make_uint4(pk[4 * k], pk[4 * k + 1], pk[4 * k + 2], pk[4 * k + 3]));
              stg_flush<64>(stg, lane, [&](int rr, int k, uint4 v) {
                if (row0 + rr < p.M)
                  reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.C) + size_t(row0 + rr) * p.ldc + col)[k] = v;
              });
            }
          }
        } else if (EPI == EPI_ADD_F32 && p.ss_out != nullptr) {
          // folded RMSNorm, producer side: r += tile (read-add-write), h = bf16(r * g_out), and
          // per 128-column block the row's sum of r^2.  Lane = (row rr = pass*4 + lane/8, 16-B
          // chunk k = lane%8) of the staged 32 x 32 fp32 block; the 8 lanes of a row reduce by
          // shuffles, per-block sums accumulate over the block's four 32-column chunks.  The
          // residual chunks of 32-column block c+1 are requested before block c is processed
          // (two register sets), so the read-add-write costs about one L2 latency per tile.
          const int k8 = lane & 7;
          auto load_old = [&](int c, float4 (&o)[8]) {
            const int col = n_t * BN + c * 32;
#pragma unroll
            for (int pass = 0; pass < 8; ++pass) {
              const int r = row0 + pass * 4 + (lane >> 3);
              o[pass] = (r < p.M && col < p.N)
                            ? __ldcg(reinterpret_cast<const float4*>(reinterpret_cast<const float*>(p.C) + size_t(r) * p.ldc +
                                                                     col + 4 * k8))
                            : make_float4(0.f, 0.f, 0.f, 0.f);
            }
          };
          float acc8[8];
#pragma unroll
          for (int i = 0; i < 8; ++i) acc8[i] = 0.f;
          auto process = [&](int c, const float4 (&old)[8]) {
            float v[32];
            tmem_ld32(tbase + c * 32, v);
            const int col = n_t * BN + c * 32;
            if (col >= p.N) return;  // warp-uniform (whole 128-column blocks: N % 128 == 0)
#pragma unroll
            for (int k = 0; k < 8; ++k)
              stg_put<128>(stg, lane, k, make_uint4(__float_as_uint(v[4 * k]), __float_as_uint(v[4 * k + 1]),
                                                    __float_as_uint(v[4 * k + 2]), __float_as_uint(v[4 * k + 3])));
            __syncwarp();
            const uint2 gg = __ldg(reinterpret_cast<const uint2*>(p.g_out + col + 4 * k8));
#pragma unroll
            for (int pass = 0; pass < 8; ++pass) {
              const int rr = pass * 4 + (lane >> 3);
              const int r = row0 + rr;
              float sq = 0.f;
              if (r < p.M) {
                const uint4 x = *reinterpret_cast<const uint4*>(stg + stg_off<128>(rr, k8));
                float4 o = old[pass];
                o.x += __uint_as_float(x.x);
                o.y += __uint_as_float(x.y);
                o.z += __uint_as_float(x.z);
                o.w += __uint_as_float(x.w);
                *reinterpret_cast<float4*>(reinterpret_cast<float*>(p.C) + size_t(r) * p.ldc + col + 4 * k8) = o;
                *reinterpret_cast<uint2*>(p.h_out + size_t(r) * p.N + col + 4 * k8) =
                    make_uint2(pack_bf16(o.x * bf16_lo(gg.x), o.y * bf16_hi(gg.x)),
                               pack_bf16(o.z * bf16_lo(gg.y), o.w * bf16_hi(gg.y)));
                sq = (o.x * o.x + o.y * o.y) + (o.z * o.z + o.w * o.w);
              }
              sq += __shfl_xor_sync(0xffffffffu, sq, 1);
              sq += __shfl_xor_sync(0xffffffffu, sq, 2);
              sq += __shfl_xor_sync(0xffffffffu, sq, 4);
              acc8[pass] += sq;
            }
            __syncwarp();
            if ((c & 3) == 3) {  // end of a 128-column block: one partial per row
              if (k8 == 0) {
#pragma unroll
                for (int pass = 0; pass < 8; ++pass) {
                  const int r = row0 + pass * 4 + (lane >> 3);
                  if (r < p.M) p.ss_out[size_t(r) * kFoldSlots + col / 128] = acc8[pass];
                }
              }
#pragma unroll
              for (int i = 0; i < 8; ++i) acc8[i] = 0.f;
            }
          };
          float4 oa[8], ob[8];
          load_old(0, oa);
#pragma unroll 1
          for (int c = 0; c < BN / 32; c += 2) {  // BN / 32 is even
            load_old(c + 1, ob);
            process(c, oa);
            if (c + 2 < BN / 32) load_old(c + 2, oa);
            process(c + 1, ob);
          }
          // the last tile of this 128-row block to finish turns the per-block sums into 1/rms
          // (the barrier orders the 4 warps' stores before thread 0's fence + arrival — one fence
          //  per tile, as in a grid barrier, instead of a full fence in every thread)
          __shared__ int s_fold_last;
          epi_bar_sync();
          const int rb = row >> 7;
          if ((row & 127) == 0) {
            __threadfence();
            s_fold_last = atomicAdd(p.fcnt + rb, 1) == p.nt - 1;
          }
          epi_bar_sync();
          if (s_fold_last) {
            __threadfence();
            if (row < p.M) {
              const float4* sp = reinterpret_cast<const float4*>(p.ss_out + size_t(row) * kFoldSlots);
              float4 x[kFoldSlots / 4];
#pragma unroll
              for (int j = 0; j < kFoldSlots / 4; ++j) x[j] = __ldcg(sp + j);
              float t = 0.f;
#pragma unroll
              for (int j = 0; j < kFoldSlots / 4; ++j) t += (x[j].x + x[j].y) + (x[j].z + x[j].w);
              p.rs_out[row] = rsqrtf(t * p.inv_d + p.rms_eps);
            }
            if ((row & 127) == 0) p.fcnt[rb] = 0;  // ready for the next launch
          }
        } else {
#pragma unroll 1
          for (int c = 0; c < BN / 32; ++c) {
            float v[32];
            tmem_ld32(tbase + c * 32, v);
            const int col = n_t * BN + c * 32;
            if (col >= p.N) continue;  // warp-uniform (N % 32 == 0)
            if constexpr (EPI == EPI_STORE_BF16 || EPI == EPI_BIAS_BF16) {
              uint32_t pk[16];
#pragma unroll
              for (int i = 0; i < 16; ++i) {
                float a0 = v[2 * i], a1 = v[2 * i + 1];
                if constexpr (EPI == EPI_BIAS_BF16) {
                  a0 += __ldg(p.bias + col + 2 * i);
                  a1 += __ldg(p.bias + col + 2 * i + 1);
                }
                pk[i] = pack_bf16(a0, a1);
              }
#pragma unroll
              for (int k = 0; k < 4; ++k) stg_put<64>(stg, lane, k, make_uint4(pk[4 * k], pk[4 * k + 1], pk[4 * k + 2], pk[4 * k + 3]));
              stg_flush<64>(stg, lane, [&](int rr, int k, uint4 x) {
                const int r = row0 + rr;
                if (r >= p.M) return;
                if (p.scat_rs) {  // TP reduce-scatter: the row's owner rank, over peer memory
                  const int own = r / p.scat_rs;
                  reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.scat[own]) +
                                           size_t(r - own * p.scat_rs) * p.ldc + col)[k] = x;
                } else {
                  reinterpret_cast<uint4*>(reinterpret_cast<__nv_bfloat16*>(p.C) + size_t(r) * p.ldc + col)[k] = x;
                }
              });
            } else {
#pragma unroll
              for (int k = 0; k < 8; ++k)
                stg_put<128>(stg, lane, k, make_uint4(__float_as_uint(v[4 * k]), __float_as_uint(v[4 * k + 1]),
                                                      __float_as_uint(v[4 * k + 2]), __float_as_uint(v[4 * k + 3])));
              stg_flush<128>(stg, lane, [&](int rr, int k, uint4 x) {
                if (row0 + rr >= p.M) return;
                float* d = reinterpret_cast<float*>(p.C) + size_t(row0 + rr) * p.ldc + col + 4 * k;
                if constexpr (EPI == EPI_ADD_F32) red_add_v4(d, x);  // residual += tile (one add per element)
                else *reinterpret_cast<uint4*>(d) = x;
              });
            }
          }
        }
}

template <int BN, int EPI>
__global__ void __launch_bounds__(kGemmThreads, 1)
    gemm_tcgen05_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                        const GemmArgs p) {
  using Cfg = GemmCfg<BN>;
  constexpr int S = Cfg::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * Cfg::kStageBytes);
  uint64_t* empty = full + S;
  uint64_t* tfull = empty + S;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  int* s_last = reinterpret_cast<int*>(tmem_slot + 1);
  uint8_t* stg_all = smem + S * Cfg::kStageBytes + 256;  // 4 x kStageWarpBytes

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], 4);
    }
    fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
  }
  if (warp == 1) tmem_alloc<Cfg::kTmemCols>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  griddep_launch_dependents();  // the next kernel may start its prologue as SMs free up
  if (warp != 0) griddep_wait();  // epilogue reads/writes C (residual, KV cache) of earlier kernels

  // work unit u = ((n_t * ksplit) + split) * mt + m_t: consecutive units share a weight slice
  const int ks = p.ksplit;
  const int num_units = p.mt * p.nt * ks;
  const int kblocks = p.K / kBK;
  auto decode_unit = [&](int u, int& m_t, int& n_t, int& sp, int& kb0, int& kb1) {
    if (p.ordered) {  // u = sp * tiles + n_t * mt + m_t
      const int tiles = p.mt * p.nt;
      sp = u / tiles;
      const int t = u - sp * tiles;
      m_t = t % p.mt;
      n_t = t / p.mt;
    } else {
      m_t = u % p.mt;
      const int r = u / p.mt;
      sp = r % ks;
      n_t = r / ks;
    }
    kb0 = sp * kblocks / ks;
    kb1 = (sp + 1) * kblocks / ks;
  };
  // stream-K ranges: CTA c owns linear iterations [rstart(c), rstart(c+1)) of t * kblocks + kb
  const int64_t skW = p.work, skG = gridDim.x;
  auto rstart = [&](int64_t c) { return c * skW / skG; };
  auto cta_of = [&](int64_t idx) { return int(((idx + 1) * skG - 1) / skW); };
  const int64_t s0 = p.sk ? rstart(blockIdx.x) : 0, e0 = p.sk ? rstart(blockIdx.x + 1) : 0;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (elect_one()) {
      const uint64_t pol_a = l2_evict_last();   // activations: re-read by every N tile
      const uint64_t pol_b = l2_evict_first();  // weights: streamed once per M-tile group
      if (p.sk) {
        const int n = int(e0 - s0);
        const int npre = min(S, n);
        for (int i = 0; i < npre; ++i) {  // PDL: weights before the wait
          const int64_t idx = s0 + i;
          const int t = int(idx / kblocks), kb = int(idx - int64_t(t) * kblocks);
          mbar_arrive_expect_tx(&full[i], Cfg::kStageBytes);
          tma_load_2d_hint(smem + i * Cfg::kStageBytes + Cfg::kABytes, &tmB, &full[i], kb * kBK, (t / p.mt) * BN, pol_b);
        }
        griddep_wait();
        for (int i = 0; i < npre; ++i) {
          const int64_t idx = s0 + i;
          const int t = int(idx / kblocks), kb = int(idx - int64_t(t) * kblocks);
          tma_load_2d_hint(smem + i * Cfg::kStageBytes, &tmA, &full[i], kb * kBK, p.a_row0 + (t % p.mt) * kBM, pol_a);
        }
        int stage = npre % S;
        uint32_t phase = (npre == S) ? 1u : 0u;
        for (int i = npre; i < n; ++i) {
          const int64_t idx = s0 + i;
          const int t = int(idx / kblocks), kb = int(idx - int64_t(t) * kblocks);
          mbar_wait(&empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * Cfg::kStageBytes;
          mbar_arrive_expect_tx(&full[stage], Cfg::kStageBytes);
          tma_load_2d_hint(sa, &tmA, &full[stage], kb * kBK, p.a_row0 + (t % p.mt) * kBM, pol_a);
          tma_load_2d_hint(sa + Cfg::kABytes, &tmB, &full[stage], kb * kBK, (t / p.mt) * BN, pol_b);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
      } else {
      int stage = 0;
      uint32_t phase = 0;
      // Programmatic dependent launch: the weight (B) tiles of the first stages do not depend on
      // the previous kernel, so they are requested before griddepcontrol.wait; the activation (A)
      // tiles, produced by the previous kernel, only after it.
      int npre = 0;
      if (blockIdx.x < num_units) {
        int m_t, n_t, sp, kb0, kb1;
        decode_unit(blockIdx.x, m_t, n_t, sp, kb0, kb1);
        npre = min(S, kb1 - kb0);
        for (int i = 0; i < npre; ++i) {
          uint8_t* sa = smem + i * Cfg::kStageBytes;
          mbar_arrive_expect_tx(&full[i], Cfg::kStageBytes);
          tma_load_2d_hint(sa + Cfg::kABytes, &tmB, &full[i], (kb0 + i) * kBK, n_t * BN, pol_b);
        }
        griddep_wait();
        for (int i = 0; i < npre; ++i)
          tma_load_2d_hint(smem + i * Cfg::kStageBytes, &tmA, &full[i], (kb0 + i) * kBK, p.a_row0 + m_t * kBM, pol_a);
      } else {
        griddep_wait();
      }
      int it = 0;
      for (int u = blockIdx.x; u < num_units; u += gridDim.x) {
        int m_t, n_t, sp, kb0, kb1;
        decode_unit(u, m_t, n_t, sp, kb0, kb1);
        for (int kb = kb0; kb < kb1; ++kb, ++it) {
          if (it < npre) {  // issued above
            if (++stage == S) { stage = 0; phase ^= 1; }
            continue;
          }
          mbar_wait(&empty[stage], phase ^ 1);
          uint8_t* sa = smem + stage * Cfg::kStageBytes;
          mbar_arrive_expect_tx(&full[stage], Cfg::kStageBytes);
          tma_load_2d_hint(sa, &tmA, &full[stage], kb * kBK, p.a_row0 + m_t * kBM, pol_a);
          tma_load_2d_hint(sa + Cfg::kABytes, &tmB, &full[stage], kb * kBK, n_t * BN, pol_b);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
      }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer
    if (elect_one()) {
      constexpr uint32_t idesc = umma_idesc_bf16(kBM, BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      int u = blockIdx.x;
      int64_t idx = s0;
      for (;;) {
        int kb0, kb1;
        if (p.sk) {  // next stream-K segment
          if (idx >= e0) break;
          const int t = int(idx / kblocks);
          kb0 = int(idx - int64_t(t) * kblocks);
          kb1 = int(min(int64_t(kblocks), int64_t(kb0) + (e0 - idx)));
          idx += kb1 - kb0;
        } else {
          if (u >= num_units) break;
          int m_t, n_t, sp;
          decode_unit(u, m_t, n_t, sp, kb0, kb1);
          u += gridDim.x;
        }
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t a_base = smem_u32(smem + stage * Cfg::kStageBytes);
          const uint32_t b_base = a_base + Cfg::kABytes;
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k) {
            umma_bf16(d_tmem, umma_desc_sw128(a_base + k * 32), umma_desc_sw128(b_base + k * 32), idesc,
                      (kb > kb0 || k > 0) ? 1u : 0u);
          }
          umma_commit(&empty[stage]);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
        umma_commit(&tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (warps 2..5)
    const int q = warp & 3;  // TMEM lane quarter this warp may access
    const int rit = q * 32 + lane;  // row inside the tile
    int acc = 0;
    uint32_t acc_phase = 0;
    uint8_t* stg = stg_all + q * Cfg::kStageWarpBytes;
    // whole tile straight from TMEM, staged through smem (coalesced stores); row = this thread's
    // row, row0 = the warp's first row
    auto epi_tmem = [&](int n_t, int row, bool row_ok, uint32_t tbase) {
      (void)row_ok;
      epi_tile_staged<BN, EPI>(p, stg, lane, n_t, row, tbase);
    };
    if (p.sk) {
      // stream-K: whole tiles straight from TMEM; a tile cut by a range boundary parks one fp32
      // partial per CTA (slot 2c for a CTA's first segment, 2c+1 for its last)
      const int bid = blockIdx.x;
      int pend[2], npend = 0;
      auto slot_of = [&](int t, int cc) { return rstart(cc) >= int64_t(t) * kblocks ? 2 * cc : 2 * cc + 1; };
      auto red32 = [&](int t, int cf, int cl) {
        const bool ok = (t % p.mt) * kBM + rit < p.M;  // partials of rows past M were never written
        return [=](int col, float (&v)[32]) {
#pragma unroll
          for (int i = 0; i < 32; ++i) v[i] = 0.f;
          for (int cc = cf; ok && cc <= cl; ++cc) {  // CTA order: deterministic
            const float4* pr = reinterpret_cast<const float4*>(p.part + (size_t(slot_of(t, cc)) * kBM + rit) * BN + col);
            float4 x[8];
#pragma unroll
            for (int i = 0; i < 8; ++i) x[i] = __ldcg(pr + i);
#pragma unroll
            for (int i = 0; i < 8; ++i) {
              v[4 * i] += x[i].x;
              v[4 * i + 1] += x[i].y;
              v[4 * i + 2] += x[i].z;
              v[4 * i + 3] += x[i].w;
            }
          }
        };
      };
      auto red16 = [&](int t, int cf, int cl, int n_t) {
        const bool ok = (t % p.mt) * kBM + rit < p.M;
        return [=](int col, float (&v)[16]) {
#pragma unroll
          for (int i = 0; i < 16; ++i) v[i] = p.bias ? __ldg(p.bias + n_t * BN + col + i) : 0.f;
          for (int cc = cf; ok && cc <= cl; ++cc) {
            const float4* pr = reinterpret_cast<const float4*>(p.part + (size_t(slot_of(t, cc)) * kBM + rit) * BN + col);
            float4 x[4];
#pragma unroll
            for (int i = 0; i < 4; ++i) x[i] = __ldcg(pr + i);
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              v[4 * i] += x[i].x;
              v[4 * i + 1] += x[i].y;
              v[4 * i + 2] += x[i].z;
              v[4 * i + 3] += x[i].w;
            }
          }
        };
      };
      for (int64_t idx = s0; idx < e0;) {
        const int t = int(idx / kblocks), kb0 = int(idx - int64_t(t) * kblocks);
        const int kb1 = int(min(int64_t(kblocks), int64_t(kb0) + (e0 - idx)));
        const int m_t = t % p.mt, n_t = t / p.mt;
        mbar_wait(&tfull[acc], acc_phase);
        tc_fence_after();
        const int row = m_t * kBM + rit;
        const bool row_ok = row < p.M;
        const uint32_t tbase = tmem_base + (uint32_t(q * 32) << 16) + acc * BN;
        if (kb0 == 0 && kb1 == kblocks) {
          epi_tmem(n_t, row, row_ok, tbase);
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&tempty[acc]);
        } else {
          float* mine = p.part + (size_t(idx == s0 ? 2 * bid : 2 * bid + 1) * kBM + rit) * BN;
#pragma unroll 1
          for (int c = 0; c < BN / 32; ++c) {
            float v[32];
            tmem_ld32(tbase + c * 32, v);
            if (row_ok) {
#pragma unroll
              for (int i = 0; i < 8; ++i)
                __stcg(reinterpret_cast<float4*>(mine + c * 32) + i,
                       make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]));
            }
          }
          tc_fence_before();
          __syncwarp();
          if (lane == 0) mbar_arrive(&tempty[acc]);
          __threadfence();
          epi_bar_sync();
          const int cf = cta_of(int64_t(t) * kblocks), cl = cta_of(int64_t(t + 1) * kblocks - 1);
          if (p.coop) {
            if (threadIdx.x == 64) atomicAdd(p.counters + t, 1);
            pend[npend++] = t;
          } else {
            if (threadIdx.x == 64) *s_last = (atomicAdd(p.counters + t, 1) == cl - cf);
            epi_bar_sync();
            if (*s_last) {
              __threadfence();
              epi_units<BN, EPI>(p, row, row_ok, n_t, 0, 1, red32(t, cf, cl), red16(t, cf, cl, n_t));
              if (threadIdx.x == 64) p.counters[t] = 0;
            }
          }
        }
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        idx += kb1 - kb0;
      }
      // cooperative reduction of the cut tiles (all CTAs are co-resident: one per SM)
      for (int i = 0; i < npend; ++i) {
        const int t = pend[i];
        const int m_t = t % p.mt, n_t = t / p.mt;
        const int row = m_t * kBM + rit;
        const bool row_ok = row < p.M;
        const int cf = cta_of(int64_t(t) * kblocks), cl = cta_of(int64_t(t + 1) * kblocks - 1);
        const int n = cl - cf + 1;
        if (threadIdx.x == 64) {
          int v;
          do {
            asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p.counters + t) : "memory");
          } while (v < n);
        }
        epi_bar_sync();
        epi_units<BN, EPI>(p, row, row_ok, n_t, bid - cf, n, red32(t, cf, cl), red16(t, cf, cl, n_t));
        epi_bar_sync();
        if (threadIdx.x == 64 && atomicAdd(p.counters + t, 1) == 2 * n - 1) p.counters[t] = 0;
      }
    } else
    for (int u = blockIdx.x; u < num_units; u += gridDim.x) {
      int m_t, n_t, sp, kb0, kb1;
      decode_unit(u, m_t, n_t, sp, kb0, kb1);
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row = m_t * kBM + rit;
      const bool row_ok = row < p.M;
      const uint32_t tbase = tmem_base + (uint32_t(q * 32) << 16) + acc * BN;
      if (ks == 1) {
        epi_tmem(n_t, row, row_ok, tbase);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
      } else if (p.ordered) {
        // ordered split-K (EPI_ADD_F32): slice sp adds its partial after slices 0..sp-1 (their
        // red.adds are visible once counters[tile] == sp), so C sees a fixed summation order
        const int tile = n_t * p.mt + m_t;
        if (sp > 0) {
          if (threadIdx.x == 64) {
            int v;
            do {
              asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p.counters + tile) : "memory");
            } while (v != sp);
          }
          epi_bar_sync();
        }
        epi_tmem(n_t, row, row_ok, tbase);
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
        if (sp + 1 < ks) {
          __threadfence();
          epi_bar_sync();
          if (threadIdx.x == 64) asm volatile("st.release.gpu.global.b32 [%0], %1;" ::"l"(p.counters + tile), "r"(sp + 1) : "memory");
        } else if (threadIdx.x == 64) {
          p.counters[tile] = 0;  // ready for the next launch (no slice waits after the last)
        }
      } else {
        // split-K: park the fp32 partial, release TMEM, the last slice of the tile reduces
        float* mine = p.part + (size_t(u) * kBM + rit) * BN;
#pragma unroll 1
        for (int c = 0; c < BN / 32; ++c) {
          float v[32];
          tmem_ld32(tbase + c * 32, v);
#pragma unroll
          for (int i = 0; i < 8; ++i)
            reinterpret_cast<float4*>(mine + c * 32)[i] = make_float4(v[4 * i], v[4 * i + 1], v[4 * i + 2], v[4 * i + 3]);
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
        __threadfence();
        epi_bar_sync();
        const int tile = n_t * p.mt + m_t;
        if (threadIdx.x == 64) *s_last = (atomicAdd(p.counters + tile, 1) == ks - 1);
        epi_bar_sync();
        if (*s_last) {
          __threadfence();
          auto part_row = [&](int s2) {
            return p.part + (size_t((n_t * ks + s2) * p.mt + m_t) * kBM + rit) * BN;
          };
          if constexpr (EPI == EPI_QKV_ROPE) {
            epi_qkv_rope<BN>(p, row, row_ok, n_t, [&](int col, float (&v)[16]) {
#pragma unroll
              for (int i = 0; i < 16; ++i) v[i] = p.bias ? __ldg(p.bias + n_t * BN + col + i) : 0.f;
              for (int s2 = 0; s2 < ks; ++s2) {
                const float* pr = part_row(s2) + col;
#pragma unroll
                for (int i = 0; i < 16; ++i) v[i] += __ldcg(pr + i);
              }
            });
          } else if constexpr (EPI == EPI_SILU_GATE) {
#pragma unroll 1
            for (int g = 0; g < BN / 128; ++g)
#pragma unroll 1
              for (int h = 0; h < 2; ++h) {
                float gv[32], uv[32];
#pragma unroll
                for (int i = 0; i < 32; ++i) gv[i] = uv[i] = 0.f;
                for (int s2 = 0; s2 < ks; ++s2) {
                  const float* pr = part_row(s2);
#pragma unroll
                  for (int i = 0; i < 32; ++i) {
                    gv[i] += __ldcg(pr + g * 128 + h * 32 + i);
                    uv[i] += __ldcg(pr + g * 128 + 64 + h * 32 + i);
                  }
                }
                const int col = n_t * (BN / 2) + g * 64 + h * 32;
                if (row_ok && col < p.N / 2) epi_silu32(p, row, col, gv, uv);
              }
          } else {
#pragma unroll 1
            for (int c = 0; c < BN / 32; ++c) {
              float v[32];
#pragma unroll
              for (int i = 0; i < 32; ++i) v[i] = 0.f;
              for (int s2 = 0; s2 < ks; ++s2) {
                const float4* pr = reinterpret_cast<const float4*>(part_row(s2) + c * 32);
#pragma unroll
                for (int i = 0; i < 8; ++i) {
                  const float4 x = __ldcg(pr + i);
                  v[4 * i] += x.x;
                  v[4 * i + 1] += x.y;
                  v[4 * i + 2] += x.z;
                  v[4 * i + 3] += x.w;
                }
              }
              const int col = n_t * BN + c * 32;
              if (row_ok && col < p.N) epi_store32<EPI>(p, row, col, v);
            }
          }
          if (threadIdx.x == 64) p.counters[tile] = 0;  // ready for the next launch
        }
      }
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
  }
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<Cfg::kTmemCols>(tmem_base);
  }
}


// ------------------------------------------------------------------------------ CTA-pair GEMM
// cta_group::2 variant for large token counts (the shapes cuBLAS also runs on CTA pairs):
// a cluster of 2 CTAs on 2 SMs computes a 256 x 256 tile with UMMA M=256 N=256 K=16 issued by
// CTA 0.  Each CTA stages its own 128 rows of A and its own 128 rows (output columns) of B per
// k-block (32 KB instead of 48 KB for a 128 x 256 single-CTA tile) and holds the fp32
// accumulator of its 128 rows x 256 columns in its own TMEM, so per SM the shared-memory
// traffic (TMA writes + MMA operand reads) per FLOP drops by a third.  The peer CTA's TMA
// loads complete on the leader's full barrier; the leader's MMA commits arrive on both CTAs'
// empty / accumulator-full barriers; both CTAs' epilogue warps release an accumulator on the
// leader's barrier.  No split-K / stream-K: used where 128 x 256 tiles already fill the SMs.
constexpr int kG2Stages = 6;
constexpr int kG2Half = 128 * kBK * 2;          // 16 KB: 128 rows x 64 k of A or of B
constexpr int kG2Stage = 2 * kG2Half;
constexpr int kG2StageWarpBytes = 32 * 256;
constexpr int kG2Smem = kG2Stages * kG2Stage + 1024 + 256 + 4 * kG2StageWarpBytes;

template <int EPI>
__global__ void __launch_bounds__(kGemmThreads, 1)
    gemm2_tcgen05_kernel(const __grid_constant__ CUtensorMap tmA, const __grid_constant__ CUtensorMap tmB,
                         const GemmArgs p) {
  constexpr int S = kG2Stages, BN = 256;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + S * kG2Stage);
  uint64_t* empty = full + S;
  uint64_t* tfull = empty + S;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  uint8_t* stg_all = smem + S * kG2Stage + 256;

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const uint32_t rank = cluster_ctarank();
  const bool leader = rank == 0;

  if (threadIdx.x == 0) {
    for (int s = 0; s < S; ++s) {
      mbar_init(&full[s], 1);
      mbar_init(&empty[s], 1);
    }
    for (int a = 0; a < 2; ++a) {
      mbar_init(&tfull[a], 1);
      mbar_init(&tempty[a], 8);  // leader's: 4 epilogue warps of each CTA
    }
    fence_mbar_init();
  }
  if (warp == 0 && lane == 0) {
    tma_prefetch_desc(&tmA);
    tma_prefetch_desc(&tmB);
  }
  cluster_sync();  // both CTAs of the pair resident before the pair-wide TMEM allocation
  if (warp == 1) tmem_alloc2<512>(tmem_slot);
  tc_fence_before();
  cluster_sync();  // barrier inits and the TMEM address visible pair-wide
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  griddep_launch_dependents();
  if (warp != 0) griddep_wait();

  const int pair = blockIdx.x >> 1, npairs = gridDim.x >> 1;
  const int mt2 = (p.M + 255) / 256;
  const int num_units = mt2 * p.nt;
  const int kblocks = p.K / kBK;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer (both CTAs)
    if (elect_one()) {
      const uint64_t pol_a = l2_evict_last();
      const uint64_t pol_b = l2_evict_first();
      const uint32_t full_leader = mapa_shared(smem_u32(full), 0);
      int stage = 0;
      uint32_t phase = 0;
      int npre = 0;
      if (pair < num_units) {  // PDL: weight halves of the first stages before the wait
        const int n_t = pair / mt2;
        npre = min(S, kblocks);
        for (int i = 0; i < npre; ++i) {
          if (leader) mbar_arrive_expect_tx(&full[i], 2 * kG2Stage);
          tma_load_2d_2cta(smem + i * kG2Stage + kG2Half, &tmB, full_leader + i * 8, i * kBK, n_t * BN + rank * 128, pol_b);
        }
        griddep_wait();
        const int m_t = pair % mt2;
        for (int i = 0; i < npre; ++i)
          tma_load_2d_2cta(smem + i * kG2Stage, &tmA, full_leader + i * 8, i * kBK, p.a_row0 + m_t * 256 + rank * 128, pol_a);
      } else {
        griddep_wait();
      }
      int it = 0;
      for (int u = pair; u < num_units; u += npairs) {
        const int m_t = u % mt2, n_t = u / mt2;
        for (int kb = 0; kb < kblocks; ++kb, ++it) {
          if (it < npre) {
            if (++stage == S) { stage = 0; phase ^= 1; }
            continue;
          }
          mbar_wait(&empty[stage], phase ^ 1);
          if (leader) mbar_arrive_expect_tx(&full[stage], 2 * kG2Stage);
          uint8_t* sa = smem + stage * kG2Stage;
          tma_load_2d_2cta(sa, &tmA, full_leader + stage * 8, kb * kBK, p.a_row0 + m_t * 256 + rank * 128, pol_a);
          tma_load_2d_2cta(sa + kG2Half, &tmB, full_leader + stage * 8, kb * kBK, n_t * BN + rank * 128, pol_b);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ MMA issuer (leader only)
    if (leader && elect_one()) {
      constexpr uint32_t idesc = umma_idesc_bf16(256, BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int u = pair; u < num_units; u += npairs) {
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BN;
        for (int kb = 0; kb < kblocks; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t a_base = smem_u32(smem + stage * kG2Stage);
          const uint32_t b_base = a_base + kG2Half;
#pragma unroll
          for (int k = 0; k < kBK / 16; ++k)
            umma_bf16_2cta(d_tmem, umma_desc_sw128(a_base + k * 32), umma_desc_sw128(b_base + k * 32), idesc,
                           (kb > 0 || k > 0) ? 1u : 0u);
          umma_commit_2cta(&empty[stage]);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
        umma_commit_2cta(&tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (both CTAs)
    const int q = warp & 3;
    uint8_t* stg = stg_all + q * kG2StageWarpBytes;
    const uint32_t tempty_leader = mapa_shared(smem_u32(tempty), 0);
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int u = pair; u < num_units; u += npairs) {
      const int m_t = u % mt2, n_t = u / mt2;
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const int row = m_t * 256 + int(rank) * 128 + q * 32 + lane;
      epi_tile_staged<BN, EPI>(p, stg, lane, n_t, row, tmem_base + (uint32_t(q * 32) << 16) + acc * BN);
      tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if (p.rel_cluster) mbar_arrive_cluster(tempty_leader + acc * 8);
        else mbar_arrive_remote(tempty_leader + acc * 8);
      }
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
    }
  }
  tc_fence_before();
  __syncthreads();
  cluster_sync();  // the peer's MMAs, commits and remote arrivals are done before TMEM is freed
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc2<512>(tmem_base);
  }
}

// ------------------------------------------------------------------------------ host side
static PFN_cuTensorMapEncodeTiled_v12000 get_encode_fn() {
  static PFN_cuTensorMapEncodeTiled_v12000 fn = nullptr;
  if (!fn) {
    void* ptr = nullptr;
    cudaDriverEntryPointQueryResult qres;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &ptr, cudaEnableDefault, &qres) == cudaSuccess &&
        qres == cudaDriverEntryPointSuccess)
      fn = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(ptr);
  }
  return fn;
}

int make_tmap_2d_bf16(CUtensorMap* out, const void* base, uint64_t rows, uint64_t cols, uint64_t row_stride_elems,
                      uint32_t box_rows, uint32_t box_cols, bool swizzle128) {
  auto fn = get_encode_fn();
  if (!fn) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {row_stride_elems * 2};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE,
                  swizzle128 ? CU_TENSOR_MAP_SWIZZLE_128B : CU_TENSOR_MAP_SWIZZLE_NONE,
                  CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    char msg[256];
    snprintf(msg, sizeof msg, "cuTensorMapEncodeTiled failed (%d): rows=%llu cols=%llu box=%ux%u", int(r),
             (unsigned long long)rows, (unsigned long long)cols, box_rows, box_cols);
    return set_error(QOS_ERR_CUDA, msg);
  }
  return QOS_OK;
}

int make_tmap_3d_bf16(CUtensorMap* out, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint32_t b0,
                      uint32_t b1, uint32_t b2) {
  auto fn = get_encode_fn();
  if (!fn) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[3] = {d0, d1, d2};
  cuuint64_t strides[2] = {d0 * 2, d0 * d1 * 2};
  cuuint32_t box[3] = {b0, b1, b2};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled (3d) failed");
  return QOS_OK;
}

// 3-D map with explicit byte strides of dims 1 and 2 (dim 0 contiguous), 128-B swizzle
int make_tmap_3d_bf16_strided(CUtensorMap* out, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint64_t s1,
                              uint64_t s2, uint32_t b0, uint32_t b1, uint32_t b2) {
  auto fn = get_encode_fn();
  if (!fn) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[3] = {d0, d1, d2};
  cuuint64_t strides[2] = {s1, s2};
  cuuint32_t box[3] = {b0, b1, b2};
  cuuint32_t estr[3] = {1, 1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled (3d strided) failed");
  return QOS_OK;
}

int make_tmap_kv5(CUtensorMap* out, const void* base, uint64_t hd, uint64_t hkv, uint64_t num_blocks, uint64_t planes,
                  uint32_t blocks_per_box) {
  auto fn = get_encode_fn();
  if (!fn) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled unavailable");
  cuuint64_t dims[5] = {hd, 16, hkv, num_blocks, planes};
  cuuint64_t strides[4] = {hd * 2, 16 * hd * 2, hkv * 16 * hd * 2, num_blocks * hkv * 16 * hd * 2};
  cuuint32_t box[5] = {64, 16, 1, blocks_per_box, 1};
  cuuint32_t estr[5] = {1, 1, 1, 1, 1};
  CUresult r = fn(out, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 5, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error(QOS_ERR_CUDA, "cuTensorMapEncodeTiled (kv 5d) failed");
  return QOS_OK;
}

template <int BN, int EPI>
static cudaError_t launch_gemm_t(const CUtensorMap& ta, const CUtensorMap& tb, const GemmArgs& a, int grid,
                                 cudaStream_t st) {
  auto kern = gemm_tcgen05_kernel<BN, EPI>;
  static std::atomic<uint64_t> attr_set{0};
  if (cudaError_t e = smem_attr_once(kern, int(GemmCfg<BN>::kSmemBytes), attr_set); e != cudaSuccess) return e;
  return launch_pdl(kern, dim3(grid), dim3(kGemmThreads), GemmCfg<BN>::kSmemBytes, st, ta, tb, a);
}

int gemm_pick_bn(int64_t M, int64_t N, int epi, int num_sms) {
  // Tile width by cost: waves x cycles per 64-deep k-block of one tile on one SM, measured on
  // B200 (tools/gemm_bench.py, ncu cycles): ~445 for 128 x 128 tiles (L2 -> smem feed bound:
  // 32 KB per 256 MMA cycles) and ~630 for 128 x 256 tiles (48 KB per 512 MMA cycles).  One
  // wave of wide tiles beats two waves of narrow ones (e.g. T = 768: QKV 33 -> ~21 us, down
  // 99 -> ~74 us); at large M this reduces to the old rule (wide once they fill the SMs).
  (void)epi;
  if (N % 256 != 0) return 128;
  const int64_t mt = (M + kBM - 1) / kBM;
  const int64_t w128 = (mt * (N / 128) + num_sms - 1) / num_sms;
  const int64_t w256 = (mt * (N / 256) + num_sms - 1) / num_sms;
  return w256 * 630 < w128 * 445 ? 256 : 128;
}

// Tile width and ordered split-K of an EPI_ADD_F32 projection (the O and down projections of
// a step below the fold threshold).  The mid-T steps (T 256-1024) leave most SMs idle with
// whole tiles (T = 512: 64 tiles of 128 x 256 on 148 SMs); slicing K fills them, but every
// extra slice serialises one more red.add epilogue of the tile.  Cost of a launch =
// waves x k-blocks per unit x c(BN) + (slices - 1) x E(BN), with c and E fitted (relative
// least squares, max error 19%, mean 4%) to the O and down projections of Llama-3-8B at
// T = 256..1536 over BN {128, 256} x slices {1..4} (tools/gemm_bench.py with QOS_GEMM_BN,
// profiles/gemm_addsplit_grid_r2.jsonl): c = 403 / 687 cycles per k-block, E = 5600 / 8500
// cycles (at BN 128 / 256; at these sizes the 128 x 256 tile is L2-fed, not MMA-bound).
// Inside the step (PDL neighbours, the residual's L2 state) a split only paid off where the model
// predicts a large gain on a long-K projection: slices are taken for K >= 8192 (down) when they
// beat the best whole-tile choice by >= 15% (in-process A/B on the 32-layer step,
// profiles/step_addsplit_r2c.jsonl: the O projection split and down at T = 512 were slower).
void gemm_pick_add_split(int64_t M, int64_t N, int64_t K, int num_sms, int64_t max_tiles, int* bn_out, int* ks_out) {
  const int64_t mt = (M + kBM - 1) / kBM, kblocks = K / kBK;
  int64_t best = INT64_MAX, best1 = INT64_MAX;
  int bn1 = 128, bns = 128, kss = 1;
  for (int bn = 128; bn <= 256; bn += 128) {
    if (bn == 256 && N % 256) continue;
    const int64_t tiles = mt * ((N + bn - 1) / bn);
    const int64_t ckb = bn == 256 ? 687 : 403, epi = bn == 256 ? 8500 : 5600;
    for (int ks = 1; ks <= 4; ++ks) {
      if (ks > 1 && (kblocks < 128 || kblocks / ks < 8 || tiles > max_tiles)) break;
      const int64_t waves = (tiles * ks + num_sms - 1) / num_sms;
      const int64_t cost = waves * ((kblocks + ks - 1) / ks) * ckb + int64_t(ks - 1) * epi;
      if (ks == 1 && cost < best1) {
        best1 = cost;
        bn1 = bn;
      }
      if (cost < best) {
        best = cost;
        bns = bn;
        kss = ks;
      }
    }
  }
  const bool split = kss > 1 && best * 100 <= best1 * 85;
  *bn_out = split ? bns : bn1;
  *ks_out = split ? kss : 1;
}

int gemm_pick_ksplit(int64_t M, int64_t N, int64_t K, int bn, int num_sms, int64_t max_units) {
  // weight-bound small-M GEMMs: split K until the units cover the SMs (>= 4 k-blocks each)
  const int64_t tiles = ((M + kBM - 1) / kBM) * ((N + bn - 1) / bn);
  int ks = 1;
  while (tiles * ks * 2 <= num_sms + num_sms / 4 && (K / kBK) / (ks * 2) >= 4 && tiles * ks * 2 <= max_units) ks *= 2;
  return ks;
}

int gemm_run(const CUtensorMap& ta, const CUtensorMap& tb, int bn, int64_t M, int64_t N, int64_t K, int epi, void* C,
             int64_t ldc, const float* bias, int num_sms, cudaStream_t st, int ksplit, float* part, int* counters,
             int a_row0, int max_ctas, const QkvRopeArgs* rope, int sk_mode, bool coop, const NormFold* fold) {
  GemmArgs a{};
  set_fold(a, fold);
  if (fold && ksplit > 1) return set_error(QOS_ERR_INVALID_ARG, "gemm: folded norm needs one pass");
  if (fold) sk_mode = 0;  // whole tiles only
  a.M = int(M);
  a.N = int(N);
  a.K = int(K);
  a.mt = int((M + kBM - 1) / kBM);
  a.nt = int((N + bn - 1) / bn);
  a.ksplit = ksplit < 1 ? 1 : ksplit;
  a.C = C;
  a.ldc = int(ldc);
  a.bias = bias;
  a.part = part;
  a.counters = counters;
  a.a_row0 = a_row0;
  a.pos = rope ? rope->pos : nullptr;
  a.slot = rope ? rope->slot : nullptr;
  a.rope = rope ? rope->tab : nullptr;
  a.kplane = rope ? reinterpret_cast<__nv_bfloat16*>(rope->kplane) : nullptr;
  a.vplane = rope ? reinterpret_cast<__nv_bfloat16*>(rope->vplane) : nullptr;
  a.H = rope ? rope->H : 0;
  a.Hkv = rope ? rope->Hkv : 0;
  a.hd = rope ? rope->hd : 0;
  if (epi == EPI_QKV_ROPE && (!rope || a.hd <= 0 || bn % a.hd))
    return set_error(QOS_ERR_INVALID_ARG, "gemm: QKV_ROPE needs rope args and BN % hd == 0");
  // EPI_ADD_F32 split-K accumulates in place in slice order (needs only the tile counters, and
  // every CTA resident so a waiting slice cannot block the one it waits for)
  a.ordered = (a.ksplit > 1 && epi == EPI_ADD_F32) ? 1 : 0;
  if (a.ordered && !coop) return set_error(QOS_ERR_INVALID_ARG, "gemm: ordered split-K needs co-resident CTAs");
  if (a.ksplit > 1 && (!counters || (!a.ordered && !part)))
    return set_error(QOS_ERR_INVALID_ARG, "gemm: split-K needs workspace");
  const int tiles = a.mt * a.nt * a.ksplit;
  int grid = tiles < num_sms ? tiles : num_sms;
  if (max_ctas > 0 && grid > max_ctas) grid = max_ctas;   // SM budget (co-scheduled streams)
  // Stream-K when whole-tile waves would leave SMs idle in the last wave (e.g. 272 tiles on
  // 148 SMs: 92%): every CTA gets tiles * kblocks / grid k-blocks; cut tiles are reduced from
  // fp32 partials (2 slots of 128 x BN per CTA in `part`, one counter per tile).
  a.sk = 0;
  a.coop = coop ? 1 : 0;
  a.work = int64_t(a.mt) * a.nt * (K / kBK);
  if (a.ksplit == 1 && sk_mode > 0 && part && counters && tiles <= 4096 && 2 * grid <= 512 && a.work >= grid) {
    const int waves = (tiles + grid - 1) / grid;
    if (sk_mode == 2 || (tiles > grid && double(tiles) < 0.95 * double(waves) * grid)) a.sk = 1;
    if (sk_mode == 2) {  // forced (tests): as many CTAs as give >= 4 k-blocks each
      int64_t g = a.work / 4;
      const int cap = max_ctas > 0 ? min(max_ctas, num_sms) : num_sms;
      grid = int(g < 1 ? 1 : g > cap ? cap : g);
    }
  }
  cudaError_t e = cudaSuccess;
#define QOS_GEMM_CASE(BNV, EPIV) \
  if (bn == BNV && epi == EPIV) e = launch_gemm_t<BNV, EPIV>(ta, tb, a, grid, st); else
  QOS_GEMM_CASE(128, EPI_STORE_BF16)
  QOS_GEMM_CASE(256, EPI_STORE_BF16)
  QOS_GEMM_CASE(128, EPI_STORE_F32)
  QOS_GEMM_CASE(256, EPI_STORE_F32)
  QOS_GEMM_CASE(128, EPI_BIAS_BF16)
  QOS_GEMM_CASE(256, EPI_BIAS_BF16)
  QOS_GEMM_CASE(128, EPI_SILU_GATE)
  QOS_GEMM_CASE(256, EPI_SILU_GATE)
  QOS_GEMM_CASE(128, EPI_ADD_F32)
  QOS_GEMM_CASE(256, EPI_ADD_F32)
  QOS_GEMM_CASE(128, EPI_QKV_ROPE)
  QOS_GEMM_CASE(256, EPI_QKV_ROPE)
  return set_error(QOS_ERR_INVALID_ARG, "gemm: bad tile/epilogue");
#undef QOS_GEMM_CASE
  if (e != cudaSuccess) return set_cuda_error(e, "gemm launch");
  return QOS_OK;
}

template <int EPI>
static cudaError_t launch_gemm2_t(const CUtensorMap& ta, const CUtensorMap& tb, const GemmArgs& a, int grid,
                                  cudaStream_t st) {
  auto kern = gemm2_tcgen05_kernel<EPI>;
  static std::atomic<uint64_t> attr_set{0};
  if (cudaError_t e = smem_attr_once(kern, int(kG2Smem), attr_set); e != cudaSuccess) return e;
  return launch_pdl_cluster(kern, dim3(grid), dim3(kGemmThreads), kG2Smem, 2, st, ta, tb, a);
}

bool gemm2_eligible(int64_t M, int64_t N, int64_t K, int num_sms) {
  // 256 x 256 pair tiles, whole N tiles; taken once the single-CTA 128 x 256 tiles fill the SMs
  // and the pair tiles need no more waves (each SM does a 128 x 256 x 64 step per k-block
  // either way; the pair kernel does it with a third less smem traffic, but pads M to 256:
  // at M = 2176 the gate/up GEMM needs 14 pair waves vs 13 single-CTA waves and is slower)
  if (N % 256 || K % kBK) return false;
  const int64_t t1 = ((M + 127) / 128) * (N / 256), t2 = ((M + 255) / 256) * (N / 256);
  if (t1 < num_sms) return false;
  const int64_t w1 = (t1 + num_sms - 1) / num_sms, w2 = (t2 + num_sms / 2 - 1) / (num_sms / 2);
  return w2 <= w1;
}

// tb: tensor map over B with 128-row boxes; ta: over A with 128-row boxes
// accumulator release of the CTA-pair epilogue: 0 = .release.cta remote arrive (default; the
// .cluster form costs a MEMBAR.ALL.GPU per arrival, waiting for the epilogue's global stores)
static int g_gemm2_rel_cluster = 0;
void set_gemm2_rel_cluster(int v) { g_gemm2_rel_cluster = v; }

int gemm2_run(const CUtensorMap& ta, const CUtensorMap& tb, int64_t M, int64_t N, int64_t K, int epi, void* C,
              int64_t ldc, const float* bias, int num_sms, cudaStream_t st, int a_row0, int max_ctas,
              const QkvRopeArgs* rope, const NormFold* fold) {
  GemmArgs a{};
  set_fold(a, fold);
  a.M = int(M);
  a.N = int(N);
  a.K = int(K);
  a.mt = int((M + 255) / 256);
  a.nt = int(N / 256);
  a.ksplit = 1;
  a.C = C;
  a.ldc = int(ldc);
  a.bias = bias;
  a.a_row0 = a_row0;
  a.pos = rope ? rope->pos : nullptr;
  a.slot = rope ? rope->slot : nullptr;
  a.rope = rope ? rope->tab : nullptr;
  a.kplane = rope ? reinterpret_cast<__nv_bfloat16*>(rope->kplane) : nullptr;
  a.vplane = rope ? reinterpret_cast<__nv_bfloat16*>(rope->vplane) : nullptr;
  a.H = rope ? rope->H : 0;
  a.Hkv = rope ? rope->Hkv : 0;
  a.hd = rope ? rope->hd : 0;
  if (epi == EPI_QKV_ROPE && (!rope || a.hd <= 0 || 256 % a.hd))
    return set_error(QOS_ERR_INVALID_ARG, "gemm2: QKV_ROPE needs rope args and 256 % hd == 0");
  a.rel_cluster = g_gemm2_rel_cluster;
  const int units = a.mt * a.nt;
  int pairs = std::min(units, (max_ctas > 0 ? std::min(max_ctas, num_sms) : num_sms) / 2);
  if (pairs < 1) pairs = 1;
  cudaError_t e;
  switch (epi) {
    case EPI_STORE_BF16: e = launch_gemm2_t<EPI_STORE_BF16>(ta, tb, a, 2 * pairs, st); break;
    case EPI_STORE_F32: e = launch_gemm2_t<EPI_STORE_F32>(ta, tb, a, 2 * pairs, st); break;
    case EPI_BIAS_BF16: e = launch_gemm2_t<EPI_BIAS_BF16>(ta, tb, a, 2 * pairs, st); break;
    case EPI_SILU_GATE: e = launch_gemm2_t<EPI_SILU_GATE>(ta, tb, a, 2 * pairs, st); break;
    case EPI_ADD_F32: e = launch_gemm2_t<EPI_ADD_F32>(ta, tb, a, 2 * pairs, st); break;
    case EPI_QKV_ROPE: e = launch_gemm2_t<EPI_QKV_ROPE>(ta, tb, a, 2 * pairs, st); break;
    default: return set_error(QOS_ERR_INVALID_ARG, "gemm2: bad epilogue");
  }
  if (e != cudaSuccess) return set_cuda_error(e, "gemm2 launch");
  return QOS_OK;
}

int gemm_check_shape(int64_t M, int64_t N, int64_t K, int epi) {
  if (M < 1 || N < 32 || K < 64) return set_error(QOS_ERR_INVALID_ARG, "gemm: M>=1, N>=32, K>=64 required");
  if (K % 64) return set_error(QOS_ERR_UNSUPPORTED, "gemm: K % 64 != 0");
  if (N % 32) return set_error(QOS_ERR_UNSUPPORTED, "gemm: N % 32 != 0");
  if (epi == EPI_SILU_GATE && N % 128) return set_error(QOS_ERR_UNSUPPORTED, "gemm: SILU_GATE needs N % 128 == 0");
  if (epi < 0 || epi > EPI_ADD_F32) return set_error(QOS_ERR_INVALID_ARG, "gemm: unknown epilogue");  // public ones
  return QOS_OK;
}

}  // namespace qos
