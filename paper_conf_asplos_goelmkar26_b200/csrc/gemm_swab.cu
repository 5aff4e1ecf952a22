// gemm_swab.cu — weight-streaming tcgen05 GEMM for small token counts (a4 / a9 / a11 / a12 /
// a13 at T <= 256, i.e. decode-heavy steps and the LM head).
//
// C[M][N] = A[M][K] · W[N][K]^T with M = tokens (small), N = output features, computed
// transposed ("swap AB"): D[128 weight rows][BNT tokens] = W_tile · A_tile^T, so the UMMA M=128
// side is filled by weights and the token count only sets UMMA N (16..256).  Below the ridge
// (T ≲ 260) these GEMMs are bound by streaming the weights once from HBM, so
// the work is split "stream-K": the linear (tile, k-block) iteration space is cut into one
// contiguous equal range per CTA (one CTA per SM), every SM streams 1/148 of the weights, and
// tiles cut by a range boundary are reduced deterministically by the last arriving CTA in CTA
// order.  Epilogues are the same fused ones as gemm.cu (bf16 / f32 store, bias, SiLU-gate,
// fp32 residual add, QKV + RoPE + paged-KV append), re-done for the transposed accumulator:
// thread = output feature, TMEM column = token, so stores are coalesced across the warp.
//
// Roles (192 threads): warp 0 TMA producer, warp 1 UMMA issuer, warps 2-5 epilogue (TMEM
// lane quarter = warp & 3), two TMEM accumulators so the epilogue of one segment overlaps the
// MMAs of the next.
#include <cstdio>
#include <cstdlib>

#include <cuda_fp16.h>

#include "common.cuh"
#include "internal.h"

namespace qos {

namespace {

constexpr int kSwThreads = 192;
constexpr int kSwBK = 64;
constexpr int kSwWBytes = 128 * kSwBK * 2;      // weight tile: 128 rows x 64 k (16 KB)
constexpr int kSwXchFloats = 2 * 16 * 128;      // epilogue exchange: 2 buffers x 16 tokens x 128 rows

template <int BNT>
struct SwCfg {
  static constexpr int kTBytes = BNT * kSwBK * 2;                  // token tile
  static constexpr int kStageBytes = kSwWBytes + kTBytes;
  static constexpr int kBudget = 200 * 1024;
  static constexpr int kStagesRaw = kBudget / kStageBytes;
  static constexpr int kStages = kStagesRaw > 12 ? 12 : kStagesRaw;
  static constexpr int kTmemCols = 2 * BNT < 32 ? 32 : 2 * BNT;
  static constexpr int kSmemBytes = kStages * kStageBytes + kSwXchFloats * 4 + 1024 /*align*/ + 256 /*barriers*/;
  static_assert(kSmemBytes <= 227 * 1024, "smem");
};

struct SwabArgs {
  int M, N, K;
  int nwt, ntt;      // weight tiles (N / 128), token tiles
  int kblocks;
  int64_t work;      // nwt * ntt * kblocks
  void* C;
  int ldc;
  const float* bias;
  float* part;       // partial slots [2 * grid][BNT][128] fp32
  int* counters;     // per tile, zero between launches
  int gran;          // range granule in k-blocks (divides kblocks)
  int coop;          // 1: split tiles reduced cooperatively after the ranges (needs co-residency)
  int a_row0;
  const int32_t* pos;
  const int32_t* slot;
  const float2* rope;
  __nv_bfloat16* kplane;
  __nv_bfloat16* vplane;
  int H, Hkv, hd;
};

QOS_DEV void sw_bar() { asm volatile("bar.sync 1, 128;" ::: "memory"); }  // the 4 epilogue warps

// CTA range boundaries of the linear iteration space
// (in granules of `gr` k-blocks, gr | kblocks: gr = kblocks gives whole tiles per CTA)
struct Ranges {
  int64_t Wg, G;
  int gr;
  QOS_DEV int64_t start(int64_t c) const { return (c * Wg / G) * gr; }
  QOS_DEV int cta_of(int64_t idx) const { return int(((idx / gr + 1) * G - 1) / Wg); }
};

// Epilogue of one (weight tile, token tile) from 16-token chunks supplied by fetch(tok0, v[16])
// (TMEM or the sum of split partials).  All 128 epilogue threads call it with the same
// arguments (the exchange barriers inside are uniform).  `xc` counts exchange-buffer uses.
template <int EPI, int BNT, typename Fetch>
QOS_DEV void swab_epilogue(const SwabArgs& p, int wt, int tt, int f, float* xch, int& xc, Fetch fetch,
                           int ch0 = 0, int chstep = 1) {
  const int tok_base = tt * BNT;
  const int mvalid = min(BNT, p.M - tok_base);
  const int gr = wt * 128 + f;  // output feature (weight row) of this thread
  for (int tok0 = ch0 * 16; tok0 < mvalid; tok0 += chstep * 16) {
    float v[16];
    fetch(tok0, v);
    const int nj = min(16, mvalid - tok0);
    if constexpr (EPI == EPI_STORE_BF16 || EPI == EPI_BIAS_BF16 || EPI == EPI_STORE_F32) {
      const float b = (EPI == EPI_BIAS_BF16) ? __ldg(p.bias + gr) : 0.f;
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        if (j < nj) {
          const size_t o = size_t(tok_base + tok0 + j) * p.ldc + gr;
          if constexpr (EPI == EPI_STORE_F32) reinterpret_cast<float*>(p.C)[o] = v[j];
          else reinterpret_cast<__nv_bfloat16*>(p.C)[o] = __float2bfloat16_rn(v[j] + b);
        }
      }
    } else if constexpr (EPI == EPI_ADD_F32) {
      float* c = reinterpret_cast<float*>(p.C);
      float old[16];
#pragma unroll
      for (int j = 0; j < 16; ++j) old[j] = j < nj ? c[size_t(tok_base + tok0 + j) * p.ldc + gr] : 0.f;
#pragma unroll
      for (int j = 0; j < 16; ++j)
        if (j < nj) c[size_t(tok_base + tok0 + j) * p.ldc + gr] = old[j] + v[j];
    } else if constexpr (EPI == EPI_SILU_GATE) {
      // rows 0..63 of the tile are gate, 64..127 the matching up rows (64-row interleave)
      float* xb = xch + (xc & 1) * (16 * 128);
      ++xc;
      if (f >= 64) {
#pragma unroll
        for (int j = 0; j < 16; ++j) xb[j * 64 + (f - 64)] = v[j];
      }
      sw_bar();
      if (f < 64) {
        const int o = wt * 64 + f;
#pragma unroll
        for (int j = 0; j < 16; ++j)
          if (j < nj)
            reinterpret_cast<__nv_bfloat16*>(p.C)[size_t(tok_base + tok0 + j) * p.ldc + o] =
                __float2bfloat16_rn(silu(v[j]) * xb[j * 64 + f]);
      }
    } else if constexpr (EPI == EPI_QKV_ROPE) {
      // rotate-half pairs (i, i + hd/2) live in rows f and f ^ (hd/2) of the same head
      float* xb = xch + (xc & 1) * (16 * 128);
      ++xc;
      const float b = p.bias ? __ldg(p.bias + gr) : 0.f;
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        v[j] += b;
        xb[j * 128 + f] = v[j];
      }
      sw_bar();
      const int hd = p.hd, half = hd >> 1;
      const int head = gr / hd, i = gr - head * hd;
      const int ii = i < half ? i : i - half;
      const int partner = f ^ half;
      const bool rot = head < p.H + p.Hkv;
#pragma unroll
      for (int j = 0; j < 16; ++j) {
        if (j >= nj) break;
        const int tok = tok_base + tok0 + j;
        float out = v[j];
        if (rot) {
          const float2 cs = __ldg(p.rope + size_t(__ldg(p.pos + tok)) * half + ii);
          const float y = xb[j * 128 + partner];
          out = i < half ? v[j] * cs.x - y * cs.y : v[j] * cs.x + y * cs.y;
        }
        if (head < p.H + p.Hkv) {
          const __nv_bfloat16 ob = __float2bfloat16_rn(out);
          if (head < p.H) {
            reinterpret_cast<__nv_bfloat16*>(p.C)[size_t(tok) * p.ldc + gr] = ob;
          } else {
            const int sl = __ldg(p.slot + tok);
            p.kplane[((size_t(sl >> 4) * p.Hkv + (head - p.H)) * 16 + (sl & 15)) * hd + i] = ob;
          }
        } else {  // V is cached in fp16
          const int sl = __ldg(p.slot + tok);
          const __half oh = __float2half_rn(out);
          reinterpret_cast<__half*>(p.vplane)[((size_t(sl >> 4) * p.Hkv + (head - p.H - p.Hkv)) * 16 + (sl & 15)) * hd + i] = oh;
        }
      }
    }
  }
}

template <int BNT, int EPI>
__global__ void __launch_bounds__(kSwThreads, 1)
    gemm_swab_kernel(const __grid_constant__ CUtensorMap tmW, const __grid_constant__ CUtensorMap tmT,
                     const SwabArgs p) {
  using Cfg = SwCfg<BNT>;
  constexpr int S = Cfg::kStages;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  float* xch = reinterpret_cast<float*>(smem + S * Cfg::kStageBytes);
  uint64_t* full = reinterpret_cast<uint64_t*>(xch + kSwXchFloats);
  uint64_t* empty = full + S;
  uint64_t* tfull = empty + S;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(tempty + 2);
  int* s_last = reinterpret_cast<int*>(tmem_slot + 1);

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
    tma_prefetch_desc(&tmW);
    tma_prefetch_desc(&tmT);
  }
  if (warp == 1) tmem_alloc<Cfg::kTmemCols>(tmem_slot);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;
  griddep_launch_dependents();
  if (warp != 0) griddep_wait();

  const Ranges rg{p.work / p.gran, int64_t(gridDim.x), p.gran};
  const int c = blockIdx.x;
  const int64_t s0 = rg.start(c), e0 = rg.start(c + 1);
  const int kbl = p.kblocks;

  if (warp == 0) {
    // ------------------------------------------------------------ TMA producer
    if (elect_one()) {
      const uint64_t pol_w = l2_evict_first();  // weights: streamed exactly once
      const uint64_t pol_t = l2_evict_last();   // token tiles: re-read by every weight tile
      const int n = int(e0 - s0);
      const int npre = min(S, n);
      // PDL: weight tiles do not depend on the previous kernel — request them before the wait
      for (int i = 0; i < npre; ++i) {
        const int64_t idx = s0 + i;
        const int t = int(idx / kbl), kb = int(idx - int64_t(t) * kbl);
        mbar_arrive_expect_tx(&full[i], Cfg::kStageBytes);
        tma_load_2d_hint(smem + i * Cfg::kStageBytes, &tmW, &full[i], kb * kSwBK, (t / p.ntt) * 128, pol_w);
      }
      griddep_wait();
      for (int i = 0; i < npre; ++i) {
        const int64_t idx = s0 + i;
        const int t = int(idx / kbl), kb = int(idx - int64_t(t) * kbl);
        tma_load_2d_hint(smem + i * Cfg::kStageBytes + kSwWBytes, &tmT, &full[i], kb * kSwBK,
                         p.a_row0 + (t % p.ntt) * BNT, pol_t);
      }
      int stage = npre % S;
      uint32_t phase = (npre == S) ? 1u : 0u;
      for (int i = npre; i < n; ++i) {
        const int64_t idx = s0 + i;
        const int t = int(idx / kbl), kb = int(idx - int64_t(t) * kbl);
        mbar_wait(&empty[stage], phase ^ 1);
        uint8_t* st = smem + stage * Cfg::kStageBytes;
        mbar_arrive_expect_tx(&full[stage], Cfg::kStageBytes);
        tma_load_2d_hint(st, &tmW, &full[stage], kb * kSwBK, (t / p.ntt) * 128, pol_w);
        tma_load_2d_hint(st + kSwWBytes, &tmT, &full[stage], kb * kSwBK, p.a_row0 + (t % p.ntt) * BNT, pol_t);
        if (++stage == S) { stage = 0; phase ^= 1; }
      }
    }
  } else if (warp == 1) {
    // ------------------------------------------------------------ UMMA issuer
    if (elect_one()) {
      constexpr uint32_t idesc = umma_idesc_bf16(128, BNT);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int64_t idx = s0; idx < e0;) {
        const int t = int(idx / kbl), kb0 = int(idx - int64_t(t) * kbl);
        const int kb1 = int(min(int64_t(kbl), int64_t(kb0) + (e0 - idx)));
        mbar_wait(&tempty[acc], acc_phase ^ 1);
        tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * BNT;
        for (int kb = kb0; kb < kb1; ++kb) {
          mbar_wait(&full[stage], phase);
          tc_fence_after();
          const uint32_t w_base = smem_u32(smem + stage * Cfg::kStageBytes);
          const uint32_t t_base = w_base + kSwWBytes;
#pragma unroll
          for (int k = 0; k < kSwBK / 16; ++k)
            umma_bf16(d_tmem, umma_desc_sw128(w_base + k * 32), umma_desc_sw128(t_base + k * 32), idesc,
                      (kb > kb0 || k > 0) ? 1u : 0u);
          umma_commit(&empty[stage]);
          if (++stage == S) { stage = 0; phase ^= 1; }
        }
        umma_commit(&tfull[acc]);
        if (++acc == 2) { acc = 0; acc_phase ^= 1; }
        idx += kb1 - kb0;
      }
    }
  } else {
    // ------------------------------------------------------------ epilogue (warps 2..5)
    const int q = warp & 3;
    const int f = q * 32 + lane;  // weight row of the tile = TMEM lane
    int acc = 0;
    uint32_t acc_phase = 0;
    int xc = 0;
    int pend[2], npend = 0;  // split tiles whose cooperative reduction runs after the range
    // sum of the parked partials of tile t (participants cf..cl, in CTA order: deterministic)
    auto reduce_fetch = [&](int t, int cf, int cl, int mvalid) {
      return [=](int tok0, float (&v)[16]) {
#pragma unroll
        for (int j = 0; j < 16; ++j) v[j] = 0.f;
        auto slot_of = [&](int cc) { return (rg.start(cc) >= int64_t(t) * kbl) ? 2 * cc : 2 * cc + 1; };
        int cc = cf;
        for (; cc + 1 <= cl; cc += 2) {  // two partials' loads in flight per step
          const float* p0 = p.part + size_t(slot_of(cc)) * BNT * 128 + size_t(tok0) * 128 + f;
          const float* p1 = p.part + size_t(slot_of(cc + 1)) * BNT * 128 + size_t(tok0) * 128 + f;
          float a0[16], a1[16];
#pragma unroll
          for (int j = 0; j < 16; ++j) {
            a0[j] = (tok0 + j < mvalid) ? __ldcg(p0 + size_t(j) * 128) : 0.f;
            a1[j] = (tok0 + j < mvalid) ? __ldcg(p1 + size_t(j) * 128) : 0.f;
          }
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = (v[j] + a0[j]) + a1[j];
        }
        if (cc <= cl) {
          const float* p0 = p.part + size_t(slot_of(cc)) * BNT * 128 + size_t(tok0) * 128 + f;
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] += (tok0 + j < mvalid) ? __ldcg(p0 + size_t(j) * 128) : 0.f;
        }
      };
    };
    for (int64_t idx = s0; idx < e0;) {
      const int t = int(idx / kbl), kb0 = int(idx - int64_t(t) * kbl);
      const int kb1 = int(min(int64_t(kbl), int64_t(kb0) + (e0 - idx)));
      const int wt = t / p.ntt, tt = t % p.ntt;
      mbar_wait(&tfull[acc], acc_phase);
      tc_fence_after();
      const uint32_t tbase = tmem_base + (uint32_t(q * 32) << 16) + acc * BNT;
      if (kb0 == 0 && kb1 == kbl) {
        swab_epilogue<EPI, BNT>(p, wt, tt, f, xch, xc, [&](int tok0, float (&v)[16]) {
          uint32_t r[16];
          tmem_ld32x32b_x16(tbase + tok0, r);
          tmem_ld_wait();
#pragma unroll
          for (int j = 0; j < 16; ++j) v[j] = __uint_as_float(r[j]);
        });
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
      } else {
        // tile cut by a range boundary: park this segment's partial in its slot
        const int mvalid = min(BNT, p.M - tt * BNT);
        const int slot = (idx == s0) ? 2 * c : 2 * c + 1;
        float* mine = p.part + size_t(slot) * BNT * 128 + f;
        for (int tok0 = 0; tok0 < mvalid; tok0 += 16) {
          uint32_t r[16];
          tmem_ld32x32b_x16(tbase + tok0, r);
          tmem_ld_wait();
#pragma unroll
          for (int j = 0; j < 16; ++j)
            if (tok0 + j < mvalid) __stcg(mine + size_t(tok0 + j) * 128, __uint_as_float(r[j]));
        }
        tc_fence_before();
        __syncwarp();
        if (lane == 0) mbar_arrive(&tempty[acc]);
        __threadfence();
        sw_bar();
        const int cf = rg.cta_of(int64_t(t) * kbl), cl = rg.cta_of(int64_t(t + 1) * kbl - 1);
        if (p.coop) {
          if (threadIdx.x == 64) atomicAdd(p.counters + t, 1);
          pend[npend++] = t;
        } else {
          if (threadIdx.x == 64) *s_last = (atomicAdd(p.counters + t, 1) == cl - cf);
          sw_bar();
          if (*s_last) {
            __threadfence();
            swab_epilogue<EPI, BNT>(p, wt, tt, f, xch, xc, reduce_fetch(t, cf, cl, mvalid));
            if (threadIdx.x == 64) p.counters[t] = 0;  // ready for the next launch
          }
        }
      }
      if (++acc == 2) { acc = 0; acc_phase ^= 1; }
      idx += kb1 - kb0;
    }
    // Cooperative reduction (all CTAs are co-resident: one per SM, grid <= SMs).  Every
    // participant of a split tile waits, after its whole range, until all partials of the tile
    // are parked, then reduces and stores its share of the 16-token chunks; the counter counts
    // to 2n (parked + done) and the last participant resets it for the next launch.
    for (int i = 0; i < npend; ++i) {
      const int t = pend[i];
      const int wt = t / p.ntt, tt = t % p.ntt;
      const int mvalid = min(BNT, p.M - tt * BNT);
      const int cf = rg.cta_of(int64_t(t) * kbl), cl = rg.cta_of(int64_t(t + 1) * kbl - 1);
      const int n = cl - cf + 1;
      if (threadIdx.x == 64) {
        int v;
        do {
          asm volatile("ld.acquire.gpu.global.b32 %0, [%1];" : "=r"(v) : "l"(p.counters + t) : "memory");
        } while (v < n);
      }
      sw_bar();
      swab_epilogue<EPI, BNT>(p, wt, tt, f, xch, xc, reduce_fetch(t, cf, cl, mvalid), c - cf, n);
      sw_bar();
      if (threadIdx.x == 64 && atomicAdd(p.counters + t, 1) == 2 * n - 1) p.counters[t] = 0;
    }
  }
  __syncthreads();
  if (warp == 1) {
    tc_fence_after();
    tmem_dealloc<Cfg::kTmemCols>(tmem_base);
  }
}

template <int BNT, int EPI>
cudaError_t launch_swab_t(const CUtensorMap& tw, const CUtensorMap& tt, const SwabArgs& a, int grid,
                          cudaStream_t st) {
  auto kern = gemm_swab_kernel<BNT, EPI>;
  static std::atomic<uint64_t> attr_set{0};
  if (cudaError_t e = smem_attr_once(kern, int(SwCfg<BNT>::kSmemBytes), attr_set); e != cudaSuccess) return e;
  return launch_pdl(kern, dim3(grid), dim3(kSwThreads), SwCfg<BNT>::kSmemBytes, st, tw, tt, a);
}

}  // namespace

int swab_pick_bnt(int64_t M) {
  int b = 16;
  while (b < M && b < 256) b *= 2;
  return b;
}

bool swab_prefer(int64_t M, int64_t N, int num_sms) {
  // B200 measurements (tools/gemm_bench.py, profiles/gemm_small_m_r1.md): the weight-streaming
  // kernel wins at very small T, and up to T = 256 when the tile kernel would leave most SMs
  // idle (few 128-wide output tiles: the O and down projections, N = d)
  // Round 2, measured inside the 32-layer step (profiles/step_swab_r2a.jsonl): taking it for
  // every projection up to T = 64 (the QKV and gate/up projections went to the tile kernel from
  // T = 17 / 33) makes decode-heavy steps 5-13% faster; at T = 96-112 it is 2% slower.
  // (Isolated op timings mislead here: an op's A tensor has exactly M rows, so the tile kernel's
  // 128-row boxes read out of bounds, which the engine's workspace-wide maps never do.)
  if (N % 128) return false;
  if (M <= 64) return true;
  if (M > 256) return false;
  const int64_t tiles = ((M + 127) / 128) * (N / 128);
  return tiles * 4 < num_sms;
}
// with K: long-K projections (the down projection, K = F) stream more weight bytes per output
// tile, so the weight-streaming kernel keeps winning up to twice as many tiles — up to T = 128
// (round 2, in-step A/B, profiles/step_swab_r2c.jsonl: at T = 96-128 it is 2% faster, at
// T = 160-256 the tile kernel is 0.4-4% faster; the round-1 bound of 256 came from isolated
// timings with out-of-bounds A boxes)
bool swab_prefer_k(int64_t M, int64_t N, int64_t K, int num_sms) {
  if (swab_prefer(M, N, num_sms)) return true;
  if (N % 128 || M > 128 || K < 8192) return false;
  return ((M + 127) / 128) * (N / 128) * 2 < num_sms;
}

static int g_swab_gran = -1;  // option swab_gran (process-wide): -1 automatic
void set_swab_gran(int v) { g_swab_gran = v; }

int swab_grid(int64_t M, int64_t N, int64_t K, int bnt, int num_sms) {
  const int64_t work = (N / 128) * ((M + bnt - 1) / bnt) * (K / kSwBK);
  const int64_t g = work / 4;  // >= 4 k-blocks (64 KB of weights) per CTA
  return int(g < 1 ? 1 : (g > num_sms ? num_sms : g));
}

int gemm_swab_run(const CUtensorMap& tw, const CUtensorMap& tt, int bnt, int64_t M, int64_t N, int64_t K, int epi,
                  void* C, int64_t ldc, const float* bias, int num_sms, cudaStream_t st, float* part, int* counters,
                  int64_t part_floats, int max_tiles, int a_row0, const QkvRopeArgs* rope, bool coop) {
  if (N % 128 || K % kSwBK) return set_error(QOS_ERR_UNSUPPORTED, "gemm_swab: N % 128, K % 64");
  SwabArgs a;
  a.M = int(M);
  a.N = int(N);
  a.K = int(K);
  a.nwt = int(N / 128);
  a.ntt = int((M + bnt - 1) / bnt);
  a.kblocks = int(K / kSwBK);
  a.work = int64_t(a.nwt) * a.ntt * a.kblocks;
  a.C = C;
  a.ldc = int(ldc);
  a.bias = bias;
  a.part = part;
  a.counters = counters;
  a.coop = coop ? 1 : 0;
  a.a_row0 = a_row0;
  a.pos = rope ? rope->pos : nullptr;
  a.slot = rope ? rope->slot : nullptr;
  a.rope = rope ? rope->tab : nullptr;
  a.kplane = rope ? reinterpret_cast<__nv_bfloat16*>(rope->kplane) : nullptr;
  a.vplane = rope ? reinterpret_cast<__nv_bfloat16*>(rope->vplane) : nullptr;
  a.H = rope ? rope->H : 0;
  a.Hkv = rope ? rope->Hkv : 0;
  a.hd = rope ? rope->hd : 0;
  if (epi == EPI_QKV_ROPE && (!rope || (a.hd != 64 && a.hd != 128)))
    return set_error(QOS_ERR_INVALID_ARG, "gemm_swab: QKV_ROPE needs rope args, hd 64/128");
  if (epi == EPI_BIAS_BF16 && !bias) return set_error(QOS_ERR_INVALID_ARG, "gemm_swab: bias");
  // Range granule: when the tiles are fewer than the SMs, split every tile into s equal
  // aligned K parts (one segment per CTA, s * tiles >= 80% of the SMs) — measured faster than
  // unaligned stream-K ranges on B200 (tools/gemm_bench.py); otherwise plain stream-K.
  const int64_t tiles = int64_t(a.nwt) * a.ntt;
  int grid = swab_grid(M, N, K, bnt, num_sms);
  a.gran = 1;
  if (tiles < num_sms) {
    for (int sp = int(num_sms / tiles); sp >= 2; --sp) {
      if (a.kblocks % sp == 0 && sp * tiles * 5 >= int64_t(num_sms) * 4 && a.kblocks / sp >= 4) {
        a.gran = a.kblocks / sp;
        grid = int(sp * tiles);
        break;
      }
    }
  }
  const char* genv = getenv("QOS_SWAB_GRAN");
  if (g_swab_gran >= 0 || genv) {  // experiment knob: force a granule (0 = whole tiles)
    int v = g_swab_gran >= 0 ? g_swab_gran : atoi(genv);
    if (v == 0) v = a.kblocks;
    while (v > 1 && a.kblocks % v) --v;
    a.gran = v < 1 ? 1 : v;
    grid = swab_grid(M, N, K, bnt, num_sms);
  }
  if (grid > a.work / a.gran) grid = int(a.work / a.gran);
  if (int64_t(a.nwt) * a.ntt > max_tiles || int64_t(2) * grid * bnt * 128 > part_floats || !part || !counters)
    return set_error(QOS_ERR_INVALID_ARG, "gemm_swab: workspace too small for the shape");
  cudaError_t e = cudaSuccess;
#define QOS_SW_CASE(B, E) \
  if (bnt == B && epi == E) e = launch_swab_t<B, E>(tw, tt, a, grid, st); else
#define QOS_SW_EPIS(B)                                                                                     \
  QOS_SW_CASE(B, EPI_STORE_BF16) QOS_SW_CASE(B, EPI_STORE_F32) QOS_SW_CASE(B, EPI_BIAS_BF16)              \
  QOS_SW_CASE(B, EPI_SILU_GATE) QOS_SW_CASE(B, EPI_ADD_F32) QOS_SW_CASE(B, EPI_QKV_ROPE)
  QOS_SW_EPIS(16)
  QOS_SW_EPIS(32)
  QOS_SW_EPIS(64)
  QOS_SW_EPIS(128)
  QOS_SW_EPIS(256)
  return set_error(QOS_ERR_INVALID_ARG, "gemm_swab: bad tile/epilogue");
#undef QOS_SW_EPIS
#undef QOS_SW_CASE
  if (e != cudaSuccess) return set_cuda_error(e, "gemm_swab launch");
  return QOS_OK;
}

}  // namespace qos
