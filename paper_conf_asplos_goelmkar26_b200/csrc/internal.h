// internal.h — declarations shared by the libqoserve translation units (not part of the ABI).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/qoserve.h"
#include "../../include/qoserve_ops.h"

namespace qos {

bool pdl_enabled();
void set_pdl(bool on);
// prefill attention: every n-th exp2 pair on the FMA pipe (0 = all on MUFU); process-wide
void set_fa_poly(int n);
void set_fa_kvfirst(int v);
void set_fa_tma5(int v);
void set_fa_psplit(int v);  // process-wide: persistent prefill attention releases P in two halves  // process-wide: persistent prefill attention loads 4-block runs in one TMA op
void set_gemm2_rel_cluster(int v);  // process-wide experiment (gemm.cu)  // process-wide: persistent prefill attention loads K/V before Q
void set_swab_gran(int v);  // weight-streaming GEMM range granule (k-blocks; -1 automatic, 0 whole tiles)

enum { EPI_STORE_BF16 = QOS_EPI_STORE_BF16, EPI_STORE_F32 = QOS_EPI_STORE_F32, EPI_BIAS_BF16 = QOS_EPI_BIAS_BF16,
       EPI_SILU_GATE = QOS_EPI_SILU_GATE, EPI_ADD_F32 = QOS_EPI_ADD_F32,
       EPI_QKV_ROPE = 5 /* internal: a4 + a5 + a6 fused (RoPE, q -> C, k/v -> paged cache; +bias) */ };

struct QkvRopeArgs {
  const int32_t* pos;
  const int32_t* slot;
  const float2* tab;
  void* kplane;
  void* vplane;
  int H, Hkv, hd;
};

// error reporting (thread-local last error; engine.cpp)
int set_error(int code, const char* msg);
int set_cuda_error(cudaError_t e, const char* where);
int count_launch(int n = 1);  // global launch counter hook (engine.cpp)

// ------------------------------------------------------------------ GEMM (gemm.cu)
int make_tmap_2d_bf16(CUtensorMap* out, const void* base, uint64_t rows, uint64_t cols, uint64_t row_stride_elems,
                      uint32_t box_rows, uint32_t box_cols, bool swizzle128);
int make_tmap_3d_bf16(CUtensorMap* out, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint32_t b0,
                      uint32_t b1, uint32_t b2);
int make_tmap_3d_bf16_strided(CUtensorMap* out, const void* base, uint64_t d0, uint64_t d1, uint64_t d2, uint64_t s1,
                              uint64_t s2, uint32_t b0, uint32_t b1, uint32_t b2);
// KV pool [2L][num_blocks][Hkv][16][hd] as a 5-D map {hd, 16, Hkv, num_blocks, 2L} with a
// {64, 16, 1, blocks_per_box, 1} box: runs of consecutive blocks of one head in one TMA op
int make_tmap_kv5(CUtensorMap* out, const void* base, uint64_t hd, uint64_t hkv, uint64_t num_blocks, uint64_t planes,
                  uint32_t blocks_per_box);
int gemm_pick_bn(int64_t M, int64_t N, int epi, int num_sms);
int gemm_check_shape(int64_t M, int64_t N, int64_t K, int epi);
int gemm_pick_ksplit(int64_t M, int64_t N, int64_t K, int bn, int num_sms, int64_t max_units);
// EPI_ADD_F32: tile width and ordered split-K slices (1 = whole tiles) by a wave cost model
void gemm_pick_add_split(int64_t M, int64_t N, int64_t K, int num_sms, int64_t max_tiles, int* bn_out, int* ks_out);
// ksplit > 1: split-K with fp32 partials in `part` ([units][128][bn]) and per-tile arrival
// counters (zero-initialised; each reducing CTA resets its own) — deterministic reduction order
// RMSNorm folded into the projections (single-pass tile kernels, no split-K / stream-K):
//   consumer (QKV, gate/up): A = bf16(r * g) rows; the accumulator of row t is scaled by
//     rs_in[t] = 1/rms(r_t) (before the bias) — diag(s)(A W) = (diag(s) A) W;
//   producer (O, down with EPI_ADD_F32): r += tile as a read-add-write, h_out = bf16(r * g_out),
//     ss_out[t][col / 128] = the sum of r^2 over that 128-column block; the last tile to finish
//     a 128-row block (arrival counter) sums each row's blocks in slot order into rs_out[t]
//     (fixed order: deterministic).
constexpr int kFoldSlots = 64;
constexpr int kFoldMinTokens = 1536;  // the engine folds the norms from this many tokens per step  // ss row stride: 128-column blocks of d <= 8192 (unused slots stay 0)
struct NormFold {
  const float* rs_in = nullptr;  // consumer: [M] 1/rms per row
  float* ss_out = nullptr;       // producer: [M][kFoldSlots] per-block sums of squares
  float* rs_out = nullptr;       // producer: [M] 1/rms, written by the last tile of each 128-row block
  int* cnt = nullptr;            // producer: [M/128 + 1] tile arrival counters (zero between launches)
  const void* g_out = nullptr;  // bf16 [d]
  void* h_out = nullptr;        // bf16 [M][d]
  int ss_n = 0, d = 0;
  float eps = 0.f;
  // TP peer group, reduce-scatter in the epilogue (EPI_STORE_BF16): row r of the partial goes to
  // its owner rank o = r / scat_rs, at scat[o] + (r - o * scat_rs) * ldc (this rank's slot of the
  // owner's receive buffer; peer memory) — the transfer overlaps the remaining tiles' MMAs
  void* scat[8] = {};
  int scat_rs = 0;
};
int gemm_run(const CUtensorMap& ta, const CUtensorMap& tb, int bn, int64_t M, int64_t N, int64_t K, int epi, void* C,
             int64_t ldc, const float* bias, int num_sms, cudaStream_t st, int ksplit = 1, float* part = nullptr,
             int* counters = nullptr, int a_row0 = 0, int max_ctas = 0, const QkvRopeArgs* rope = nullptr,
             int sk_mode = 1, bool coop = true, const NormFold* fold = nullptr);
// CTA-pair (cta_group::2) GEMM with 256 x 256 tiles for large M (gemm.cu); ta / tb: tensor
// maps with 128-row boxes over A and B.  gemm2_eligible: the shapes it takes.
bool gemm2_eligible(int64_t M, int64_t N, int64_t K, int num_sms);
int gemm2_run(const CUtensorMap& ta, const CUtensorMap& tb, int64_t M, int64_t N, int64_t K, int epi, void* C,
              int64_t ldc, const float* bias, int num_sms, cudaStream_t st, int a_row0 = 0, int max_ctas = 0,
              const QkvRopeArgs* rope = nullptr, const NormFold* fold = nullptr);
// sk_mode: 0 no stream-K, 1 automatic (last-wave quantisation), 2 always (needs part/counters:
// part >= 512 x 128 x 256 fp32, counters >= 4096); coop as in gemm_swab_run.

// ------------------------------------------------------------------ small-T GEMM (gemm_swab.cu)
// Swap-AB weight-streaming GEMM: tw = weight map (box 128 x 64), tt = token map (box bnt x 64).
// Requires N % 128 == 0.  part: >= 2 * grid * bnt * 128 floats; counters: >= (N/128) * ceil(M/bnt).
// coop: split tiles are reduced by all their participants after their ranges (spin-waits on
// the other CTAs of the grid: only when no concurrent kernel can hold SMs indefinitely —
// false in the two-stream mode, where the last arriving CTA reduces alone).
int swab_pick_bnt(int64_t M);
bool swab_prefer(int64_t M, int64_t N, int num_sms);  // automatic kernel choice
bool swab_prefer_k(int64_t M, int64_t N, int64_t K, int num_sms);  // + long-K rule (the engine's choice)
int swab_grid(int64_t M, int64_t N, int64_t K, int bnt, int num_sms);
int gemm_swab_run(const CUtensorMap& tw, const CUtensorMap& tt, int bnt, int64_t M, int64_t N, int64_t K, int epi,
                  void* C, int64_t ldc, const float* bias, int num_sms, cudaStream_t st, float* part, int* counters,
                  int64_t part_floats, int max_tiles, int a_row0, const QkvRopeArgs* rope, bool coop = true);

// ------------------------------------------------------------------ synthetic generator (gen.cu)
enum GenKind { GEN_LINEAR = 0, GEN_EMBED = 1, GEN_NORM = 2, GEN_BIAS = 3 };
uint64_t fnv1a64(const char* s);
// dst[r * dst_ld + c] = gen(name, (row0 + r) * src_cols + col0 + c) for r < rows, c < cols
cudaError_t gen_fill_bf16(void* dst, int64_t dst_ld, int64_t rows, int64_t cols, uint64_t seed, uint64_t name_hash,
                          int64_t row0, int64_t col0, int64_t src_cols, int kind, int fan_in, cudaStream_t st);
cudaError_t gen_fill_bf16_ex(void* dst, int64_t dst_ld, int64_t rows, int64_t cols, uint64_t seed, uint64_t name_hash,
                             int64_t row0, int64_t col0, int64_t src_cols, int kind, int fan_in, int interleave,
                             cudaStream_t st);
cudaError_t gen_fill_f32_bias(float* dst, int64_t n, uint64_t seed, uint64_t name_hash, int64_t off, cudaStream_t st);
// KV fill: positions [0, n) of one request, one layer, K (bf16) or V (fp16 = 1) plane
cudaError_t kvfill_launch(void* plane, const int32_t* d_table, int n_tokens, int hkv_local, int hkv_global,
                          int kv_head0, int hd, uint64_t seed, uint64_t name_hash, int fp16, cudaStream_t st);

// ------------------------------------------------------------------ elementwise (elementwise.cu)
cudaError_t launch_token_patch(int32_t* dst, const int32_t* src, int n, int vocab, cudaStream_t st);
cudaError_t launch_embed_rmsnorm(const int32_t* tokens, const void* emb, const void* g, float* resid, void* out,
                                 int T, int d, float eps, cudaStream_t st);
cudaError_t launch_rmsnorm(const float* x, const void* g, void* out, int T, int d, float eps, cudaStream_t st);
cudaError_t launch_gather_rmsnorm(const float* x, const int32_t* rows, const void* g, void* out, int R, int d,
                                  float eps, cudaStream_t st);
// copy rows between host-layout [n][Hkv][hd] buffers and the paged plane (positions pos0..)
cudaError_t launch_kv_scatter(void* plane, const int32_t* d_table_row, int pos0, int n, int Hkv, int hd,
                              const void* src, cudaStream_t st);
cudaError_t launch_kv_gather(const void* plane, const int32_t* d_table_row, int pos0, int n, int Hkv, int hd, void* dst,
                             cudaStream_t st);
// apply block-table updates: triples (row, col, block)
cudaError_t launch_table_update(int32_t* tables, int table_w, const int32_t* triples, int n, cudaStream_t st);
// tp > 1: resid += add (bf16 all-reduced partial); out = RMSNorm(resid) * g  (out may alias add)
cudaError_t launch_add_rmsnorm(float* resid, const void* add, const void* g, void* out, int T, int d, float eps,
                               cudaStream_t st);
cudaError_t launch_add_f32(float* resid, const void* add_bf16, size_t n, cudaStream_t st);
// [tp][R][Vl] -> [R][tp*Vl]
cudaError_t launch_unshard_logits(const float* in, float* out, int R, int Vl, int tp, cudaStream_t st);
// in-process peer group (tp > 1 without NCCL): pointers to every rank's buffer, rank order
constexpr int kMaxPeers = 8;
struct PeerPtrs {
  const void* p[kMaxPeers];
};
// resid += sum_k parts[k] (bf16, fp32 sum in rank order); out = RMSNorm(resid) * g if g != NULL
cudaError_t launch_peer_add_rmsnorm(const PeerPtrs& parts, int tp, float* resid, const void* g, void* out, int T, int d,
                                    float eps, cudaStream_t st);
// two-shot: rank `rank` reduces rows [row0, row0+nrows) into its residual, normalises them and
// stores the bf16 rows into every rank's h (hs); g == NULL: stores the fp32 residual rows into
// every rank's residual (resids) instead
cudaError_t launch_peer_rs_norm_ag(const PeerPtrs& parts, const PeerPtrs& hs, const PeerPtrs& resids, int tp, int rank,
                                   int row0, int nrows, const void* g, int d, float eps, cudaStream_t st);
// out[R][tp*Vl] <- rank k's [R][Vl] slice
cudaError_t launch_peer_gather_logits(const PeerPtrs& loc, int tp, int R, int Vl, float* out, cudaStream_t st);
constexpr int kArgmaxMaxSlices = 8;
// part: [R][kArgmaxMaxSlices] scratch, cnt: [R] zero-initialised counters (NULL: one CTA per row)
cudaError_t launch_argmax(const void* logits, int logits_f32, int R, int V, int32_t* out, cudaStream_t st,
                          float2* part = nullptr, int* cnt = nullptr);
cudaError_t launch_f32_to_bf16(const float* x, void* y, int64_t n, cudaStream_t st);

// ------------------------------------------------------------------ attention (attention.cu)
struct DecodeItem {      // one split-K work item: (decode row, kv head, key range)
  int32_t row;           // token row in the batch (q / out row)
  int32_t table;         // block-table row (device) of the request
  int32_t kv_head;       // local kv head
  int32_t key0, key1;    // key range [key0, key1)
  int32_t part;          // partial slot of this item
  int32_t part_base;     // first partial slot of this (row, kv head); its splits follow
  int32_t nsplit;        // splits of this (row, kv head); 1 = no partial, store directly
  int32_t counter;       // arrival counter of this (row, kv head) for the fused combine
};
struct PrefillItem {     // one (chunk, q-tile, kv head) work item
  int32_t row0;          // first token row of the tile
  int32_t npos;          // positions in this tile
  int32_t pos0;          // absolute position of row0
  int32_t table;         // block-table row
  int32_t kv_head;
  int32_t pad;           // 1: duplicate that fills a CTA's group of q tiles (computes, stores nothing)
  int32_t grp_last;      // last position over the q tiles one CTA processes together (their
                         // key-tile count and the block clamp of the shared K/V tiles)
};
struct AttnLaunch {
  const void* q;          // [T][H][hd] bf16, row stride q_ld (elements)
  int q_ld;
  void* out;              // [T][H][hd] (bf16 or f32), row stride out_ld
  int out_ld;
  int out_f32;
  const CUtensorMap* kv_tmap;  // 3D map over the KV pool (host copy; passed by value)
  int layer;
  int H, Hkv, hd;
  int num_blocks;
  const int32_t* tables;  // [max_requests][table_w]
  int table_w;
  float scale_log2;       // log2(e) / sqrt(hd)
  int q_tiles = 1;        // prefill: q tiles per CTA sharing every K/V tile (1 or 2)
  int decode_stages = 8;  // decode: K/V ring depth in (block, head) tiles (8 or 4)
  int decode_persist = 0; // decode: persistent CTAs looping over the item list (ring depth 8)
  const int32_t* cta_off = nullptr;  // prefill, persistent mode: CTA c runs items [cta_off[c], cta_off[c+1])
  const CUtensorMap* q_tmap = nullptr;  // prefill, persistent mode: 3-D map {hd, H, rows} over q with a
                                        // {64, H/Hkv, 128/(H/Hkv)} box (NULL: built per launch)
  int q_rows = 0;                       // rows the q map covers (its dim 2)
  int n_cta = 0;                        // persistent modes: CTAs (pair mode: CTA pairs)
  int pair = 0;                         // prefill: CTA-pair kernel (cta_group::2; q_tiles 2, hd 128)
  const CUtensorMap* kv_tmap5 = nullptr;  // prefill, persistent: 5-D map, 4-block boxes (make_tmap_kv5)
};
int prefill_pair_max_clusters();        // co-resident CTA pairs of the pair kernel (0: unavailable)
cudaError_t launch_decode_attention(const AttnLaunch& a, const DecodeItem* items, int n_items, float* partials,
                                    int* counters, cudaStream_t st);
cudaError_t launch_prefill_attention_tc(const AttnLaunch& a, const PrefillItem* items, int n_items, cudaStream_t st);
int prefill_tc_positions_per_tile(int group);

}  // namespace qos
