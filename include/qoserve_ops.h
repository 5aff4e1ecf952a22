/*
 * qoserve_ops.h — kernel-level entry points of libqoserve.so, one per step of the hybrid
 * iteration (SURVEY.md §8(a) rows a3, a4/a9/a11/a12/a13, a5+a6, a7+a8).  They exist so each
 * row can be checked against the fp64 oracle on inputs the TEST builds on the host (no oracle
 * input ever comes from the CUDA path) and timed on its own.  Same conventions as qoserve.h.
 */
#ifndef QOSERVE_OPS_H_
#define QOSERVE_OPS_H_

#include "qoserve.h"

#ifdef __cplusplus
extern "C" {
#endif

/* GEMM epilogues (a4, a9, a11, a12, a13). */
enum {
  QOS_EPI_STORE_BF16 = 0, /* C bf16 [M][N] = acc                                              */
  QOS_EPI_STORE_F32 = 1,  /* C f32  [M][N] = acc                                              */
  QOS_EPI_BIAS_BF16 = 2,  /* C bf16 [M][N] = acc + bias[n]  (bias: device f32 [N]; Qwen QKV)   */
  QOS_EPI_SILU_GATE = 3,  /* C bf16 [M][N/2]: B rows are gate/up interleaved in groups of 64:  */
                          /*   B rows [128j, 128j+64) = gate rows [64j, 64j+64),               */
                          /*   B rows [128j+64, 128j+128) = up rows [64j, 64j+64);             */
                          /*   C[m][64j+c] = silu(acc[m][128j+c]) * acc[m][128j+64+c]          */
  QOS_EPI_ADD_F32 = 4     /* C f32  [M][N] += acc  (residual-stream accumulate, a9/a12 + a3)  */
};

/* C = epi(A · B^T) with A device bf16 [M][K] row-major (K contiguous), B device bf16 [N][K]
 * row-major (nn.Linear weight layout), fp32 accumulation on tcgen05 tensor cores.
 * Requires K % 64 == 0, N % 32 == 0 (N % 128 == 0 for SILU_GATE), 16-byte aligned rows.
 * M may be any value >= 1.  Stream-ordered. */
int qos_op_gemm(const void* A, const void* B, void* C, int64_t M, int64_t N, int64_t K, int epi,
                const float* bias, void* stream);
/* Same with an explicit kernel choice:
 *   ksplit = 0   automatic (the engine's choice): the weight-streaming kernel when
 *                N % 128 == 0 and M <= 16, or M <= 32 with fewer output tiles of 128 than SMs,
 *                or M <= 256 with fewer than SMs/4 tiles (SMs/2 when K >= 8192) (env
 *                QOS_GEMM_SWAB=0 disables it), else the CTA-pair kernel when N % 256 == 0 and
 *                128 x 256 tiles fill the SMs (env QOS_GEMM_2CTA=0 disables it), else the tile
 *                kernel with the tile width of fewer cost-weighted waves and no split-K (env
 *                QOS_GEMM_SPLITK=1: automatic split-K);
 *   ksplit >= 1  the tile kernel (128-token x 128/256-feature tiles) with that split-K factor:
 *                each of `ksplit` CTAs accumulates a K slice of a tile, parks an fp32 partial,
 *                and the last one to arrive sums the slices in slice order (deterministic);
 *   ksplit <= -2 the tile kernel in stream-K mode: the (tile, k-block) space cut into equal
 *                contiguous ranges, one per CTA; tiles cut by a range boundary are summed from
 *                fp32 partials in CTA order (deterministic).  Never chosen automatically: on
 *                B200 the unaligned ranges lose the L2 reuse of lock-step whole-tile waves
 *                (1.5-1.8x slower at T = 2176, tools/gemm_bench.py).
 *   ksplit = -1  the weight-streaming kernel (requires N % 128 == 0): computes C^T tile by
 *                tile as W_tile(128 rows) · A^T on tcgen05 (token count = UMMA N), the
 *                (tile, k-block) space split in equal contiguous ranges over the SMs
 *                ("stream-K"); tiles cut by a range boundary are summed by their last
 *                arriving CTA in CTA order (deterministic).
 *   ksplit = -3  the CTA-pair kernel (requires N % 256 == 0): clusters of 2 CTAs on 2 SMs,
 *                256 x 256 tiles, UMMA M = 256 (tcgen05 cta_group::2); each CTA stages its
 *                128 rows of A and 128 of the tile's 256 rows of B, no split-K. */
int qos_op_gemm_ex(const void* A, const void* B, void* C, int64_t M, int64_t N, int64_t K, int epi,
                   const float* bias, int ksplit, void* stream);

/* a3: out[t][:] = bf16( x[t][:] / sqrt(mean(x[t]^2) + eps) * g[:] ), x device f32 [T][d],
 * g device bf16 [d], out device bf16 [T][d].  Stream-ordered. */
int qos_op_rmsnorm(const float* x, const void* g, void* out, int32_t T, int32_t d, float eps,
                   void* stream);

/* Write / read cached K and V of `req` at `layer`, positions [pos0, pos0+n), as host 16-bit
 * patterns [n][Hkv_local][hd] (Hkv_local = this rank's kv heads): K in bf16, V in IEEE fp16
 * (the cache keeps V in fp16 so P.V runs as one fp16 MMA; reading r-v16).  The
 * blocks must be allocated.  qos_kv_write does not change the cached length.  Synchronous. */
int qos_kv_write(qos_engine_t* eng, int32_t layer, int64_t req, int32_t pos0, int32_t n,
                 const uint16_t* k_bf16, const uint16_t* v_f16);
int qos_kv_read(qos_engine_t* eng, int32_t layer, int64_t req, int32_t pos0, int32_t n,
                uint16_t* k_bf16, uint16_t* v_f16);

/* a4 + a5 + a6 (fused): the layer's QKV projection of normalised activations h (host bf16
 * [T][d], T = token rows of `batch`, chunks then decodes) with RoPE on q and k at each row's
 * position and k, v appended to the paged cache at `layer` — the epilogue the step uses.
 * q_out: host bf16 [T][H_local * hd] post-RoPE q.  Does not change cached lengths.  Synchronous. */
int qos_op_qkv_rope_append(qos_engine_t* eng, int32_t layer, const qos_batch* batch,
                           const uint16_t* h_bf16, uint16_t* q_out_bf16);

/* a7 + a8: attention of the batch's token rows at `layer` over the paged cache (which must
 * already hold every key the rows attend to: chunk keys 0..kv_start+len-1, decode keys
 * 0..ctx_len).  q: host bf16 [T][H_local][hd] (post-RoPE); out: host f32 [T][H_local][hd]
 * (the fp32 accumulator before the bf16 store, reading s10).  Synchronous. */
int qos_op_attention(qos_engine_t* eng, int32_t layer, const qos_batch* batch,
                     const uint16_t* q_bf16, float* out_f32);

#ifdef __cplusplus
}
#endif
#endif /* QOSERVE_OPS_H_ */
