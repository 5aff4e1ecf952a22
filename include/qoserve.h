/*
 * qoserve.h — C ABI of libqoserve.so, the B200 (sm_100a) hybrid-batch forward step under the
 * QoServe scheduler (Goel et al., "QoServe: Breaking the Silos of LLM Inference Serving",
 * ASPLOS'26; text in PAPER.md).
 *
 * What one call computes.  QoServe builds each iteration from ALL requests in the decode queue
 * plus prefill chunk(s) taken from deadline-selected prefill requests (§3.1
 * step 1; Algorithm 1 lines 2, 17-20 = PAPER.md:755, 770-773) and dispatches them as ONE fused
 * prefill+decode token batch (PAPER.md:542-545 step 5; §3.3 "fused
 * prefill-decode MLP") to a vLLM engine with tensor parallelism and PagedAttention
 * (§3.6).  Chunk sizes change every iteration at no extra cost
 * (§3.6.1), so the step must reach exactly the result of the plain causal
 * forward for any chunk split (§2.1), and its latency must be predictable
 * from (chunk_len, n_decode, ctx) for the dynamic-chunking predictor (§3.6.1).
 *
 * Model: decoder-only pre-norm transformer, Llama/Qwen2 convention (reading s1-s3 in
 * DESIGN.md §2): RMSNorm, rotate-half RoPE, GQA (kv head = h / (H/Hkv)), SwiGLU, untied LM
 * head, optional QKV bias.  Precision (reading s4): bf16 weights / activations / KV cache,
 * fp32 accumulation, fp32 softmax and norm statistics, fp32 residual stream.
 *
 * Conventions (all calls):
 *   - Return value: QOS_OK (0) or a negative QOS_ERR_*; no exception or abort crosses the ABI.
 *     qos_last_error() returns a thread-local message for the last failing call.
 *   - Pointers are plain host pointers unless documented "device".  Caller-owned inputs are
 *     only read during the call.  The engine owns weights, KV pool, block tables, workspaces
 *     (or borrows caller-provided device arenas, see qos_engine_create).
 *   - `stream` is a cudaStream_t passed as void* (NULL = legacy default stream).
 *   - An engine is single-threaded: calls on one engine must not overlap.
 *   - Under tensor parallelism every rank is called with the same arguments (rank 0's
 *     scheduler broadcasts the descriptor); KV tables are identical on every rank.
 *   - There is no CPU fallback: every compute step runs in this library's sm_100a kernels.
 */
#ifndef QOSERVE_H_
#define QOSERVE_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* ---------------------------------------------------------------- return codes, dtypes */
enum {
  QOS_OK = 0,
  QOS_ERR_INVALID_ARG = -1,   /* bad pointer / shape / descriptor field                    */
  QOS_ERR_OOM = -2,           /* KV pool or device memory exhausted (state unchanged)       */
  QOS_ERR_UNKNOWN_REQ = -3,   /* request id has no KV table                                */
  QOS_ERR_BAD_KV_START = -4,  /* kv_start / ctx_len != the request's cached length         */
  QOS_ERR_NOT_ALLOCATED = -5, /* the step would write past the request's allocated blocks  */
  QOS_ERR_CUDA = -6,          /* CUDA runtime / driver error (message in qos_last_error)   */
  QOS_ERR_COMM = -7,          /* NCCL error or peer-group abort; the communicator is aborted */
  QOS_ERR_UNSUPPORTED = -8    /* shape the kernels do not support (e.g. head_dim != 64/128) */
};

enum { QOS_F32 = 0, QOS_BF16 = 1 };

typedef struct qos_engine qos_engine_t;  /* opaque; one per (process, GPU, TP rank) */

/* ---------------------------------------------------------------- model / engine config */
typedef struct {
  int32_t n_layers, d_model, n_heads, n_kv_heads, head_dim, ffn_dim, vocab;
  float rope_theta, rms_eps;
  int32_t qkv_bias;         /* 1: q/k/v projections carry a bias (Qwen2)                    */
  int32_t block_size;       /* KV block size in tokens; must be 16 (reading s12)             */
  int64_t num_blocks;       /* KV pool size in blocks (per rank)                             */
  int32_t max_seq_len;      /* max tokens per request; block-table width = ceil(/16)         */
  int32_t max_requests;     /* max live requests (block-table rows)                          */
  int32_t max_batch_tokens; /* max T = sum(chunk_len) + n_decode per step                    */
  int32_t max_batch_rows;   /* max R = n_prefill + n_decode per step; max_batch_rows x       */
                            /* n_kv_heads/tp <= 65536 (decode work items; QOS_ERR_UNSUPPORTED) */
} qos_model_cfg;

typedef struct {
  uint64_t weight_bytes;    /* this rank's weight shard                                     */
  uint64_t kv_bytes;        /* KV pool: L x {K,V} x num_blocks x Hkv/tp x 16 x hd x 2 B      */
  uint64_t workspace_bytes; /* activations, metadata, split-K partials for max_batch_tokens  */
} qos_mem_sizes;

typedef struct {            /* optional caller-provided DEVICE arenas (256-byte aligned);    */
  void* weights;            /* any NULL member is cudaMalloc'ed by the engine. Ownership of  */
  void* kv;                 /* provided arenas stays with the caller, who must keep them      */
  void* workspace;          /* alive until qos_engine_destroy.                                */
} qos_mem;

/* Sizes of the three arenas for `cfg` at TP degree `tp_size`. */
int qos_engine_mem_sizes(const qos_model_cfg* cfg, int tp_size, qos_mem_sizes* out);

/* Create an engine on CUDA device `device` for TP rank `tp_rank` of `tp_size`.
 * nccl_uid: the 128-byte ncclUniqueId shared by all ranks (rank 0 creates it with
 * qos_nccl_unique_id and broadcasts it, e.g. over torch.distributed); NULL iff tp_size == 1.
 * Sharding: rank r owns q heads [r*H/tp, (r+1)*H/tp), kv heads
 * [r*Hkv/tp, ...), FFN columns [r*F/tp, ...), the matching rows of o_proj / down_proj, and
 * vocab rows [r*V/tp, ...) of lm_head; embeddings and norms are replicated.
 * Requires tp_size | n_kv_heads, tp_size | n_heads, tp_size | ffn_dim, tp_size | vocab. */
int qos_engine_create(const qos_model_cfg* cfg, int device, int tp_rank, int tp_size,
                      const uint8_t* nccl_uid, const qos_mem* mem, qos_engine_t** out);
int qos_engine_destroy(qos_engine_t* eng);

/* In-process peer group: the alternative to NCCL for tp_size > 1 when all TP ranks of one model
 * live in ONE process (one engine and one host thread per rank, on one GPU or on GPUs with peer
 * access over NVLink/NVSwitch).  The all-reduce after the O and down projections
 * (vLLM TP, §3.6) is then one kernel per rank that reads every
 * rank's bf16 partial straight from its workspace (peer loads), sums in fp32 in rank order (all
 * ranks get bit-identical results) and fuses the residual add and the next RMSNorm
 * (SURVEY.md §8(f) NEXT-2); the vocab-parallel logits are gathered the same way.  Ordering is by
 * CUDA events: at each collective every rank records "partial ready", the host threads meet at a
 * barrier (so every record precedes every wait), and each rank's stream waits on its peers'
 * events — no kernel spins on another rank.
 * Every rank must issue the same sequence of qos_hybrid_step / qos_profile_step calls, from its
 * own thread, concurrently.  A rank that does not reach a collective within
 * QOS_GROUP_TIMEOUT_MS (env, default 120000) aborts the group: the waiting calls return
 * QOS_ERR_COMM and the group stays unusable.
 * qos_group_create: tp_size in 2..8.  qos_group_destroy: after all its engines are destroyed
 * (QOS_ERR_INVALID_ARG otherwise).  qos_engine_create_peer: as qos_engine_create with
 * tp_size = the group's size; the ranks need identical configs; ranks on different devices
 * enable peer access both ways (QOS_ERR_UNSUPPORTED without it); QOS_ERR_INVALID_ARG if the rank
 * is already taken. */
typedef struct qos_group qos_group_t;
int qos_group_create(int tp_size, qos_group_t** out);
int qos_group_destroy(qos_group_t* group);
/* Cross-process form of the peer group: one process (and one engine) per rank on one node, e.g.
 * one process per GPU under torchrun.  Rank 0 calls qos_group_unique_id (a NUL-terminated POSIX
 * shared-memory name in 64 bytes) and broadcasts it (e.g. over torch.distributed); every rank
 * then calls qos_group_open with it (rank 0 creates the segment, the others wait for it up to
 * QOS_GROUP_TIMEOUT_MS) and qos_engine_create_peer with tp_rank = its group rank.  Engine
 * creation and destruction are collective: each rank exports its workspace (CUDA IPC memory
 * handle) and its two sync events (interprocess events) and maps its peers'; the barrier is a
 * spin barrier in the segment.  Collectives, ordering, abort and results are as above.  The
 * segment is unlinked when the last rank destroys its group. */
int qos_group_unique_id(uint8_t out[64]);
int qos_group_open(const uint8_t id[64], int tp_size, int tp_rank, qos_group_t** out);
int qos_engine_create_peer(const qos_model_cfg* cfg, int device, int tp_rank, qos_group_t* group,
                           const qos_mem* mem, qos_engine_t** out);

/* This rank's slice under tensor parallelism (pure host function):
 * q heads [head0, head0+n_heads), kv heads [kv_head0, +n_kv_heads), FFN columns
 * [ffn0, +ffn), vocab rows [vocab0, +vocab) of lm_head.  o_proj / down_proj take the matching
 * input columns; their partial outputs are summed by the all-reduce. */
typedef struct {
  int32_t n_heads, n_kv_heads, ffn, vocab;
  int32_t head0, kv_head0, ffn0, vocab0;
} qos_shard;
int qos_shard_plan(const qos_model_cfg* cfg, int tp_rank, int tp_size, qos_shard* out);

/* 128-byte ncclUniqueId for tp_size > 1 (call on rank 0 only). */
int qos_nccl_unique_id(uint8_t out[128]);

/* Fill this rank's weight shard with the synthetic generator of DESIGN.md §3:
 * w = bf16_rne(f(a)), a = ((splitmix64((seed ^ fnv1a64(name)) + i) >> 40) - 2^23) / 2^23,
 * i the flat row-major index in the Hugging Face tensor `name`; f per kind (linear:
 * a * fp32(1/sqrt(fan_in)); embed: a; norm: 1 + 0.1 a; bias: 0.02 a).  Synchronous. */
int qos_engine_load_synthetic(qos_engine_t* eng, uint64_t seed);

/* Copy rows [row0, row0+nrows) of this rank's shard of HF tensor `name` (e.g.
 * "model.layers.3.mlp.up_proj.weight", shard-local row numbering) to host bf16 bits. */
int qos_engine_read_weight(qos_engine_t* eng, const char* name, int64_t row0, int64_t nrows,
                           uint16_t* out_bf16);

/* ---------------------------------------------------------------- paged KV (a6 storage, D7) */
/* Grow req's block table to ceil(n_tokens_total / 16) blocks, taking the lowest free block
 * indices in ascending order (reading s12).  All-or-nothing: QOS_ERR_OOM leaves every table
 * unchanged.  Never shrinks.  The device copy of the table row is updated stream-ordered on
 * the engine's internal stream before the next step.  KV is held only while needed
 * (§3.4). */
int qos_kv_alloc(qos_engine_t* eng, int64_t req, int32_t n_tokens_total);
/* Release all of req's blocks (QOS_ERR_UNKNOWN_REQ if it has none).  The blocks and the table
 * row are reusable at once on the host side.  Ordering: the engine's own device work (KV fills,
 * table flushes, op entry points) waits for the last step enqueued through qos_hybrid_step; a
 * later qos_hybrid_step on ANOTHER caller stream is not ordered after an in-flight step that
 * read the freed blocks -- use one stream for steps, or synchronise before reusing them. */
int qos_kv_free(qos_engine_t* eng, int64_t req);
/* Inspect req's table: writes min(cap, n) block ids to out, n to *n_out. */
int qos_kv_table(qos_engine_t* eng, int64_t req, int32_t* out, int32_t cap, int32_t* n_out);
/* Same, read back from the DEVICE copy of the table (flushes pending updates; synchronous). */
int qos_kv_table_device(qos_engine_t* eng, int64_t req, int32_t* out, int32_t cap, int32_t* n_out);
/* Tokens of req already in the cache (what the next kv_start / ctx_len must equal). */
int qos_kv_cached_len(qos_engine_t* eng, int64_t req, int32_t* out);
/* Number of free blocks. */
int qos_kv_free_blocks(qos_engine_t* eng, int64_t* out);
/* Fill positions [0, n_tokens) of req, every layer, with synthetic K/V (DESIGN.md §3:
 * name "kvfill.{layer}.{k|v}.{req}", i = (pos*Hkv + h)*hd + j over GLOBAL kv heads, value
 * bf16_rne(a) for K, fp16_rne(a) for V) and set its cached length to n_tokens.  Used by benches / profiling where
 * a decode's prefix need not come from a prefill.  Synchronous. */
int qos_kv_fill_synthetic(qos_engine_t* eng, int64_t req, int32_t n_tokens, uint64_t seed);

/* ---------------------------------------------------------------- the hybrid step (a1..a14) */
typedef struct {
  int64_t req;
  int32_t kv_start;        /* == cached length of req (strict append, no recompute)          */
  int32_t chunk_len;       /* >= 1 prefill tokens at positions kv_start .. kv_start+len-1    */
  const int32_t* tokens;   /* host, [chunk_len] token ids in [0, vocab)                      */
} qos_prefill_chunk;

typedef struct {
  int64_t req;
  int32_t ctx_len;         /* cached tokens; the new token sits at position ctx_len and     */
  int32_t token;           /* attends ctx_len + 1 keys (reading s7)                          */
} qos_decode;

typedef struct {
  int32_t n_prefill;
  const qos_prefill_chunk* prefill;  /* host array [n_prefill]; distinct requests            */
  int32_t n_decode;
  const qos_decode* decode;          /* host array [n_decode]; distinct from the chunks'     */
} qos_batch;

/* One hybrid-batch forward iteration.
 * Rows of the outputs: one per chunk (its LAST token, reading s8) in descriptor order, then one
 * per decode in descriptor order; R = n_prefill + n_decode.
 *   logits      : [R][vocab] of logits_dtype (QOS_F32 | QOS_BF16), or NULL;
 *   next_tokens : [R] int32 greedy argmax (lowest index on ties), or NULL;
 *   outputs_on_host = 0: both are DEVICE pointers and the call is stream-ordered/asynchronous;
 *   outputs_on_host = 1: both are HOST pointers; the call copies them back and synchronises.
 * Effects: appends the K/V of every processed token to the paged cache and advances the
 * requests' cached lengths by chunk_len / 1.  Errors are detected before any device work
 * (INVALID_ARG, UNKNOWN_REQ, BAD_KV_START, NOT_ALLOCATED); state is then unchanged. */
int qos_hybrid_step(qos_engine_t* eng, const qos_batch* batch, void* logits, int logits_dtype,
                    int32_t* next_tokens, int outputs_on_host, void* stream);
/* The same, with the decodes' input tokens read from DEVICE memory when the step runs:
 * decode_tokens_dev[i] (int32, device, >= n_decode entries) replaces batch->decode[i].token, so
 * a serving loop can feed one step's next_tokens (device, e.g. next_tokens + n_prefill of the
 * previous step when the decode set keeps its order) into the next step and build / enqueue
 * that step on the host while the previous one still runs (chunk sizes change
 * every iteration "at no additional cost").  Stream-ordered: the read happens on `stream` after
 * the work already enqueued there.  Values are clamped to [0, vocab) (the engine's argmax output
 * always is in range); the descriptor's decode tokens are still range-checked on the host.
 * decode_tokens_dev = NULL: exactly qos_hybrid_step. */
int qos_hybrid_step_ex(qos_engine_t* eng, const qos_batch* batch, void* logits, int logits_dtype,
                       int32_t* next_tokens, int outputs_on_host, void* stream, const int32_t* decode_tokens_dev);

/* Device-timed latency of one synthetic step for the scheduler's iteration-time model
 * (replaces the paper's Vidur-profiled random forest, §3.6.1): a chunk of
 * chunk_len tokens at kv_start 0 plus n_decode decodes with contexts ctx_lens[j] (host), on
 * scratch requests with synthetic KV.  Runs 3 warm-up steps, then `reps` steps each timed with
 * CUDA events on the engine stream; *ms_out = median.  Synchronous; scratch KV is freed. */
int qos_profile_step(qos_engine_t* eng, int32_t chunk_len, int32_t n_decode,
                     const int32_t* ctx_lens, int32_t reps, float* ms_out);
/* Same with an explicit chunk kv_start (prefix already cached), warm-up step count and p95
 * output (`warmup` < 0 selects the default of 3). */
int qos_profile_step_ex(qos_engine_t* eng, int32_t chunk_len, int32_t kv_start,
                        int32_t n_decode, const int32_t* ctx_lens, int32_t warmup, int32_t reps,
                        float* ms_median, float* ms_p95);

/* Execution options (defaults in parentheses; the QOS_* environment variables of the same
 * meaning set the defaults at engine creation):
 *   "overlap_attn" (1)     run prefill attention on a high-priority side stream concurrently
 *                          with the decode attention of the same layer
 *   "gemm_splitk" (0)      split-K of the tile GEMM for weight-bound small-M projections (off:
 *                          slower at every shape the engine gives the tile kernel — the QKV
 *                          GEMM at T 33..128 takes 26 us split vs 17 us unsplit; the weight-
 *                          streaming kernel covers the small-T O and down projections)
 *   "dual_stream" (0)      prefill rows and decode rows as two sub-batches on two streams
 *                          (measured slower on B200; kept for experiments), with
 *                          "dual_min_prefill" (512), "dual_min_decode" (16),
 *                          "dual_sms_prefill" / "dual_sms_decode" (0 = all SMs)
 *   "gemm_swab" (1)        weight-streaming swap-AB GEMM for small token counts: 0 never,
 *                          1 automatic (small T, or T <= 256 with few output tiles), 2 always
 *                          (where N % 128 == 0); env QOS_GEMM_SWAB
 *   "gemm_streamk" (0)     stream-K mode of the tile GEMM: 0 never, 1 when whole-tile waves
 *                          leave > 5% of the last wave idle, 2 always (experiments; slower on
 *                          B200 at large T: ranges out of phase lose L2 reuse); env QOS_GEMM_STREAMK
 *   "pdl" (1)              programmatic dependent launch of the step's kernel chain (each
 *                          kernel's prologue and weight prefetch overlap the previous kernel's
 *                          tail); process-wide, env QOS_PDL
 *   "decode_round_split" (1) decode split-K ranges: the key blocks of a decode in a rounded
 *                          number of near-equal block-aligned ranges (0: fixed 64..512-key
 *                          ranges with a short last one)
 *   "decode_split" (4096)  decode split-K: the longest key range tried first (power of two,
 *                          64..65536); halved while the step has fewer than 4 items per SM
 *   "fa_poly" (4)          prefill attention: every n-th exp2 pair on the FMA pipe by a
 *                          polynomial, the rest on MUFU (0 = all MUFU; -1 = measurement-only
 *                          variant without the softmax, results invalid); process-wide,
 *                          env QOS_FA_POLY
 *   "fa_qtiles" (1)        prefill attention: q tiles (128 rows each) per CTA sharing every
 *                          K/V tile (1: two CTAs per SM with 2-deep K/V rings; 2: one CTA per
 *                          SM, half the L2 -> SM traffic, 4-deep rings; measured ~6% more
 *                          cycles than 1, tools/ncu_ab.py)
 *   "tp_twoshot" (-1)      peer-group TP reduction: 0 one-shot (every rank reads all partials of
 *                          all rows), 1 two-shot (each rank reduces + normalises a row slice and
 *                          stores it into every peer: ~2(tp-1)/tp of one partial per rank instead
 *                          of tp-1), -1 automatic (two-shot when tp >= 4)
 *   "attn_order" (0)       with overlap_attn: 0 prefill attention first on a high-priority side
 *                          stream; 1 decode first, prefill on a normal-priority side stream; 2
 *                          decode first, prefill high priority (measured equal within noise)
 *   "tp_scatter" (1)       peer-group two-shot reduction with the reduce-scatter fused into the O /
 *                          down GEMM epilogue: each partial row is stored straight into its owner
 *                          rank's receive slot (peer memory) while the remaining tiles compute
 *                          (one-pass tile kernels only; else the reducer reads the peers' partials)
 *   "fa_persist" (1)       prefill attention (fa_qtiles 1) as persistent CTAs, 2 per SM, each
 *                          running a host-dealt list of work items back to back (LPT greedy by
 *                          key tiles); the next item's Q is staged under the current epilogue
 *                          (0: one CTA per work item)
 *   "gemm_2cta" (1)        CTA-pair GEMM (tcgen05 cta_group::2, 256 x 256 tiles) where it
 *                          needs no more waves than 128 x 256 single-CTA tiles; env QOS_GEMM_2CTA
 *   "add_split" (1)        ordered in-place split-K of the residual-add projections below the
 *                          norm-fold threshold (down projection at mid T; slices add in a fixed
 *                          order, so results stay deterministic); env QOS_ADD_SPLIT
 *   "gemm_sms" (0)         SM budget of the step's GEMM grids (0 = all; experiments)
 *   "swab_gran" (-1)       weight-streaming GEMM range granule in k-blocks (-1 automatic, 0 whole
 *                          tiles); process-wide, experiments (profiles/step_swabgran_r2a.jsonl:
 *                          the automatic granule is best in-step)
 *   "gemm_bn" (0)          force the tile width (128 / 256) of the QKV and gate/up tile GEMMs
 *                          (0 = the wave-cost choice; experiments: in-step A/B in
 *                          profiles/step_bn_r2a.jsonl found the automatic choice best)
 *   "shares_device" (0)    1: another engine may run kernels concurrently on this GPU (e.g. two
 *                          engines on two streams of one process).  Switches off the GEMM paths
 *                          that need every CTA of a grid resident at once (the weight-streaming
 *                          kernel's cooperative reduction, the ordered split-K): two such grids
 *                          sharing the SMs could each wait on CTAs the other keeps out.  Set
 *                          automatically for peer-group ranks on one device.
 *   "fa_tma5" (1)          prefill attention (persistent): a K/V tile whose 4 paged blocks have
 *                          consecutive ids is loaded as one 5-D TMA box per 64-dim half;
 *                          process-wide
 *   "fa_psplit" (1)        prefill attention (persistent): P released to the P.V MMAs in two
 *                          halves of 32 keys; process-wide
 *   "fa_kvfirst" (0)       prefill attention (persistent): an item's first K/V tile issued before
 *                          its Q (measured neutral); process-wide
 *   "fa_item_cost" (2)     per-item overhead, in key tiles, of the host's LPT dealing of prefill
 *                          items to persistent CTAs (measured insensitive)
 *   "fa_pair" (0)          prefill attention on CTA pairs (tcgen05 cta_group::2, each CTA staging
 *                          half of every K and V tile; hd 128; measured 30-40% slower)
 *   "decode_persist" (0)   decode attention as persistent CTAs looping over the item list
 *                          (measured slower at small steps, equal at the bench step)
 *   "decode_items_per_sm" (4)  split decode key ranges until the work list has this many items
 *                          per SM; 0: 1 per SM when decodes average < 3072 keys (faster small
 *                          steps; its latency-model fit is not validated), else 4
 *   "gemm2_rel_cluster" (0) CTA-pair GEMM accumulator release with .release.cluster instead of
 *                          the default CTA-scope remote arrive (experiment); process-wide
 * Results do not depend on the options (parity tests run with the defaults and variants). */
int qos_engine_set_option(qos_engine_t* eng, const char* name, int64_t value);

/* ---------------------------------------------------------------- per-kernel timing (a15) */
enum {
  QOS_T_META = 0, QOS_T_EMBED, QOS_T_NORM, QOS_T_GEMM_QKV, QOS_T_ROPE_APPEND, QOS_T_PREFILL_ATTN,
  QOS_T_DECODE_ATTN, QOS_T_GEMM_O, QOS_T_GEMM_GATEUP, QOS_T_GEMM_DOWN, QOS_T_ALLREDUCE,
  QOS_T_HEAD, QOS_T_ARGMAX, QOS_T_COUNT
};
/* When enabled, every kernel class of each step is bracketed by CUDA events on the step's
 * stream (no host synchronisation).  qos_last_step_timing returns the per-class summed device
 * ms and bracket counts of all steps since timing was enabled or since its previous call, and
 * resets the accumulation (it synchronises on the last recorded event). */
int qos_engine_set_timing(qos_engine_t* eng, int enable);
int qos_last_step_timing(qos_engine_t* eng, float ms[QOS_T_COUNT], int32_t launches[QOS_T_COUNT]);
/* Host->device bytes (descriptor metadata + table updates) and device->host bytes (outputs
 * when outputs_on_host) moved by the last qos_hybrid_step. */
int qos_last_step_io(qos_engine_t* eng, int64_t* h2d_bytes, int64_t* d2h_bytes);
/* Total kernel launches issued by this library in this process (the bench's gpu_launches). */
int qos_engine_launch_count(qos_engine_t* eng, int64_t* out);

const char* qos_strerror(int code);
const char* qos_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* QOSERVE_H_ */
