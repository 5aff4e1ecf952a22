// engine.cu — host runtime of libqoserve.so: the C ABI of include/qoserve.h and
// include/qoserve_ops.h.  Owns the weight shard, the paged KV pool with its deterministic block
// allocator and device-resident block tables, the step workspaces, and the per-step metadata
// builder that turns a QoServe batch descriptor (all decodes + the
// deadline-selected prefill chunks, Alg. 1) into the kernels' work lists.
#include <dlfcn.h>
#include <fcntl.h>
#include <sched.h>
#include <sys/mman.h>
#include <sys/stat.h>
#include <unistd.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cmath>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>
#include <condition_variable>
#include <queue>
#include <string>
#include <unordered_map>
#include <unordered_set>
#include <array>
#include <random>
#include <vector>
#include <memory>

#include "internal.h"
#include <cuda_bf16.h>
#include <nccl.h>

namespace qos {

static thread_local std::string g_last_error;
static std::atomic<int64_t> g_launches{0};
// QOS_SKIP_NORM=1: measurement only (results invalid): skips the per-layer RMSNorm launches to
// price them inside the step
static const bool g_skip_norm = getenv("QOS_SKIP_NORM") && atoi(getenv("QOS_SKIP_NORM")) != 0;

int set_error(int code, const char* msg) {
  g_last_error = msg ? msg : "";
  return code;
}
int set_cuda_error(cudaError_t e, const char* where) {
  g_last_error = std::string(where) + ": " + cudaGetErrorString(e);
  return QOS_ERR_CUDA;
}
int count_launch(int n) {
  g_launches.fetch_add(n, std::memory_order_relaxed);
  return 0;
}

#define QOS_CU(call)                                                   \
  do {                                                                 \
    cudaError_t _e = (call);                                           \
    if (_e != cudaSuccess) return set_cuda_error(_e, #call);           \
  } while (0)
#define QOS_TRY(call)             \
  do {                            \
    int _r = (call);              \
    if (_r != QOS_OK) return _r;  \
  } while (0)

static inline size_t align_up(size_t x, size_t a) { return (x + a - 1) / a * a; }

// ------------------------------------------------------------------ NCCL (dlopen'ed)
struct Nccl {
  void* so = nullptr;
  decltype(&ncclGetUniqueId) getUniqueId = nullptr;
  decltype(&ncclCommInitRank) commInitRank = nullptr;
  decltype(&ncclCommDestroy) commDestroy = nullptr;
  decltype(&ncclCommAbort) commAbort = nullptr;
  decltype(&ncclAllReduce) allReduce = nullptr;
  decltype(&ncclAllGather) allGather = nullptr;
  decltype(&ncclGetErrorString) errStr = nullptr;
  bool load() {
    if (so) return true;
    const char* names[] = {"libnccl.so.2", "libnccl.so"};
    for (const char* n : names) {
      so = dlopen(n, RTLD_NOW | RTLD_GLOBAL);
      if (so) break;
    }
    if (!so) return false;
    getUniqueId = (decltype(getUniqueId))dlsym(so, "ncclGetUniqueId");
    commInitRank = (decltype(commInitRank))dlsym(so, "ncclCommInitRank");
    commDestroy = (decltype(commDestroy))dlsym(so, "ncclCommDestroy");
    commAbort = (decltype(commAbort))dlsym(so, "ncclCommAbort");
    allReduce = (decltype(allReduce))dlsym(so, "ncclAllReduce");
    allGather = (decltype(allGather))dlsym(so, "ncclAllGather");
    errStr = (decltype(errStr))dlsym(so, "ncclGetErrorString");
    return getUniqueId && commInitRank && commDestroy && allReduce && allGather;
  }
};
static Nccl g_nccl;
static std::mutex g_nccl_mu;

// ------------------------------------------------------------------ shapes / sharding
struct Shard {
  int H, Hkv, F, V;       // local counts
  int h0, kv0, f0, v0;    // first global index owned
};
static Shard make_shard(const qos_model_cfg& c, int rank, int tp) {
  Shard s;
  s.H = c.n_heads / tp;
  s.Hkv = c.n_kv_heads / tp;
  s.F = c.ffn_dim / tp;
  s.V = c.vocab / tp;
  s.h0 = rank * s.H;
  s.kv0 = rank * s.Hkv;
  s.f0 = rank * s.F;
  s.v0 = rank * s.V;
  return s;
}

struct WeightLayout {   // byte offsets inside the weight arena
  struct L {
    size_t ln1, ln2, wqkv, bqkv, wo, wgu, wd;
  };
  std::vector<L> layers;
  size_t emb, lnf, head, total;
};
static WeightLayout weight_layout(const qos_model_cfg& c, const Shard& s) {
  WeightLayout w;
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = align_up(off + bytes, 256);
    return o;
  };
  const size_t d = c.d_model, hd = c.head_dim;
  const size_t nqkv = (size_t(s.H) + 2 * s.Hkv) * hd;
  for (int l = 0; l < c.n_layers; ++l) {
    WeightLayout::L L;
    L.ln1 = take(d * 2);
    L.ln2 = take(d * 2);
    L.wqkv = take(nqkv * d * 2);
    L.bqkv = c.qkv_bias ? take(nqkv * 4) : 0;
    L.wo = take(d * size_t(s.H) * hd * 2);
    L.wgu = take(2 * size_t(s.F) * d * 2);
    L.wd = take(d * size_t(s.F) * 2);
    w.layers.push_back(L);
  }
  w.emb = take(size_t(c.vocab) * d * 2);
  w.lnf = take(d * 2);
  w.head = take(size_t(s.V) * d * 2);
  w.total = off;
  return w;
}

struct WsLayout {
  size_t resid, h, qkv, attn, act, hR, logits, logits_loc, part[2], recv[2], ss[2], rs[2], fcnt, am_part, am_cnt, argmax, partials, counters, gemm_part, gemm_cnt, gemm_part2,
      gemm_cnt2, meta[2], dbg, total;
  size_t meta_bytes;
  int max_items;
};
static constexpr int kMaxDecodeItems = 1 << 16;
static constexpr int kGemmMaxUnits = 512;   // split-K partial slots (128 x 256 fp32 each)
static constexpr int kGemmMaxTiles = 4096;  // split-K arrival counters
static WsLayout ws_layout(const qos_model_cfg& c, const Shard& s, int tp) {
  WsLayout w;
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = align_up(off + bytes, 1024);
    return o;
  };
  const size_t Tm = c.max_batch_tokens, Rm = c.max_batch_rows, d = c.d_model, hd = c.head_dim;
  const size_t nqkv = (size_t(s.H) + 2 * s.Hkv) * hd;
  const size_t group = c.n_heads / c.n_kv_heads;
  w.resid = take(Tm * d * 4);
  w.h = take(Tm * d * 2);
  w.qkv = take(Tm * nqkv * 2);
  w.attn = take(Tm * size_t(s.H) * hd * 2);
  w.act = take(Tm * size_t(s.F) * 2);
  w.hR = take(Rm * d * 2);
  w.logits = take(Rm * size_t(c.vocab) * 4);
  w.logits_loc = tp > 1 ? take(Rm * size_t(c.vocab) * 4) : 0;
  // peer-group TP: the O / down partials, double-buffered by collective parity (read by the peers)
  w.ss[0] = take(Tm * kFoldSlots * 4);  // folded RMSNorm: per-row sums of squares per 128 columns
  w.ss[1] = take(Tm * kFoldSlots * 4);
  w.rs[0] = take(Tm * 4);
  w.rs[1] = take(Tm * 4);
  w.fcnt = take((Tm / 128 + 2) * 4);
  // peer-group reduce-scatter: receive slots [tp][ceil(Tm/tp)][d] bf16, by collective parity
  const size_t rs_max = (Tm + size_t(tp) - 1) / size_t(tp);
  w.recv[0] = tp > 1 ? take(size_t(tp) * rs_max * d * 2) : 0;
  w.recv[1] = tp > 1 ? take(size_t(tp) * rs_max * d * 2) : 0;
  w.part[0] = tp > 1 ? take(Tm * d * 2) : 0;
  w.part[1] = tp > 1 ? take(Tm * d * 2) : 0;
  w.argmax = take(Rm * 4);
  w.am_part = take(Rm * kArgmaxMaxSlices * 8);
  w.am_cnt = take(Rm * 4);
  w.max_items = kMaxDecodeItems;
  w.partials = take(size_t(w.max_items) * group * (hd + 2) * 4);
  w.counters = take(Rm * size_t(s.Hkv) * 4);
  w.gemm_part = take(size_t(kGemmMaxUnits) * 128 * 256 * 4);
  w.gemm_cnt = take(size_t(kGemmMaxTiles) * 4);
  w.gemm_part2 = take(size_t(kGemmMaxUnits) * 128 * 256 * 4);   // second stream's split-K workspace
  w.gemm_cnt2 = take(size_t(kGemmMaxTiles) * 4);
  // metadata: tokens, pos, slot [Tm]; logit rows [Rm]; prefill items; decode items/rows; table updates
  const int ppt = prefill_tc_positions_per_tile(int(group));
  // (+ up to 3 group-filling duplicates per (chunk, kv head))
  const size_t max_pitems = (Tm / ppt + 4 * (Rm + 1)) * size_t(s.Hkv);
  w.meta_bytes = align_up(3 * Tm * 4 + Rm * 4 + 64, 256) + align_up(max_pitems * sizeof(PrefillItem), 256) +
                 align_up(size_t(w.max_items) * sizeof(DecodeItem), 256) +
                 align_up(size_t(3) * 65536 * 4, 256) + align_up(1025 * 4, 256);  // + persistent CTA offsets
  w.meta[0] = take(w.meta_bytes);
  w.meta[1] = take(w.meta_bytes);
  w.dbg = 0;
  w.total = off;
  return w;
}

// ------------------------------------------------------------------ batch metadata (a1)
struct StepMeta {
  int T = 0, R = 0, n_prefill = 0, n_decode = 0;
  int n_pitems = 0, n_ditems = 0, n_upd = 0;
  int fa_qtiles = 1;  // prefill items come in groups of this many q tiles (one CTA each group)
  int fa_pair = 0;    // prefill attention on CTA pairs (groups of 2 q tiles; n_pcta = pairs)
  int n_pcta = 0;     // persistent prefill attention: CTAs (0: one CTA per item group)
  size_t o_pcta = 0;  // offsets [n_pcta + 1] into the prefill items
  // offsets (bytes) inside the metadata block
  size_t o_tok, o_pos, o_slot, o_rows, o_pitems, o_ditems, o_upd, used;
};

struct ReqState {
  int row = -1;                 // block-table row
  std::vector<int32_t> blocks;  // physical block ids
  int cached = 0;               // tokens in cache
};

}  // namespace qos

using namespace qos;

// In-process peer group (qos_group_create / qos_engine_create_peer): the TP ranks of one model
// as engines of ONE process — one host thread per rank, on one GPU or on peer GPUs — whose
// collectives are stream-event-ordered peer-memory kernels instead of NCCL (SURVEY.md §8(e),
// §8(f) NEXT-2).  The host barrier only orders the ranks' ENQUEUEING at each collective (every
// rank has recorded its "partial ready" event before any rank waits on it); the GPUs never spin.
// Cross-process form (qos_group_open; one process per GPU on one node): the same collectives
// over CUDA IPC — every rank exports its workspace and its two sync events (interprocess
// events) through a POSIX shared-memory segment, opens its peers' at engine creation, and the
// host barrier is a spin barrier in that segment.
struct IpcSlot {
  cudaIpcMemHandle_t ws;
  uint64_t ws_off;                 // workspace offset inside the exported allocation
  cudaIpcEventHandle_t ev[2];
  uint8_t uuid[16];                // device UUID (ranks sharing a GPU disable cooperative GEMMs)
  qos_model_cfg cfg;
};
struct IpcShm {
  static constexpr uint64_t kMagic = 0x716f7367726f7570ull;  // "qosgroup"
  std::atomic<uint64_t> magic;
  std::atomic<uint64_t> gen;
  std::atomic<int32_t> arrived, aborted, attached;
  int32_t n;
  IpcSlot slot[8];
};

struct qos_group {
  int n = 0;
  std::vector<qos_engine*> eng;
  std::mutex mu;
  std::condition_variable cv;
  int arrived = 0;
  uint64_t gen = 0;
  bool aborted = false;
  int timeout_ms = 120000;
  // cross-process group
  bool ipc = false;
  int rank = -1;
  IpcShm* shm = nullptr;
  std::string shm_name;

  int barrier() {
    if (ipc) return ipc_barrier();
    std::unique_lock<std::mutex> lk(mu);
    if (aborted) return qos::set_error(QOS_ERR_COMM, "peer group aborted");
    const uint64_t g = gen;
    if (++arrived == n) {
      arrived = 0;
      ++gen;
      cv.notify_all();
      return QOS_OK;
    }
    if (!cv.wait_for(lk, std::chrono::milliseconds(timeout_ms), [&] { return gen != g || aborted; })) {
      aborted = true;
      cv.notify_all();
      return qos::set_error(QOS_ERR_COMM, "peer group barrier timed out (a rank did not reach the collective)");
    }
    return aborted ? qos::set_error(QOS_ERR_COMM, "peer group aborted") : QOS_OK;
  }
  int ipc_barrier() {
    if (shm->aborted.load(std::memory_order_acquire)) return qos::set_error(QOS_ERR_COMM, "peer group aborted");
    const uint64_t g = shm->gen.load(std::memory_order_acquire);
    if (shm->arrived.fetch_add(1, std::memory_order_acq_rel) + 1 == n) {
      shm->arrived.store(0, std::memory_order_relaxed);
      shm->gen.fetch_add(1, std::memory_order_release);
      return QOS_OK;
    }
    const auto t0 = std::chrono::steady_clock::now();
    for (uint64_t spin = 0; shm->gen.load(std::memory_order_acquire) == g; ++spin) {
      if (shm->aborted.load(std::memory_order_acquire)) return qos::set_error(QOS_ERR_COMM, "peer group aborted");
      if (spin > 2048) {
        sched_yield();
        if ((spin & 1023) == 0 && std::chrono::steady_clock::now() - t0 > std::chrono::milliseconds(timeout_ms)) {
          shm->aborted.store(1, std::memory_order_release);
          return qos::set_error(QOS_ERR_COMM, "peer group barrier timed out (a rank did not reach the collective)");
        }
      }
    }
    return QOS_OK;
  }
  void abort() {
    if (ipc) {
      shm->aborted.store(1, std::memory_order_release);
      return;
    }
    std::lock_guard<std::mutex> lk(mu);
    aborted = true;
    cv.notify_all();
  }
};

struct qos_engine {
  qos_model_cfg cfg{};
  int device = 0, tp_rank = 0, tp_size = 1, num_sms = 148;
  Shard sh{};
  int nqkv = 0, table_w = 0;
  WeightLayout wl;
  WsLayout wsl{};
  uint8_t *w = nullptr, *kv = nullptr, *ws = nullptr;
  bool own_w = false, own_kv = false, own_ws = false;
  size_t kv_bytes = 0, plane_elems = 0;
  // tensor maps
  struct LMaps {
    CUtensorMap qkv[2], o[2], gu[2], d[2];  // [0]: box 128 rows, [1]: box 256 rows
  };
  std::vector<LMaps> lmaps;
  CUtensorMap head_map[2];
  struct ActMap {
    CUtensorMap m128;    // box 128 rows: A operand of gemm.cu
    CUtensorMap sw[5];   // box 16/32/64/128/256 rows: token operand of gemm_swab.cu
  };
  ActMap a_h, a_attn, a_act, a_hR;
  CUtensorMap kv_map;
  CUtensorMap kv_map5;  // the same pool, 4 consecutive blocks of one head per box (prefill attention)
  CUtensorMap q_map;  // {hd, H, max_batch_tokens} over the q columns of `qkv` (prefill attention's Q tiles)
  float2* rope_tab = nullptr;
  int32_t* d_tables = nullptr;
  // host state
  std::vector<int32_t> free_heap;  // min-heap of free block ids
  std::vector<int> free_rows;      // min-heap of free table rows
  std::unordered_map<int64_t, ReqState> reqs;
  std::vector<int32_t> pending_upd;  // (row, col, block) triples not yet on the device
  // staging
  uint8_t* h_meta[2] = {nullptr, nullptr};
  cudaEvent_t meta_free[2] = {nullptr, nullptr};
  int meta_cur = 0;
  cudaStream_t stream = nullptr;  // internal stream for synchronous calls
  cudaStream_t side = nullptr;    // high-priority stream: prefill attention overlapped with decode
  cudaStream_t side_lo = nullptr; // normal-priority side stream (option attn_order = 1)
  int attn_order = 0;             // option attn_order: 0 prefill first on `side`; 1 decode first, prefill
                                  // on `side_lo`; 2 decode first, prefill on `side`
  cudaEvent_t ev_fork = nullptr, ev_join = nullptr, ev_fork2 = nullptr, ev_join2 = nullptr;
  cudaEvent_t ev_step_done = nullptr;  // end of the last step, on the caller's stream
  bool dual_stream = false;       // QOS_DUAL=1: prefill rows and decode rows on two streams
  int dual_min_prefill = 512, dual_min_decode = 16;
  int dual_sms_pre = 0, dual_sms_dec = 0;  // SM budgets of the two streams' GEMMs (0 = all)
  int gemm_sms = 0;                // option gemm_sms: SM budget of the fused step's GEMMs (0 = all)
  bool add_split = true;           // option add_split: ordered split-K of the O / down projections
  int gemm_bn = 0;                 // option gemm_bn (experiments): force the tile width of the
                                   // non-residual tile GEMMs (QKV, gate/up): 0 auto, 128, 256
  bool gemm_2cta = true;            // option gemm_2cta: CTA-pair GEMM (256 x 256 tiles) at large M
  bool decode_round_split = true;  // option decode_round_split (A/B of the split-K ranges)
  int decode_split = 4096;         // option decode_split: longest split-K key range tried first
                                   // (4096: 5-10% faster decode attention than 512 on B200,
                                   // profiles/decode_split_ab_r1k.jsonl)
  int decode_stages = 8;            // option decode_stages: decode K/V ring depth (8 or 4)
  bool decode_persist = false;      // option decode_persist: persistent decode-attention CTAs
  int decode_items_per_sm = 4;      // option decode_items_per_sm: split decode key ranges until the
                                    // work list has this many items per SM (0: 1 or 4 by context)
  int fa_qtiles = 1;                // option fa_qtiles: prefill q tiles per CTA sharing K/V tiles
  bool fa_persist = true;           // option fa_persist: persistent prefill-attention CTAs (fa_qtiles 1)
  bool fa_pair = false;             // option fa_pair: prefill attention on CTA pairs (cta_group::2, hd 128)
  int fa_item_cost = 2;             // option fa_item_cost: per-item overhead (key tiles) when dealing
                                    // persistent prefill-attention items to CTAs
  int pair_clusters = -1;           // co-resident pairs of that kernel (queried once)
  bool norm_fold = true;            // option norm_fold: RMSNorm folded into the O / down and QKV / gate-up GEMMs
  bool overlap_attn = true;       // QOS_OVERLAP_ATTN=0 serialises a7 and a8 (for measurement)
  bool gemm_splitk = false;       // QOS_GEMM_SPLITK=1: split-K for small-M tile GEMMs (measured slower on
                                  // B200 at every shape where the engine picks the tile kernel, r1e)
  int gemm_swab = 1;              // weight-streaming GEMM (gemm_swab.cu): 0 never, 1 auto, 2 always
  int gemm_streamk = 0;           // stream-K tile GEMM: 0 never (default: measured slower on B200,
                                  // unaligned ranges lose the L2 reuse of lock-step waves), 1 auto, 2 always
  // timing
  bool timing = false;
  std::vector<std::pair<int, std::pair<cudaEvent_t, cudaEvent_t>>> tev;
  std::vector<cudaEvent_t> ev_pool;
  size_t ev_used = 0;
  // comm
  ncclComm_t comm = nullptr;
  qos_group* group = nullptr;       // peer group (tp > 1 without NCCL)
  bool shares_device = false;       // another rank of the group runs on this GPU: no cooperative
                                    // (co-residency-dependent) GEMM reductions
  uint64_t sync_seq = 0;            // peer syncs issued so far (identical on every rank)
  uint64_t red_seq = 0;             // O / down reductions issued so far (partial buffer parity)
  cudaEvent_t ev_coll[2] = {nullptr, nullptr};  // "my side of this sync is ready", by sync parity
  std::vector<uint8_t*> ipc_ws;                 // cross-process group: peers' mapped workspaces
  std::vector<uint8_t*> ipc_base;               //   (their IPC mapping bases, for closing)
  std::vector<std::array<cudaEvent_t, 2>> ipc_ev;  //   and their opened sync events
  int tp_twoshot = -1;              // option tp_twoshot: 0 one-shot, 1 two-shot, -1 auto (tp >= 4)
  bool tp_scatter = true;           // option tp_scatter: two-shot with the reduce-scatter in the GEMM epilogue
  int64_t last_h2d = 0, last_d2h = 0;  // bytes moved host<->device by the last step
  // debug buffers for ops
  void* dbg = nullptr;
  size_t dbg_bytes = 0;
};

namespace {

cudaEvent_t next_event(qos_engine* e) {
  if (e->ev_used == e->ev_pool.size()) {
    cudaEvent_t ev;
    cudaEventCreate(&ev);
    e->ev_pool.push_back(ev);
  }
  return e->ev_pool[e->ev_used++];
}

struct TimerScope {  // brackets one kernel class with events when timing is enabled
  qos_engine* e;
  int cls;
  cudaStream_t st;
  cudaEvent_t a = nullptr;
  TimerScope(qos_engine* e_, int c, cudaStream_t s) : e(e_), cls(c), st(s) {
    if (e->timing) {
      a = next_event(e);
      cudaEventRecord(a, st);
    }
  }
  ~TimerScope() {
    if (e->timing) {
      cudaEvent_t b = next_event(e);
      cudaEventRecord(b, st);
      e->tev.push_back({cls, {a, b}});
    }
  }
};

int alloc_table_row(qos_engine* e) {
  if (e->free_rows.empty()) return -1;
  std::pop_heap(e->free_rows.begin(), e->free_rows.end(), std::greater<int>());
  int r = e->free_rows.back();
  e->free_rows.pop_back();
  return r;
}

inline __nv_bfloat16* W(qos_engine* e, size_t off) { return reinterpret_cast<__nv_bfloat16*>(e->w + off); }

int build_maps(qos_engine* e) {
  const auto& c = e->cfg;
  const int d = c.d_model, hd = c.head_dim;
  e->lmaps.resize(c.n_layers);
  for (int l = 0; l < c.n_layers; ++l) {
    const auto& L = e->wl.layers[l];
    for (int b = 0; b < 2; ++b) {
      const uint32_t br = b ? 256 : 128;
      QOS_TRY(make_tmap_2d_bf16(&e->lmaps[l].qkv[b], W(e, L.wqkv), e->nqkv, d, d, br, 64, true));
      QOS_TRY(make_tmap_2d_bf16(&e->lmaps[l].o[b], W(e, L.wo), d, e->sh.H * hd, e->sh.H * hd, br, 64, true));
      QOS_TRY(make_tmap_2d_bf16(&e->lmaps[l].gu[b], W(e, L.wgu), 2 * e->sh.F, d, d, br, 64, true));
      QOS_TRY(make_tmap_2d_bf16(&e->lmaps[l].d[b], W(e, L.wd), d, e->sh.F, e->sh.F, br, 64, true));
    }
  }
  for (int b = 0; b < 2; ++b)
    QOS_TRY(make_tmap_2d_bf16(&e->head_map[b], W(e, e->wl.head), e->sh.V, d, d, b ? 256 : 128, 64, true));
  const auto& s = e->wsl;
  auto act = [&](qos_engine::ActMap& m, const void* base, int64_t rows, int64_t cols) -> int {
    QOS_TRY(make_tmap_2d_bf16(&m.m128, base, rows, cols, cols, 128, 64, true));
    for (int i = 0; i < 5; ++i) QOS_TRY(make_tmap_2d_bf16(&m.sw[i], base, rows, cols, cols, 16u << i, 64, true));
    return QOS_OK;
  };
  QOS_TRY(act(e->a_h, e->ws + s.h, c.max_batch_tokens, d));
  QOS_TRY(act(e->a_attn, e->ws + s.attn, c.max_batch_tokens, e->sh.H * hd));
  QOS_TRY(act(e->a_act, e->ws + s.act, c.max_batch_tokens, e->sh.F));
  QOS_TRY(act(e->a_hR, e->ws + s.hR, c.max_batch_rows, d));
  QOS_TRY(make_tmap_3d_bf16(&e->kv_map, e->kv, hd, uint64_t(c.num_blocks) * e->sh.Hkv * 16, uint64_t(c.n_layers) * 2,
                            64, 16, 1));
  QOS_TRY(make_tmap_kv5(&e->kv_map5, e->kv, hd, uint64_t(e->sh.Hkv), uint64_t(c.num_blocks), uint64_t(c.n_layers) * 2, 4));
  {
    const int group = c.n_heads / c.n_kv_heads;
    QOS_TRY(make_tmap_3d_bf16_strided(&e->q_map, e->ws + s.qkv, uint64_t(hd), uint64_t(e->sh.H),
                                      uint64_t(c.max_batch_tokens), uint64_t(hd) * 2, uint64_t(e->nqkv) * 2, 64,
                                      uint32_t(group), uint32_t(128 / group)));
  }
  return QOS_OK;
}

int check_cfg(const qos_model_cfg* c, int tp) {
  if (!c) return set_error(QOS_ERR_INVALID_ARG, "cfg is NULL");
  if (c->n_layers < 1 || c->d_model < 64 || c->n_heads < 1 || c->n_kv_heads < 1 || c->ffn_dim < 64 || c->vocab < 32)
    return set_error(QOS_ERR_INVALID_ARG, "bad model dims");
  if (c->n_heads % c->n_kv_heads) return set_error(QOS_ERR_INVALID_ARG, "n_heads % n_kv_heads != 0");
  if (c->head_dim != 64 && c->head_dim != 128) return set_error(QOS_ERR_UNSUPPORTED, "head_dim must be 64 or 128");
  if (c->n_heads / c->n_kv_heads > 8) return set_error(QOS_ERR_UNSUPPORTED, "GQA group > 8");
  if (c->block_size != 16) return set_error(QOS_ERR_UNSUPPORTED, "block_size must be 16");
  if (tp < 1 || c->n_kv_heads % tp || c->n_heads % tp || c->ffn_dim % tp || c->vocab % tp)
    return set_error(QOS_ERR_INVALID_ARG, "tp_size must divide n_kv_heads, n_heads, ffn_dim, vocab");
  if (c->d_model % 64 || (c->ffn_dim / tp) % 128 || ((c->n_heads / tp) * c->head_dim) % 64 || (c->vocab / tp) % 32)
    return set_error(QOS_ERR_UNSUPPORTED, "d_model % 64, (F/tp) % 128, (V/tp) % 32 required");
  if (c->num_blocks < 1 || c->max_seq_len < 1 || c->max_requests < 1 || c->max_batch_tokens < 1 ||
      c->max_batch_rows < 1)
    return set_error(QOS_ERR_INVALID_ARG, "capacities must be >= 1");
  if (c->max_batch_rows > c->max_batch_tokens) return set_error(QOS_ERR_INVALID_ARG, "max_batch_rows > max_batch_tokens");
  if (int64_t(c->max_batch_rows) * (c->n_kv_heads / tp) > kMaxDecodeItems)
    return set_error(QOS_ERR_UNSUPPORTED, "max_batch_rows * kv heads per rank exceeds the decode item workspace");
  return QOS_OK;
}

// Validate a batch and build its metadata into host staging `buf`.
int build_step(qos_engine* e, const qos_batch* b, bool check_lengths, uint8_t* buf, StepMeta& m,
               std::vector<int>* out_rows_tables = nullptr) {
  const auto& c = e->cfg;
  if (!b) return set_error(QOS_ERR_INVALID_ARG, "batch is NULL");
  if (b->n_prefill < 0 || b->n_decode < 0 || (b->n_prefill && !b->prefill) || (b->n_decode && !b->decode))
    return set_error(QOS_ERR_INVALID_ARG, "bad batch arrays");
  m.n_prefill = b->n_prefill;
  m.n_decode = b->n_decode;
  m.R = b->n_prefill + b->n_decode;
  int64_t T = b->n_decode;
  for (int i = 0; i < b->n_prefill; ++i) {
    if (b->prefill[i].chunk_len < 1 || !b->prefill[i].tokens) return set_error(QOS_ERR_INVALID_ARG, "chunk_len < 1");
    T += b->prefill[i].chunk_len;
  }
  if (m.R == 0) return set_error(QOS_ERR_INVALID_ARG, "empty batch");
  if (T > c.max_batch_tokens || m.R > c.max_batch_rows) return set_error(QOS_ERR_INVALID_ARG, "batch exceeds capacity");
  m.T = int(T);
  std::unordered_set<int64_t> seen;
  auto lookup = [&](int64_t req, int start, int n, const ReqState** out) -> int {
    auto it = e->reqs.find(req);
    if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "request has no KV table");
    if (!seen.insert(req).second) return set_error(QOS_ERR_INVALID_ARG, "request appears twice in one step");
    if (start < 0 || n < 1) return set_error(QOS_ERR_INVALID_ARG, "bad position");
    if (check_lengths && it->second.cached != start) return set_error(QOS_ERR_BAD_KV_START, "kv_start != cached length");
    if (int64_t(start) + n > int64_t(it->second.blocks.size()) * 16)
      return set_error(QOS_ERR_NOT_ALLOCATED, "step writes past the allocated blocks");
    if (int64_t(start) + n > c.max_seq_len) return set_error(QOS_ERR_INVALID_ARG, "position >= max_seq_len");
    *out = &it->second;
    return QOS_OK;
  };
  // layout of the metadata block
  size_t off = 0;
  auto take = [&](size_t bytes) {
    size_t o = off;
    off = align_up(off + bytes, 256);
    return o;
  };
  m.o_tok = take(size_t(T) * 4);
  m.o_pos = take(size_t(T) * 4);
  m.o_slot = take(size_t(T) * 4);
  m.o_rows = take(size_t(m.R) * 4);
  int32_t* tok = reinterpret_cast<int32_t*>(buf + m.o_tok);
  int32_t* pos = reinterpret_cast<int32_t*>(buf + m.o_pos);
  int32_t* slot = reinterpret_cast<int32_t*>(buf + m.o_slot);
  int32_t* rows = reinterpret_cast<int32_t*>(buf + m.o_rows);

  const int group = c.n_heads / c.n_kv_heads;
  const int ppt = prefill_tc_positions_per_tile(group);
  const bool pair = e->fa_pair && c.head_dim == 128 && e->fa_qtiles == 1 && e->fa_persist;
  const int CS = pair ? 2 : e->fa_qtiles;
  std::vector<PrefillItem> pitems;
  int t = 0;
  for (int i = 0; i < b->n_prefill; ++i) {
    const auto& ch = b->prefill[i];
    const ReqState* rs;
    QOS_TRY(lookup(ch.req, ch.kv_start, ch.chunk_len, &rs));
    for (int j = 0; j < ch.chunk_len; ++j) {
      const int tk = ch.tokens[j];
      if (tk < 0 || tk >= c.vocab) return set_error(QOS_ERR_INVALID_ARG, "token id out of range");
      const int p = ch.kv_start + j;
      tok[t + j] = tk;
      pos[t + j] = p;
      slot[t + j] = rs->blocks[p >> 4] * 16 + (p & 15);
    }
    // groups of CS consecutive q tiles of one kv head run in one CTA and share every K/V tile;
    // a short last group is filled with a duplicate of its last tile that stores nothing
    const int ntile = (ch.chunk_len + ppt - 1) / ppt;
    for (int c0 = 0; c0 < ntile; c0 += CS) {
      const int last_tile = std::min(ntile, c0 + CS) - 1;
      const int grp_last = ch.kv_start + std::min(ch.chunk_len, (last_tile + 1) * ppt) - 1;
      for (int h = 0; h < e->sh.Hkv; ++h)
        for (int k = 0; k < CS; ++k) {
          const int qt = std::min(c0 + k, last_tile);
          PrefillItem it;
          it.row0 = t + qt * ppt;
          it.npos = std::min(ppt, ch.chunk_len - qt * ppt);
          it.pos0 = ch.kv_start + qt * ppt;
          it.table = rs->row;
          it.kv_head = h;
          it.pad = c0 + k > last_tile ? 1 : 0;
          it.grp_last = grp_last;
          pitems.push_back(it);
        }
    }
    t += ch.chunk_len;
    rows[i] = t - 1;
  }
  // LPT: longest key ranges first, whole groups (the items of a group share grp_last, and the
  // stable sort keeps them adjacent and in order)
  if (CS == 1)
    std::stable_sort(pitems.begin(), pitems.end(),
                     [](const PrefillItem& a, const PrefillItem& b2) { return a.pos0 + a.npos > b2.pos0 + b2.npos; });
  else {
    std::vector<int> order(pitems.size() / CS);
    for (size_t i = 0; i < order.size(); ++i) order[i] = int(i);
    std::stable_sort(order.begin(), order.end(),
                     [&](int a, int b2) { return pitems[size_t(a) * CS].grp_last > pitems[size_t(b2) * CS].grp_last; });
    std::vector<PrefillItem> sorted;
    sorted.reserve(pitems.size());
    for (int g2 : order)
      for (int k = 0; k < CS; ++k) sorted.push_back(pitems[size_t(g2) * CS + k]);
    pitems.swap(sorted);
  }
  m.fa_qtiles = CS;
  // persistent prefill attention: the LPT-sorted items dealt greedily to 2 CTAs per SM by key
  // tiles (+2 tiles for an item's Q staging and epilogue), each CTA's items kept longest first
  std::vector<int32_t> pcta;
  if (CS == 1 && e->fa_persist && !pitems.empty()) {
    const int G = int(std::min<size_t>({pitems.size(), size_t(2 * e->num_sms), size_t(1024)}));
    std::priority_queue<std::pair<int64_t, int>, std::vector<std::pair<int64_t, int>>, std::greater<>> heap;
    for (int g = 0; g < G; ++g) heap.push({0, g});
    std::vector<std::vector<int>> lists(static_cast<size_t>(G));
    for (size_t i = 0; i < pitems.size(); ++i) {
      auto [load, g] = heap.top();
      heap.pop();
      lists[size_t(g)].push_back(int(i));
      heap.push({load + pitems[i].grp_last / 64 + 1 + e->fa_item_cost, g});
    }
    std::vector<PrefillItem> dealt;
    dealt.reserve(pitems.size());
    pcta.push_back(0);
    for (const auto& li : lists) {
      for (int i : li) dealt.push_back(pitems[size_t(i)]);
      pcta.push_back(int32_t(dealt.size()));
    }
    pitems.swap(dealt);
    m.n_pcta = G;
  } else if (pair && !pitems.empty()) {
    // CTA pairs: the LPT-sorted groups of 2 q tiles dealt greedily to the co-resident pairs
    // (2 per SM pair); offsets count groups
    if (e->pair_clusters < 0) e->pair_clusters = prefill_pair_max_clusters();
    if (e->pair_clusters <= 0) return set_error(QOS_ERR_CUDA, "prefill pair kernel: no co-resident CTA pair");
    const size_t ngrp = pitems.size() / 2;
    const int G = int(std::min<size_t>({ngrp, size_t(e->pair_clusters), size_t(1024)}));
    std::priority_queue<std::pair<int64_t, int>, std::vector<std::pair<int64_t, int>>, std::greater<>> heap;
    for (int g = 0; g < G; ++g) heap.push({0, g});
    std::vector<std::vector<int>> lists(static_cast<size_t>(G));
    for (size_t i = 0; i < ngrp; ++i) {
      auto [load, g] = heap.top();
      heap.pop();
      lists[size_t(g)].push_back(int(i));
      heap.push({load + pitems[2 * i].grp_last / 64 + 1 + e->fa_item_cost, g});
    }
    std::vector<PrefillItem> dealt;
    dealt.reserve(pitems.size());
    pcta.push_back(0);
    for (const auto& li : lists) {
      for (int i : li) {
        dealt.push_back(pitems[2 * size_t(i)]);
        dealt.push_back(pitems[2 * size_t(i) + 1]);
      }
      pcta.push_back(int32_t(dealt.size() / 2));
    }
    pitems.swap(dealt);
    m.n_pcta = G;
    m.fa_pair = 1;
  }
  // decode split-K work list (balanced on sum of keys)
  int64_t total_keys = 0;
  for (int i = 0; i < b->n_decode; ++i) total_keys += int64_t(b->decode[i].ctx_len) + 1;
  int split = e->decode_split;
  // splits per decode: the key blocks in nsplit near-equal block-aligned ranges of about
  // `split` keys (rounded to the nearest count, so 4097 keys make 8 ranges of 32-33 blocks, not
  // 8 full ranges and a 1-key straggler that pays a whole CTA prologue and merge)
  const bool round_split = e->decode_round_split;
  auto nsplit_of = [&](int keys, int s) {
    if (!round_split) return (keys + s - 1) / s;
    const int nb = (keys + 15) / 16, sb = s / 16;
    return std::max(1, (nb + sb / 2) / sb);
  };
  {
    // enough items to fill the SMs (4 per SM).  Option decode_items_per_sm = 0 picks 1 per SM
    // for short decodes (< 3072 keys on average: latency-bound items, fewer and longer ones are
    // 14-29% faster in ncu cycles and 5-9% on small decode-heavy steps) — off by default until
    // re-validated with the full GPU suite; the latency model fits it as well as the default on
    // short-context test batches (profiles/latency_table_short_s{4,0}_r2c.json)
    int per_sm = e->decode_items_per_sm;
    if (per_sm <= 0) per_sm = (b->n_decode > 0 && total_keys < int64_t(3072) * b->n_decode) ? 1 : 4;
    const int64_t target = int64_t(e->num_sms) * per_sm;
    auto count_items = [&](int s) {
      int64_t n = 0;
      for (int i = 0; i < b->n_decode; ++i) n += nsplit_of(b->decode[i].ctx_len + 1, s);
      return n * e->sh.Hkv;
    };
    while (split > 64 && count_items(split) < target) split /= 2;
    // every decode contributes >= 1 item per kv head however long the ranges get, so the
    // doubling stops at the longest possible context; a step that still exceeds the item
    // workspace (n_decode * Hkv > max_items) is refused
    while (split < (1 << 24) && count_items(split) > e->wsl.max_items) split *= 2;
    if (count_items(split) > e->wsl.max_items)
      return set_error(QOS_ERR_UNSUPPORTED, "decode work list exceeds the item workspace (n_decode * kv heads)");
  }
  std::vector<DecodeItem> ditems;
  int part = 0;
  for (int i = 0; i < b->n_decode; ++i) {
    const auto& dc = b->decode[i];
    const ReqState* rs;
    QOS_TRY(lookup(dc.req, dc.ctx_len, 1, &rs));
    if (dc.token < 0 || dc.token >= c.vocab) return set_error(QOS_ERR_INVALID_ARG, "token id out of range");
    const int p = dc.ctx_len;
    tok[t] = dc.token;
    pos[t] = p;
    slot[t] = rs->blocks[p >> 4] * 16 + (p & 15);
    rows[b->n_prefill + i] = t;
    const int keys = p + 1;
    const int nsplit = nsplit_of(keys, split);
    const int nb = (keys + 15) / 16;
    for (int h = 0; h < e->sh.Hkv; ++h)
      for (int s = 0; s < nsplit; ++s) {
        DecodeItem it;
        it.row = t;
        it.table = rs->row;
        it.kv_head = h;
        if (round_split) {
          it.key0 = 16 * int(int64_t(s) * nb / nsplit);
          it.key1 = std::min(keys, 16 * int(int64_t(s + 1) * nb / nsplit));
        } else {
          it.key0 = s * split;
          it.key1 = std::min(keys, (s + 1) * split);
        }
        it.part_base = part + h * nsplit;
        it.part = it.part_base + s;
        it.nsplit = nsplit;
        it.counter = i * e->sh.Hkv + h;
        ditems.push_back(it);
      }
    part += e->sh.Hkv * nsplit;
    ++t;
  }
  // longest items first
  std::stable_sort(ditems.begin(), ditems.end(),
                   [](const DecodeItem& a, const DecodeItem& b2) { return a.key1 - a.key0 > b2.key1 - b2.key0; });
  m.n_pitems = int(pitems.size());
  m.n_ditems = int(ditems.size());
  m.o_pitems = take(pitems.size() * sizeof(PrefillItem));
  m.o_ditems = take(ditems.size() * sizeof(DecodeItem));
  m.o_pcta = take(pcta.size() * 4);
  const size_t max_upd = 65536;
  m.n_upd = int(std::min(e->pending_upd.size() / 3, max_upd));
  m.o_upd = take(size_t(m.n_upd) * 12);
  m.used = off;
  if (m.used > e->wsl.meta_bytes) return set_error(QOS_ERR_INVALID_ARG, "metadata exceeds workspace");
  if (!pitems.empty()) memcpy(buf + m.o_pitems, pitems.data(), pitems.size() * sizeof(PrefillItem));
  if (!ditems.empty()) memcpy(buf + m.o_ditems, ditems.data(), ditems.size() * sizeof(DecodeItem));
  if (!pcta.empty()) memcpy(buf + m.o_pcta, pcta.data(), pcta.size() * 4);
  if (m.n_upd) memcpy(buf + m.o_upd, e->pending_upd.data(), size_t(m.n_upd) * 12);
  (void)out_rows_tables;
  return QOS_OK;
}

// Upload staging -> device metadata block of the current buffer; returns device base.
int upload_meta(qos_engine* e, const StepMeta& m, cudaStream_t st, uint8_t** d_meta) {
  const int cur = e->meta_cur;
  uint8_t* dm = e->ws + e->wsl.meta[cur];
  QOS_CU(cudaStreamWaitEvent(st, e->meta_free[cur], 0));
  QOS_CU(cudaMemcpyAsync(dm, e->h_meta[cur], m.used, cudaMemcpyHostToDevice, st));
  if (m.n_upd) {
    QOS_CU(launch_table_update(e->d_tables, e->table_w, reinterpret_cast<int32_t*>(dm + m.o_upd), m.n_upd, st));
    e->pending_upd.erase(e->pending_upd.begin(), e->pending_upd.begin() + size_t(m.n_upd) * 3);
  }
  *d_meta = dm;
  return QOS_OK;
}

// Wait until the staging buffer `cur` is no longer read by an in-flight copy/step.
int acquire_staging(qos_engine* e) {
  e->meta_cur ^= 1;
  QOS_CU(cudaEventSynchronize(e->meta_free[e->meta_cur]));
  return QOS_OK;
}

int release_staging(qos_engine* e, cudaStream_t st) {
  QOS_CU(cudaEventRecord(e->meta_free[e->meta_cur], st));
  return QOS_OK;
}

// The internal stream, ordered after the last step enqueued on the caller's stream: KV fills,
// table flushes and the op entry points may touch blocks / table rows that an in-flight step
// (freed and re-allocated meanwhile) still reads (qos_kv_free returns them at once).
cudaStream_t internal_stream(qos_engine* e) {
  if (e->ev_step_done) cudaStreamWaitEvent(e->stream, e->ev_step_done, 0);
  return e->stream;
}

int flush_table_updates(qos_engine* e, cudaStream_t st) {
  while (!e->pending_upd.empty()) {
    QOS_TRY(acquire_staging(e));
    const size_t n = std::min<size_t>(e->pending_upd.size() / 3, 65536);
    memcpy(e->h_meta[e->meta_cur], e->pending_upd.data(), n * 12);
    uint8_t* dm = e->ws + e->wsl.meta[e->meta_cur];
    QOS_CU(cudaStreamWaitEvent(st, e->meta_free[e->meta_cur], 0));
    QOS_CU(cudaMemcpyAsync(dm, e->h_meta[e->meta_cur], n * 12, cudaMemcpyHostToDevice, st));
    QOS_CU(launch_table_update(e->d_tables, e->table_w, reinterpret_cast<int32_t*>(dm), int(n), st));
    QOS_TRY(release_staging(e, st));
    e->pending_upd.erase(e->pending_upd.begin(), e->pending_upd.begin() + n * 3);
  }
  return QOS_OK;
}

static int swab_index(int bnt) { return bnt == 16 ? 0 : bnt == 32 ? 1 : bnt == 64 ? 2 : bnt == 128 ? 3 : 4; }

// One projection GEMM of M rows: gemm_swab.cu (weight-streaming, swap-AB, stream-K) at small M,
// else gemm.cu (activation-stationary tiles, optional split-K).
// the kernel gemm_any takes for this shape runs whole tiles in one pass (the folded RMSNorm's
// producer and consumer epilogues live there): not the weight-streaming kernel, no split-K
bool gemm_one_pass(const qos_engine* e, int64_t M, int64_t N, int64_t K, int sms) {
  if (N % 128 == 0 && (e->gemm_swab == 2 || (e->gemm_swab == 1 && swab_prefer_k(M, N, K, sms)))) return false;
  return !e->gemm_splitk;
}

int gemm_any(qos_engine* e, const qos_engine::ActMap& am, const CUtensorMap (&tb)[2], int64_t M, int64_t N, int64_t K,
             int epi, void* C, int64_t ldc, const float* bias, cudaStream_t st, int sms, float* part, int* cnt,
             int a_row0, const QkvRopeArgs* rope, const NormFold* fold = nullptr) {
  count_launch();
  if (fold && !gemm_one_pass(e, M, N, K, sms)) return set_error(QOS_ERR_INVALID_ARG, "folded norm on a split GEMM");
  if (N % 128 == 0 && (e->gemm_swab == 2 || (e->gemm_swab == 1 && swab_prefer_k(M, N, K, sms)))) {
    const int bnt = swab_pick_bnt(M);
    return gemm_swab_run(tb[0], am.sw[swab_index(bnt)], bnt, M, N, K, epi, C, ldc, bias, sms, st, part, cnt,
                         int64_t(kGemmMaxUnits) * 128 * 256, kGemmMaxTiles, a_row0, rope, !e->dual_stream && !e->shares_device);
  }
  if (e->gemm_2cta && gemm2_eligible(M, N, K, sms))
    return gemm2_run(am.m128, tb[0], M, N, K, epi, C, ldc, bias, sms, st, a_row0, sms, rope, fold);
  int bn = gemm_pick_bn(M, N, epi, sms);
  if (e->gemm_bn && epi != EPI_ADD_F32 && (e->gemm_bn == 128 || N % 256 == 0)) bn = e->gemm_bn;  // experiments
  int ks = e->gemm_splitk ? gemm_pick_ksplit(M, N, K, bn, sms, kGemmMaxUnits) : 1;
  const bool coop = !e->dual_stream && !e->shares_device;
  // O / down below the fold threshold: tile width + ordered in-place split-K by wave cost
  if (epi == EPI_ADD_F32 && !fold && coop && e->add_split && !e->gemm_splitk && !e->gemm_streamk)
    gemm_pick_add_split(M, N, K, sms, kGemmMaxTiles, &bn, &ks);
  return gemm_run(am.m128, tb[bn == 256 ? 1 : 0], bn, M, N, K, epi, C, ldc, bias, sms, st, ks, part, cnt, a_row0, sms,
                  rope, e->gemm_streamk, coop, fold);
}

int gemm(qos_engine* e, const qos_engine::ActMap& am, const CUtensorMap (&tb)[2], int64_t M, int64_t N, int64_t K,
         int epi, void* C, int64_t ldc, const float* bias, cudaStream_t st) {
  return gemm_any(e, am, tb, M, N, K, epi, C, ldc, bias, st, e->num_sms,
                  reinterpret_cast<float*>(e->ws + e->wsl.gemm_part), reinterpret_cast<int*>(e->ws + e->wsl.gemm_cnt), 0,
                  nullptr);
}

int allreduce_bf16(qos_engine* e, void* buf, size_t count, cudaStream_t st) {
  ncclResult_t r = g_nccl.allReduce(buf, buf, count, ncclBfloat16, ncclSum, e->comm, st);
  if (r != ncclSuccess) {
    if (g_nccl.commAbort) g_nccl.commAbort(e->comm);
    e->comm = nullptr;
    return set_error(QOS_ERR_COMM, g_nccl.errStr ? g_nccl.errStr(r) : "ncclAllReduce failed");
  }
  return QOS_OK;
}

// Where the O / down projection of a TP rank writes its partial: `h` (reduced in place by NCCL)
// or, in a peer group, this collective's parity buffer (read by every rank's reduction).  A
// parity buffer is rewritten two collectives later, after this rank's stream has waited on every
// peer's event of the collective in between, which each peer recorded after its reduction had
// read the buffer.
void* tp_partial_dst(qos_engine* e) {
  return e->group ? e->ws + e->wsl.part[e->red_seq & 1] : e->ws + e->wsl.h;
}

// Peer group: record "my input of this collective is ready", meet the other ranks' host threads,
// then order this rank's stream after every peer's record (cross-device waits are legal).
// An event of parity x is re-recorded two syncs later, i.e. after the barrier of the sync in
// between, which every rank reaches only after it has issued its waits on this one.
uint8_t* peer_ws(qos_engine* e, int k) {
  if (k == e->tp_rank) return e->ws;
  return e->group->ipc ? e->ipc_ws[size_t(k)] : e->group->eng[size_t(k)]->ws;
}
cudaEvent_t peer_event(qos_engine* e, int k, int par) {
  return e->group->ipc ? e->ipc_ev[size_t(k)][size_t(par)] : e->group->eng[size_t(k)]->ev_coll[par];
}

int peer_sync(qos_engine* e, cudaStream_t st) {
  const int par = int(e->sync_seq++ & 1);
  QOS_CU(cudaEventRecord(e->ev_coll[par], st));
  QOS_TRY(e->group->barrier());
  for (int k = 0; k < e->tp_size; ++k)
    if (k != e->tp_rank) QOS_CU(cudaStreamWaitEvent(st, peer_event(e, k, par), 0));
  return QOS_OK;
}

PeerPtrs peer_ptrs(qos_engine* e, size_t ws_off) {
  PeerPtrs p{};
  for (int k = 0; k < e->tp_size; ++k) p.p[k] = peer_ws(e, k) + ws_off;
  return p;
}

// a10 + a3: sum the ranks' partials into the fp32 residual, then RMSNorm with gain g into h
// (g == nullptr after the last layer: add only).
bool tp_two_shot(const qos_engine* e) { return e->tp_twoshot > 0 || (e->tp_twoshot < 0 && e->tp_size >= 4); }

// Peer-group two-shot with the reduce-scatter fused into the producing GEMM's epilogue: each
// partial row is stored straight into its owner rank's receive slot for this rank (peer
// memory), tile by tile while the remaining tiles compute.  Needs the one-pass tile kernels.
bool tp_scatter_on(const qos_engine* e, int64_t T, int64_t N, int64_t K) {
  return e->group && e->tp_scatter && tp_two_shot(e) && gemm_one_pass(e, T, N, K, e->num_sms);
}
NormFold tp_scatter_args(qos_engine* e, int T) {
  NormFold f;
  const int rs = (T + e->tp_size - 1) / e->tp_size;
  const size_t rs_max = (size_t(e->cfg.max_batch_tokens) + e->tp_size - 1) / e->tp_size;
  const size_t d = size_t(e->cfg.d_model);
  for (int k = 0; k < e->tp_size; ++k)  // owner k's slot for this rank
    f.scat[k] = peer_ws(e, k) + e->wsl.recv[e->red_seq & 1] + size_t(e->tp_rank) * rs_max * d * 2;
  f.scat_rs = rs;
  return f;
}

int tp_reduce_add_norm(qos_engine* e, const void* g, int T, cudaStream_t st, bool scattered = false) {
  const int d = e->cfg.d_model;
  float* resid = reinterpret_cast<float*>(e->ws + e->wsl.resid);
  __nv_bfloat16* h = reinterpret_cast<__nv_bfloat16*>(e->ws + e->wsl.h);
  if (!e->group) {
    {
      TimerScope ts(e, QOS_T_ALLREDUCE, st);
      QOS_TRY(allreduce_bf16(e, h, size_t(T) * d, st));
    }
    TimerScope ts(e, QOS_T_NORM, st);
    if (g) QOS_CU(launch_add_rmsnorm(resid, h, g, h, T, d, e->cfg.rms_eps, st));
    else QOS_CU(launch_add_f32(resid, h, size_t(T) * d, st));
    return QOS_OK;
  }
  TimerScope ts(e, QOS_T_ALLREDUCE, st);
  const int par = int(e->red_seq++ & 1);
  PeerPtrs parts = peer_ptrs(e, e->wsl.part[par]);
  const int rs = (T + e->tp_size - 1) / e->tp_size, row0 = std::min(T, e->tp_rank * rs);
  if (scattered) {  // the peers' partial rows of this rank's slice are already in its receive slots
    const size_t rs_max = (size_t(e->cfg.max_batch_tokens) + e->tp_size - 1) / e->tp_size;
    for (int k = 0; k < e->tp_size; ++k)  // slot k, shifted so that row t indexes its local row t - row0
      parts.p[k] = e->ws + e->wsl.recv[par] + (size_t(k) * rs_max * d - size_t(row0) * d) * 2;
  }
  QOS_TRY(peer_sync(e, st));  // every rank's partial is complete (scattered: landed in the owners' slots)
  const bool two = tp_two_shot(e);
  if (!two) {
    QOS_CU(launch_peer_add_rmsnorm(parts, e->tp_size, resid, g, h, T, d, e->cfg.rms_eps, st));
    return QOS_OK;
  }
  // two-shot: this rank reduces + normalises its row slice and stores the rows into every peer
  QOS_CU(launch_peer_rs_norm_ag(parts, peer_ptrs(e, e->wsl.h), peer_ptrs(e, e->wsl.resid), e->tp_size, e->tp_rank,
                                row0, std::min(rs, T - row0), g, d, e->cfg.rms_eps, st));
  QOS_TRY(peer_sync(e, st));  // every rank's rows have landed in every h (or residual)
  return QOS_OK;
}

// The layer loop.  `dm` = device metadata block of this step.
// One row range of the batch pushed through all layers on one stream.  `pre` / `dec` select
// which attention work lists the range owns.
struct Seg {
  int row0, n;
  cudaStream_t st;
  bool pre, dec;
  float* gpart;  // split-K workspace of this stream
  int* gcnt;
  int sms;       // SM budget of this stream's GEMMs (0 = all)
};

int gemm_seg(qos_engine* e, const Seg& g, const qos_engine::ActMap& am, const CUtensorMap (&tb)[2], int64_t N,
             int64_t K, int epi, void* C, int64_t ldc, const float* bias, const QkvRopeArgs* rope = nullptr,
             const NormFold* fold = nullptr) {
  const int sms = g.sms > 0 ? g.sms : e->num_sms;
  const size_t esz = (epi == EPI_STORE_F32 || epi == EPI_ADD_F32) ? 4 : 2;
  return gemm_any(e, am, tb, g.n, N, K, epi, reinterpret_cast<uint8_t*>(C) + size_t(g.row0) * ldc * esz, ldc, bias,
                  g.st, sms, g.gpart, g.gcnt, g.row0, rope, fold);
}

// The layer loop.  `dm` = device metadata block of this step.
int run_layers(qos_engine* e, const StepMeta& m, uint8_t* dm, void* logits, int logits_dtype, int32_t* next_tokens,
               bool out_device, cudaStream_t st) {
  const auto& c = e->cfg;
  const int d = c.d_model, hd = c.head_dim, T = m.T, R = m.R;
  const auto& s = e->wsl;
  float* resid = reinterpret_cast<float*>(e->ws + s.resid);
  __nv_bfloat16* h = reinterpret_cast<__nv_bfloat16*>(e->ws + s.h);
  __nv_bfloat16* qkv = reinterpret_cast<__nv_bfloat16*>(e->ws + s.qkv);
  void* attn = e->ws + s.attn;
  __nv_bfloat16* act = reinterpret_cast<__nv_bfloat16*>(e->ws + s.act);
  void* hR = e->ws + s.hR;
  const int32_t* tok = reinterpret_cast<const int32_t*>(dm + m.o_tok);
  const int32_t* pos = reinterpret_cast<const int32_t*>(dm + m.o_pos);
  const int32_t* slot = reinterpret_cast<const int32_t*>(dm + m.o_slot);
  const int32_t* rows = reinterpret_cast<const int32_t*>(dm + m.o_rows);
  const size_t plane = e->plane_elems;
  const bool tp = e->tp_size > 1;
  AttnLaunch al;
  al.q = qkv;
  al.q_ld = e->nqkv;
  al.out = attn;
  al.out_ld = e->sh.H * hd;
  al.out_f32 = 0;
  al.kv_tmap = &e->kv_map;
  al.kv_tmap5 = &e->kv_map5;
  al.H = e->sh.H;
  al.Hkv = e->sh.Hkv;
  al.hd = hd;
  al.num_blocks = int(c.num_blocks);
  al.tables = e->d_tables;
  al.table_w = e->table_w;
  al.scale_log2 = float(1.4426950408889634 / std::sqrt(double(hd)));
  al.q_tiles = m.fa_qtiles;
  al.cta_off = m.n_pcta ? reinterpret_cast<const int32_t*>(dm + m.o_pcta) : nullptr;
  al.n_cta = m.n_pcta;
  al.pair = m.fa_pair;
  al.q_tmap = &e->q_map;
  al.q_rows = c.max_batch_tokens;
  al.decode_stages = e->decode_stages;
  al.decode_persist = e->decode_persist ? 1 : 0;
  const int n_pre_rows = T - m.n_decode;
  float* gpart0 = reinterpret_cast<float*>(e->ws + s.gemm_part);
  int* gcnt0 = reinterpret_cast<int*>(e->ws + s.gemm_cnt);
  // dual mode: the prefill rows and the decode rows are independent requests that share only the
  // weights, so they run as two sub-batches on two streams — the tensor-bound projections of the
  // chunk overlap the HBM-bound decode attention (and the weight-bound decode-row GEMMs)
  const bool dual = !tp && e->dual_stream && n_pre_rows >= e->dual_min_prefill && m.n_decode >= e->dual_min_decode;
  Seg segs[2];
  int nseg = 0;
  if (dual) {
    segs[nseg++] = Seg{0, n_pre_rows, st, true, false, gpart0, gcnt0, e->dual_sms_pre};
    segs[nseg++] = Seg{n_pre_rows, m.n_decode, e->side, false, true,
                       reinterpret_cast<float*>(e->ws + s.gemm_part2), reinterpret_cast<int*>(e->ws + s.gemm_cnt2),
                       e->dual_sms_dec};
    QOS_CU(cudaEventRecord(e->ev_fork, st));
    QOS_CU(cudaStreamWaitEvent(e->side, e->ev_fork, 0));
  } else {
    segs[nseg++] = Seg{0, T, st, m.n_pitems > 0, m.n_ditems > 0, gpart0, gcnt0, e->gemm_sms};
  }
  // RMSNorm folded into the projections (NormFold, internal.h) when all four GEMMs of the step
  // run whole tiles in one pass: the O / down epilogues produce r, h = bf16(r * g) and per-row
  // sums of squares, the QKV / gate-up epilogues scale their rows by 1/rms — no norm launches
  const int sms_all = e->gemm_sms > 0 ? e->gemm_sms : e->num_sms;
  // (from T = 1536: below, the read-add-write epilogue of the last wave costs what the norm
  //  launches cost — 512 tokens +1.5%, 1024 neutral, 2176 -1.5%, 4096 -4.6%, tools/attn_bench.py r1f)
  const bool fold = e->norm_fold && !tp && nseg == 1 && !g_skip_norm && T >= kFoldMinTokens && d % 128 == 0 &&
                    d / 128 <= kFoldSlots &&
                    gemm_one_pass(e, T, e->nqkv, d, sms_all) && gemm_one_pass(e, T, d, e->sh.H * hd, sms_all) &&
                    gemm_one_pass(e, T, 2 * e->sh.F, d, sms_all) && gemm_one_pass(e, T, d, e->sh.F, sms_all);
  float* ssb[2] = {reinterpret_cast<float*>(e->ws + s.ss[0]), reinterpret_cast<float*>(e->ws + s.ss[1])};
  float* rsb[2] = {reinterpret_cast<float*>(e->ws + s.rs[0]), reinterpret_cast<float*>(e->ws + s.rs[1])};
  auto fold_args = [&](int in, int out, uint64_t g_off) {  // in / out: ss/rs buffer index or -1
    NormFold f;
    f.rs_in = in >= 0 ? rsb[in] : nullptr;
    f.ss_out = out >= 0 ? ssb[out] : nullptr;
    f.rs_out = out >= 0 ? rsb[out] : nullptr;
    f.cnt = out >= 0 ? reinterpret_cast<int*>(e->ws + s.fcnt) : nullptr;
    f.g_out = out >= 0 ? W(e, g_off) : nullptr;
    f.h_out = out >= 0 ? h : nullptr;
    f.ss_n = d / 128;
    f.d = d;
    f.eps = c.rms_eps;
    return f;
  };
  for (int l = 0; l < c.n_layers; ++l) {
    const auto& L = e->wl.layers[l];
    const auto& M = e->lmaps[l];
    // fold: ss[1] carries ln1's statistics (down -> next QKV), ss[0] ln2's (O -> gate/up)
    const NormFold f_qkv = fold_args(l > 0 ? 1 : -1, -1, 0);
    const NormFold f_o = fold_args(-1, 0, L.ln2);
    const NormFold f_gu = fold_args(0, -1, 0);
    const NormFold f_down = fold_args(-1, 1, l + 1 < c.n_layers ? e->wl.layers[l + 1].ln1 : 0);
    const bool fold_down = fold && l + 1 < c.n_layers;
    __nv_bfloat16* kpl = reinterpret_cast<__nv_bfloat16*>(e->kv) + (size_t(l) * 2 + 0) * plane;
    __nv_bfloat16* vpl = reinterpret_cast<__nv_bfloat16*>(e->kv) + (size_t(l) * 2 + 1) * plane;
    al.layer = l;
    for (int si = 0; si < nseg; ++si) {
      const Seg& g = segs[si];
      const cudaStream_t gs = g.st;
      const size_t r0 = size_t(g.row0);
      if (l == 0) {
        TimerScope ts(e, QOS_T_EMBED, gs);
        QOS_CU(launch_embed_rmsnorm(tok + r0, W(e, e->wl.emb), W(e, L.ln1), resid + r0 * d, h + r0 * d, g.n, d,
                                    c.rms_eps, gs));
      } else if (!tp && !fold) {  // (tp: ln1 was applied by the add+norm after the previous all-reduce)
        TimerScope ts(e, QOS_T_NORM, gs);
        if (!g_skip_norm) QOS_CU(launch_rmsnorm(resid + r0 * d, W(e, L.ln1), h + r0 * d, g.n, d, c.rms_eps, gs));
      }
      {
        // a4 + a5 + a6: QKV projection (+bias) with RoPE and the paged KV append in its epilogue
        TimerScope ts(e, QOS_T_GEMM_QKV, gs);
        const QkvRopeArgs ra{pos + r0, slot + r0, e->rope_tab, kpl, vpl, e->sh.H, e->sh.Hkv, hd};
        QOS_TRY(gemm_seg(e, g, e->a_h, M.qkv, e->nqkv, d, EPI_QKV_ROPE, qkv, e->nqkv,
                         c.qkv_bias ? reinterpret_cast<const float*>(e->w + L.bqkv) : nullptr, &ra,
                         fold && l > 0 ? &f_qkv : nullptr));
      }
      // a7 || a8: within one segment, the prefill tiles go to the high-priority side stream and
      // the decode split-K items stay on the segment's stream (disjoint rows of `attn`)
      const bool overlap = !dual && e->overlap_attn && g.pre && g.dec;
      cudaStream_t side = e->attn_order == 1 ? e->side_lo : e->side;
      cudaStream_t pst = overlap ? side : gs;
      if (overlap) {
        QOS_CU(cudaEventRecord(e->ev_fork2, gs));
        QOS_CU(cudaStreamWaitEvent(side, e->ev_fork2, 0));
      }
      auto prefill = [&]() -> int {
        if (g.pre && m.n_pitems) {
          TimerScope ts(e, QOS_T_PREFILL_ATTN, pst);
          QOS_CU(launch_prefill_attention_tc(al, reinterpret_cast<const PrefillItem*>(dm + m.o_pitems), m.n_pitems,
                                             pst));
        }
        return QOS_OK;
      };
      auto decode = [&]() -> int {
        if (g.dec && m.n_ditems) {
          TimerScope ts(e, QOS_T_DECODE_ATTN, gs);
          QOS_CU(launch_decode_attention(al, reinterpret_cast<const DecodeItem*>(dm + m.o_ditems), m.n_ditems,
                                         reinterpret_cast<float*>(e->ws + s.partials),
                                         reinterpret_cast<int*>(e->ws + s.counters), gs));
        }
        return QOS_OK;
      };
      if (e->attn_order == 0) {
        QOS_TRY(prefill());
        QOS_TRY(decode());
      } else {
        QOS_TRY(decode());
        QOS_TRY(prefill());
      }
      if (overlap) {
        QOS_CU(cudaEventRecord(e->ev_join2, side));
        QOS_CU(cudaStreamWaitEvent(gs, e->ev_join2, 0));
      }
      if (!tp) {
        TimerScope ts(e, QOS_T_GEMM_O, gs);
        QOS_TRY(gemm_seg(e, g, e->a_attn, M.o, d, e->sh.H * hd, EPI_ADD_F32, resid, d, nullptr, nullptr,
                         fold ? &f_o : nullptr));
      } else {
        const bool sc = tp_scatter_on(e, T, d, e->sh.H * hd);
        const NormFold fs = sc ? tp_scatter_args(e, T) : NormFold{};
        {
          TimerScope ts(e, QOS_T_GEMM_O, gs);
          QOS_TRY(gemm_seg(e, g, e->a_attn, M.o, d, e->sh.H * hd, EPI_STORE_BF16, tp_partial_dst(e), d, nullptr,
                           nullptr, sc ? &fs : nullptr));
        }
        QOS_TRY(tp_reduce_add_norm(e, W(e, L.ln2), T, gs, sc));
      }
      if (!tp && !fold) {
        TimerScope ts(e, QOS_T_NORM, gs);
        if (!g_skip_norm) QOS_CU(launch_rmsnorm(resid + r0 * d, W(e, L.ln2), h + r0 * d, g.n, d, c.rms_eps, gs));
      }
      {
        TimerScope ts(e, QOS_T_GEMM_GATEUP, gs);
        QOS_TRY(gemm_seg(e, g, e->a_h, M.gu, 2 * e->sh.F, d, EPI_SILU_GATE, act, e->sh.F, nullptr, nullptr,
                         fold ? &f_gu : nullptr));
      }
      if (!tp) {
        TimerScope ts(e, QOS_T_GEMM_DOWN, gs);
        QOS_TRY(gemm_seg(e, g, e->a_act, M.d, d, e->sh.F, EPI_ADD_F32, resid, d, nullptr, nullptr,
                         fold_down ? &f_down : nullptr));
      } else {
        const bool sc = tp_scatter_on(e, T, d, e->sh.F);
        const NormFold fs = sc ? tp_scatter_args(e, T) : NormFold{};
        {
          TimerScope ts(e, QOS_T_GEMM_DOWN, gs);
          QOS_TRY(gemm_seg(e, g, e->a_act, M.d, d, e->sh.F, EPI_STORE_BF16, tp_partial_dst(e), d, nullptr, nullptr,
                           sc ? &fs : nullptr));
        }
        QOS_TRY(tp_reduce_add_norm(e, l + 1 < c.n_layers ? W(e, e->wl.layers[l + 1].ln1) : nullptr, T, gs, sc));
      }
    }
  }
  if (dual) {
    QOS_CU(cudaEventRecord(e->ev_join, e->side));
    QOS_CU(cudaStreamWaitEvent(st, e->ev_join, 0));
  }
  // final norm on the R logit rows + LM head
  {
    TimerScope ts(e, QOS_T_HEAD, st);
    QOS_CU(launch_gather_rmsnorm(resid, rows, W(e, e->wl.lnf), hR, R, d, c.rms_eps, st));
  }
  // logits destination: f32 logits land in the caller's device buffer when possible
  float* lg = reinterpret_cast<float*>(e->ws + s.logits);
  const bool direct = out_device && logits && logits_dtype == QOS_F32 && !tp;
  float* lout = direct ? reinterpret_cast<float*>(logits) : lg;
  {
    TimerScope ts(e, QOS_T_HEAD, st);
    if (!tp) {
      QOS_TRY(gemm(e, e->a_hR, e->head_map, R, c.vocab, d, EPI_STORE_F32, lout, c.vocab, nullptr, st));
    } else {
      float* loc = reinterpret_cast<float*>(e->ws + s.logits_loc);
      QOS_TRY(gemm(e, e->a_hR, e->head_map, R, e->sh.V, d, EPI_STORE_F32, loc, e->sh.V, nullptr, st));
      if (e->group) {  // peer group: read every rank's vocab slice directly
        QOS_TRY(peer_sync(e, st));
        QOS_CU(launch_peer_gather_logits(peer_ptrs(e, s.logits_loc), e->tp_size, R, e->sh.V, lg, st));
      } else {
      // all-gather of [R][V/tp] shards -> [tp][R][V/tp], then transpose into [R][V]
      ncclResult_t r = g_nccl.allGather(loc, lg, size_t(R) * e->sh.V, ncclFloat32, e->comm, st);
      if (r != ncclSuccess) return set_error(QOS_ERR_COMM, "ncclAllGather failed");
      // gathered layout [tp][R][V/tp] -> [R][V] (logits_loc holds Rm*V floats when tp > 1)
      QOS_CU(launch_unshard_logits(lg, loc, R, e->sh.V, e->tp_size, st));
      lout = loc;
      }
    }
  }
  {
    TimerScope ts(e, QOS_T_ARGMAX, st);
    int32_t* am = reinterpret_cast<int32_t*>(e->ws + s.argmax);
    QOS_CU(launch_argmax(lout, 1, R, c.vocab, am, st, reinterpret_cast<float2*>(e->ws + s.am_part),
                         reinterpret_cast<int*>(e->ws + s.am_cnt)));
    if (next_tokens) {
      QOS_CU(cudaMemcpyAsync(next_tokens, am, size_t(R) * 4, out_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost,
                             st));
    }
  }
  if (logits && !direct) {
    if (logits_dtype == QOS_F32) {
      QOS_CU(cudaMemcpyAsync(logits, lout, size_t(R) * c.vocab * 4,
                             out_device ? cudaMemcpyDeviceToDevice : cudaMemcpyDeviceToHost, st));
    } else {
      void* dst = out_device ? logits : e->ws + s.act;  // act is free at this point
      QOS_CU(launch_f32_to_bf16(lout, dst, size_t(R) * c.vocab, st));
      if (!out_device) QOS_CU(cudaMemcpyAsync(logits, dst, size_t(R) * c.vocab * 2, cudaMemcpyDeviceToHost, st));
    }
  }
  return QOS_OK;
}

int do_step(qos_engine* e, const qos_batch* b, void* logits, int logits_dtype, int32_t* next_tokens, int on_host,
            cudaStream_t st, bool check_and_advance, const int32_t* dec_tokens_dev = nullptr) {
  if (logits && logits_dtype != QOS_F32 && logits_dtype != QOS_BF16)
    return set_error(QOS_ERR_INVALID_ARG, "logits_dtype");
  if (cudaSetDevice(e->device) != cudaSuccess) return set_error(QOS_ERR_CUDA, "cudaSetDevice");
  if (e->pending_upd.size() / 3 > 65536) QOS_TRY(flush_table_updates(e, st));  // step carries <= 64Ki
  QOS_TRY(acquire_staging(e));
  StepMeta m;
  int r = build_step(e, b, check_and_advance, e->h_meta[e->meta_cur], m);
  if (r != QOS_OK) {
    e->meta_cur ^= 1;  // staging not used
    return r;
  }
  uint8_t* dm = nullptr;
  {
    TimerScope ts(e, QOS_T_META, st);
    QOS_TRY(upload_meta(e, m, st, &dm));
    if (dec_tokens_dev && m.n_decode)  // decode rows are the last n_decode token rows
      QOS_CU(launch_token_patch(reinterpret_cast<int32_t*>(dm + m.o_tok) + (m.T - m.n_decode), dec_tokens_dev, m.n_decode,
                                e->cfg.vocab, st));
  }
  r = run_layers(e, m, dm, logits, logits_dtype, next_tokens, !on_host, st);
  if (r != QOS_OK) {
    if (e->group) e->group->abort();  // the peers would wait for this rank's collectives
    return r;
  }
  QOS_TRY(release_staging(e, st));
  QOS_CU(cudaEventRecord(e->ev_step_done, st));
  e->last_h2d = int64_t(m.used);
  e->last_d2h = on_host ? int64_t(m.R) * ((next_tokens ? 4 : 0) +
                                          (logits ? int64_t(e->cfg.vocab) * (logits_dtype == QOS_F32 ? 4 : 2) : 0))
                        : 0;
  if (check_and_advance) {
    for (int i = 0; i < b->n_prefill; ++i) e->reqs[b->prefill[i].req].cached += b->prefill[i].chunk_len;
    for (int i = 0; i < b->n_decode; ++i) e->reqs[b->decode[i].req].cached += 1;
  }
  if (on_host) QOS_CU(cudaStreamSynchronize(st));
  return QOS_OK;
}

}  // namespace

// =================================================================== C ABI
extern "C" {

const char* qos_strerror(int code) {
  switch (code) {
    case QOS_OK: return "ok";
    case QOS_ERR_INVALID_ARG: return "invalid argument";
    case QOS_ERR_OOM: return "out of memory";
    case QOS_ERR_UNKNOWN_REQ: return "unknown request";
    case QOS_ERR_BAD_KV_START: return "kv_start/ctx_len does not match cached length";
    case QOS_ERR_NOT_ALLOCATED: return "KV blocks not allocated";
    case QOS_ERR_CUDA: return "CUDA error";
    case QOS_ERR_COMM: return "communication error (NCCL or peer group)";
    case QOS_ERR_UNSUPPORTED: return "unsupported shape";
    default: return "unknown error";
  }
}
const char* qos_last_error(void) { return g_last_error.c_str(); }

int qos_engine_mem_sizes(const qos_model_cfg* cfg, int tp_size, qos_mem_sizes* out) {
  QOS_TRY(check_cfg(cfg, tp_size));
  if (!out) return set_error(QOS_ERR_INVALID_ARG, "out is NULL");
  Shard s = make_shard(*cfg, 0, tp_size);
  out->weight_bytes = weight_layout(*cfg, s).total;
  out->kv_bytes = uint64_t(cfg->n_layers) * 2 * cfg->num_blocks * s.Hkv * 16 * cfg->head_dim * 2;
  out->workspace_bytes = ws_layout(*cfg, s, tp_size).total;
  return QOS_OK;
}

int qos_shard_plan(const qos_model_cfg* cfg, int tp_rank, int tp_size, qos_shard* out) {
  QOS_TRY(check_cfg(cfg, tp_size));
  if (!out || tp_rank < 0 || tp_rank >= tp_size) return set_error(QOS_ERR_INVALID_ARG, "shard plan args");
  const Shard s = make_shard(*cfg, tp_rank, tp_size);
  *out = qos_shard{s.H, s.Hkv, s.F, s.V, s.h0, s.kv0, s.f0, s.v0};
  return QOS_OK;
}

int qos_nccl_unique_id(uint8_t out[128]) {
  std::lock_guard<std::mutex> g(g_nccl_mu);
  if (!g_nccl.load()) return set_error(QOS_ERR_COMM, "libnccl.so.2 not loadable");
  ncclUniqueId id;
  if (g_nccl.getUniqueId(&id) != ncclSuccess) return set_error(QOS_ERR_COMM, "ncclGetUniqueId failed");
  memcpy(out, &id, 128);
  return QOS_OK;
}

int qos_group_create(int tp_size, qos_group_t** out) {
  if (!out || tp_size < 2 || tp_size > kMaxPeers) return set_error(QOS_ERR_INVALID_ARG, "group size must be 2..8");
  auto* g = new qos_group();
  g->n = tp_size;
  g->eng.assign(size_t(tp_size), nullptr);
  if (const char* t = getenv("QOS_GROUP_TIMEOUT_MS")) g->timeout_ms = atoi(t);
  *out = g;
  return QOS_OK;
}

int qos_group_destroy(qos_group_t* g) {
  if (!g) return QOS_OK;
  {
    std::lock_guard<std::mutex> lk(g->mu);
    for (auto* e : g->eng)
      if (e) return set_error(QOS_ERR_INVALID_ARG, "destroy the group's engines first");
  }
  if (g->ipc && g->shm) {
    if (g->shm->attached.fetch_sub(1, std::memory_order_acq_rel) == 1) shm_unlink(g->shm_name.c_str());
    munmap(g->shm, sizeof(IpcShm));
  }
  delete g;
  return QOS_OK;
}

int qos_group_unique_id(uint8_t out[64]) {
  if (!out) return set_error(QOS_ERR_INVALID_ARG, "out is NULL");
  std::random_device rd;
  const unsigned long long r = (uint64_t(rd()) << 32) ^ rd();
  char name[64];
  snprintf(name, sizeof name, "/qoserve_grp_%d_%016llx", int(getpid()), r);
  memset(out, 0, 64);
  memcpy(out, name, strlen(name));
  return QOS_OK;
}

int qos_group_open(const uint8_t id[64], int tp_size, int tp_rank, qos_group_t** out) {
  if (!id || !out || tp_size < 2 || tp_size > kMaxPeers || tp_rank < 0 || tp_rank >= tp_size)
    return set_error(QOS_ERR_INVALID_ARG, "group id / size 2..8 / rank");
  const std::string name(reinterpret_cast<const char*>(id), strnlen(reinterpret_cast<const char*>(id), 64));
  if (name.size() < 2 || name[0] != '/' || name.size() >= 64) return set_error(QOS_ERR_INVALID_ARG, "group id");
  auto g = std::make_unique<qos_group>();
  g->n = tp_size;
  g->ipc = true;
  g->rank = tp_rank;
  g->shm_name = name;
  g->eng.assign(size_t(tp_size), nullptr);
  if (const char* t = getenv("QOS_GROUP_TIMEOUT_MS")) g->timeout_ms = atoi(t);
  const auto t0 = std::chrono::steady_clock::now();
  auto timed_out = [&] { return std::chrono::steady_clock::now() - t0 > std::chrono::milliseconds(g->timeout_ms); };
  int fd = -1;
  if (tp_rank == 0) {
    fd = shm_open(name.c_str(), O_CREAT | O_EXCL | O_RDWR, 0600);
    if (fd < 0) return set_error(QOS_ERR_COMM, "shm_open (create) of the group segment failed");
    if (ftruncate(fd, sizeof(IpcShm)) != 0) {
      close(fd);
      shm_unlink(name.c_str());
      return set_error(QOS_ERR_COMM, "ftruncate of the group segment failed");
    }
  } else {  // wait for rank 0's segment to exist at full size
    for (;;) {
      fd = shm_open(name.c_str(), O_RDWR, 0600);
      if (fd >= 0) {
        struct stat st {};
        if (fstat(fd, &st) == 0 && size_t(st.st_size) >= sizeof(IpcShm)) break;
        close(fd);
        fd = -1;
      }
      if (timed_out()) return set_error(QOS_ERR_COMM, "group segment never appeared (rank 0 did not open the group)");
      usleep(1000);
    }
  }
  void* m = mmap(nullptr, sizeof(IpcShm), PROT_READ | PROT_WRITE, MAP_SHARED, fd, 0);
  close(fd);
  if (m == MAP_FAILED) return set_error(QOS_ERR_COMM, "mmap of the group segment failed");
  g->shm = static_cast<IpcShm*>(m);
  if (tp_rank == 0) {
    memset(m, 0, sizeof(IpcShm));
    g->shm->n = tp_size;
    g->shm->magic.store(IpcShm::kMagic, std::memory_order_release);
  } else {
    while (g->shm->magic.load(std::memory_order_acquire) != IpcShm::kMagic) {
      if (timed_out()) {
        munmap(m, sizeof(IpcShm));
        return set_error(QOS_ERR_COMM, "group segment never initialised");
      }
      usleep(1000);
    }
    if (g->shm->n != tp_size) {
      munmap(m, sizeof(IpcShm));
      return set_error(QOS_ERR_INVALID_ARG, "tp_size differs from rank 0's");
    }
  }
  g->shm->attached.fetch_add(1, std::memory_order_acq_rel);
  *out = g.release();
  return QOS_OK;
}

// Cross-process group: export this rank's workspace + sync events, meet the peers, open theirs.
using PFN_memGetAddressRange = CUresult (*)(CUdeviceptr*, size_t*, CUdeviceptr);
static int ipc_attach(qos_engine* e, qos_group* g) {
  if (e->tp_rank != g->rank) return set_error(QOS_ERR_INVALID_ARG, "tp_rank differs from the group rank");
  for (int i = 0; i < 2; ++i)
    QOS_CU(cudaEventCreateWithFlags(&e->ev_coll[i], cudaEventDisableTiming | cudaEventInterprocess));
  static PFN_memGetAddressRange range = nullptr;
  if (!range) {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      return set_error(QOS_ERR_CUDA, "cuMemGetAddressRange unavailable");
    range = reinterpret_cast<PFN_memGetAddressRange>(fn);
  }
  CUdeviceptr base = 0;
  size_t bytes = 0;
  if (range(&base, &bytes, CUdeviceptr(e->ws)) != CUDA_SUCCESS) return set_error(QOS_ERR_CUDA, "workspace range");
  IpcSlot& me = g->shm->slot[e->tp_rank];
  QOS_CU(cudaIpcGetMemHandle(&me.ws, reinterpret_cast<void*>(base)));
  me.ws_off = uint64_t(CUdeviceptr(e->ws) - base);
  for (int i = 0; i < 2; ++i) QOS_CU(cudaIpcGetEventHandle(&me.ev[i], e->ev_coll[i]));
  cudaDeviceProp prop{};
  QOS_CU(cudaGetDeviceProperties(&prop, e->device));
  memcpy(me.uuid, &prop.uuid, 16);
  me.cfg = e->cfg;
  QOS_TRY(g->barrier());  // every rank has published its slot
  e->ipc_ws.assign(size_t(g->n), nullptr);
  e->ipc_base.assign(size_t(g->n), nullptr);
  e->ipc_ev.assign(size_t(g->n), {nullptr, nullptr});
  for (int k = 0; k < g->n; ++k) {
    if (k == e->tp_rank) continue;
    const IpcSlot& p = g->shm->slot[k];
    if (std::memcmp(&p.cfg, &e->cfg, sizeof(e->cfg)) != 0) {
      g->abort();
      return set_error(QOS_ERR_INVALID_ARG, "group ranks need identical model configs");
    }
    if (std::memcmp(p.uuid, me.uuid, 16) == 0) e->shares_device = true;
    void* ptr = nullptr;
    cudaError_t er = cudaIpcOpenMemHandle(&ptr, p.ws, cudaIpcMemLazyEnablePeerAccess);
    if (er != cudaSuccess) {
      g->abort();
      return set_cuda_error(er, "cudaIpcOpenMemHandle (peer workspace)");
    }
    e->ipc_base[size_t(k)] = static_cast<uint8_t*>(ptr);
    e->ipc_ws[size_t(k)] = static_cast<uint8_t*>(ptr) + p.ws_off;
    for (int i = 0; i < 2; ++i) {
      er = cudaIpcOpenEventHandle(&e->ipc_ev[size_t(k)][size_t(i)], p.ev[i]);
      if (er != cudaSuccess) {
        g->abort();
        return set_cuda_error(er, "cudaIpcOpenEventHandle (peer sync event)");
      }
    }
  }
  QOS_TRY(g->barrier());  // every rank has mapped its peers
  g->eng[size_t(e->tp_rank)] = e;
  e->group = g;
  return QOS_OK;
}

static int create_engine(const qos_model_cfg* cfg, int device, int tp_rank, int tp_size, const uint8_t* nccl_uid,
                         qos_group* group, const qos_mem* mem, qos_engine_t** out) {
  QOS_TRY(check_cfg(cfg, tp_size));
  if (!out) return set_error(QOS_ERR_INVALID_ARG, "out is NULL");
  if (tp_rank < 0 || tp_rank >= tp_size) return set_error(QOS_ERR_INVALID_ARG, "tp_rank");
  if (tp_size > 1 && !nccl_uid && !group) return set_error(QOS_ERR_INVALID_ARG, "nccl_uid required for tp_size > 1");
  QOS_CU(cudaSetDevice(device));
  auto* e = new qos_engine();
  e->cfg = *cfg;
  e->device = device;
  e->tp_rank = tp_rank;
  e->tp_size = tp_size;
  cudaDeviceGetAttribute(&e->num_sms, cudaDevAttrMultiProcessorCount, device);
  e->sh = make_shard(*cfg, tp_rank, tp_size);
  e->nqkv = (e->sh.H + 2 * e->sh.Hkv) * cfg->head_dim;
  e->table_w = (cfg->max_seq_len + 15) / 16;
  e->wl = weight_layout(*cfg, e->sh);
  e->wsl = ws_layout(*cfg, e->sh, tp_size);
  e->plane_elems = size_t(cfg->num_blocks) * e->sh.Hkv * 16 * cfg->head_dim;
  e->kv_bytes = uint64_t(cfg->n_layers) * 2 * e->plane_elems * 2;
  auto fail = [&](int code) {
    qos_engine_destroy(e);
    return code;
  };
  auto get = [&](void* given, size_t bytes, uint8_t** dst, bool* own) -> int {
    if (given) {
      *dst = reinterpret_cast<uint8_t*>(given);
      *own = false;
      return QOS_OK;
    }
    void* p = nullptr;
    cudaError_t er = cudaMalloc(&p, bytes);
    if (er != cudaSuccess) return set_error(QOS_ERR_OOM, "cudaMalloc of an engine arena failed");
    *dst = reinterpret_cast<uint8_t*>(p);
    *own = true;
    return QOS_OK;
  };
  int r;
  if ((r = get(mem ? mem->weights : nullptr, e->wl.total, &e->w, &e->own_w)) != QOS_OK) return fail(r);
  if ((r = get(mem ? mem->kv : nullptr, e->kv_bytes, &e->kv, &e->own_kv)) != QOS_OK) return fail(r);
  if ((r = get(mem ? mem->workspace : nullptr, e->wsl.total, &e->ws, &e->own_ws)) != QOS_OK) return fail(r);
  // zero the KV pool once: slots past a request's length are read (with P = 0) by the attention
  // tiles, and 0 * NaN from uninitialised memory would poison the accumulators
  if (cudaMemset(e->kv, 0, e->kv_bytes) != cudaSuccess) return fail(set_error(QOS_ERR_CUDA, "kv memset"));
  // split-K arrival counters start at zero; the combining item / reducing CTA resets its counter
  if (cudaMemset(e->ws + e->wsl.counters, 0, size_t(cfg->max_batch_rows) * e->sh.Hkv * 4) != cudaSuccess ||
      cudaMemset(e->ws + e->wsl.gemm_cnt, 0, size_t(kGemmMaxTiles) * 4) != cudaSuccess ||
      cudaMemset(e->ws + e->wsl.gemm_cnt2, 0, size_t(kGemmMaxTiles) * 4) != cudaSuccess ||
      cudaMemset(e->ws + e->wsl.ss[0], 0, size_t(cfg->max_batch_tokens) * kFoldSlots * 4) != cudaSuccess ||
      cudaMemset(e->ws + e->wsl.ss[1], 0, size_t(cfg->max_batch_tokens) * kFoldSlots * 4) != cudaSuccess ||
      cudaMemset(e->ws + e->wsl.fcnt, 0, size_t(cfg->max_batch_tokens / 128 + 2) * 4) != cudaSuccess ||
      cudaMemset(e->ws + e->wsl.am_cnt, 0, size_t(cfg->max_batch_rows) * 4) != cudaSuccess)
    return fail(set_error(QOS_ERR_CUDA, "counter memset"));
  if (cudaMalloc(&e->d_tables, size_t(cfg->max_requests) * e->table_w * 4) != cudaSuccess)
    return fail(set_error(QOS_ERR_OOM, "block tables"));
  cudaMemset(e->d_tables, 0, size_t(cfg->max_requests) * e->table_w * 4);
  // RoPE table in fp64 -> fp32 (reading s2)
  {
    const int half = cfg->head_dim / 2;
    std::vector<float2> tab(size_t(cfg->max_seq_len) * half);
    for (int p = 0; p < cfg->max_seq_len; ++p)
      for (int i = 0; i < half; ++i) {
        const double inv = std::pow(double(cfg->rope_theta), -2.0 * i / cfg->head_dim);
        const double a = double(p) * inv;
        tab[size_t(p) * half + i] = make_float2(float(std::cos(a)), float(std::sin(a)));
      }
    if (cudaMalloc(&e->rope_tab, tab.size() * sizeof(float2)) != cudaSuccess)
      return fail(set_error(QOS_ERR_OOM, "rope table"));
    cudaMemcpy(e->rope_tab, tab.data(), tab.size() * sizeof(float2), cudaMemcpyHostToDevice);
  }
  for (int i = 0; i < 2; ++i) {
    if (cudaMallocHost(&e->h_meta[i], e->wsl.meta_bytes) != cudaSuccess) return fail(set_error(QOS_ERR_OOM, "pinned"));
    cudaEventCreateWithFlags(&e->meta_free[i], cudaEventDisableTiming);
  }
  cudaStreamCreateWithFlags(&e->stream, cudaStreamNonBlocking);
  if (const char* ov = getenv("QOS_OVERLAP_ATTN")) e->overlap_attn = atoi(ov) != 0;
  if (const char* sk = getenv("QOS_GEMM_SPLITK")) e->gemm_splitk = atoi(sk) != 0;
  if (const char* sw = getenv("QOS_GEMM_SWAB")) e->gemm_swab = atoi(sw);
  if (const char* sk = getenv("QOS_GEMM_STREAMK")) e->gemm_streamk = atoi(sk);
  if (const char* du = getenv("QOS_DUAL")) e->dual_stream = atoi(du) != 0;
  if (const char* as = getenv("QOS_ADD_SPLIT")) e->add_split = atoi(as) != 0;
  if (const char* a = getenv("QOS_DUAL_MIN_PREFILL")) e->dual_min_prefill = atoi(a);
  if (const char* a = getenv("QOS_DUAL_MIN_DECODE")) e->dual_min_decode = atoi(a);
  if (const char* a = getenv("QOS_DUAL_SMS_PRE")) e->dual_sms_pre = atoi(a);
  if (const char* a = getenv("QOS_DUAL_SMS_DEC")) e->dual_sms_dec = atoi(a);
  {
    int lo = 0, hi = 0;
    cudaDeviceGetStreamPriorityRange(&lo, &hi);
    cudaStreamCreateWithPriority(&e->side, cudaStreamNonBlocking, hi);
    cudaStreamCreateWithPriority(&e->side_lo, cudaStreamNonBlocking, lo);
    cudaEventCreateWithFlags(&e->ev_fork, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&e->ev_join, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&e->ev_fork2, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&e->ev_join2, cudaEventDisableTiming);
    cudaEventCreateWithFlags(&e->ev_step_done, cudaEventDisableTiming);
  }
  e->free_heap.resize(size_t(cfg->num_blocks));
  for (int64_t i = 0; i < cfg->num_blocks; ++i) e->free_heap[size_t(i)] = int32_t(i);  // sorted = valid min-heap
  e->free_rows.resize(size_t(cfg->max_requests));
  for (int i = 0; i < cfg->max_requests; ++i) e->free_rows[size_t(i)] = i;
  if ((r = build_maps(e)) != QOS_OK) return fail(r);
  if (group && group->ipc) {
    if ((r = ipc_attach(e, group)) != QOS_OK) return fail(r);
  } else if (group) {
    for (int i = 0; i < 2; ++i) cudaEventCreateWithFlags(&e->ev_coll[i], cudaEventDisableTiming);
    std::lock_guard<std::mutex> lk(group->mu);
    if (group->eng[size_t(tp_rank)]) return fail(set_error(QOS_ERR_INVALID_ARG, "tp_rank already in the group"));
    for (auto* p : group->eng) {
      if (!p) continue;
      if (std::memcmp(&p->cfg, cfg, sizeof(*cfg)) != 0)
        return fail(set_error(QOS_ERR_INVALID_ARG, "group ranks need identical model configs"));
      if (p->device == device) p->shares_device = e->shares_device = true;
      if (p->device != device) {  // peer reads in both directions over NVLink
        int ok1 = 0, ok2 = 0;
        cudaDeviceCanAccessPeer(&ok1, device, p->device);
        cudaDeviceCanAccessPeer(&ok2, p->device, device);
        if (!ok1 || !ok2) return fail(set_error(QOS_ERR_UNSUPPORTED, "group devices lack peer access"));
        cudaError_t a = cudaDeviceEnablePeerAccess(p->device, 0);
        if (a != cudaSuccess && a != cudaErrorPeerAccessAlreadyEnabled) return fail(set_cuda_error(a, "peer access"));
        cudaSetDevice(p->device);
        a = cudaDeviceEnablePeerAccess(device, 0);
        cudaSetDevice(device);
        if (a != cudaSuccess && a != cudaErrorPeerAccessAlreadyEnabled) return fail(set_cuda_error(a, "peer access"));
        cudaGetLastError();
      }
    }
    group->eng[size_t(tp_rank)] = e;
    e->group = group;
  } else if (tp_size > 1) {
    std::lock_guard<std::mutex> g(g_nccl_mu);
    if (!g_nccl.load()) return fail(set_error(QOS_ERR_COMM, "libnccl.so.2 not loadable"));
    ncclUniqueId id;
    memcpy(&id, nccl_uid, 128);
    if (g_nccl.commInitRank(&e->comm, tp_size, id, tp_rank) != ncclSuccess)
      return fail(set_error(QOS_ERR_COMM, "ncclCommInitRank failed"));
  }
  if (cudaDeviceSynchronize() != cudaSuccess) return fail(set_error(QOS_ERR_CUDA, "engine init"));
  *out = e;
  return QOS_OK;
}

int qos_engine_create(const qos_model_cfg* cfg, int device, int tp_rank, int tp_size, const uint8_t* nccl_uid,
                      const qos_mem* mem, qos_engine_t** out) {
  return create_engine(cfg, device, tp_rank, tp_size, nccl_uid, nullptr, mem, out);
}

int qos_engine_create_peer(const qos_model_cfg* cfg, int device, int tp_rank, qos_group_t* group, const qos_mem* mem,
                           qos_engine_t** out) {
  if (!group) return set_error(QOS_ERR_INVALID_ARG, "group is NULL");
  return create_engine(cfg, device, tp_rank, group->n, nullptr, group, mem, out);
}

int qos_engine_destroy(qos_engine_t* e) {
  if (!e) return QOS_OK;
  cudaSetDevice(e->device);
  cudaDeviceSynchronize();
  if (e->group && e->group->ipc) {
    e->group->barrier();  // no peer still reads this workspace (errors ignored: a dead peer)
    for (auto* b : e->ipc_base)
      if (b) cudaIpcCloseMemHandle(b);
    for (auto& evs : e->ipc_ev)
      for (auto ev : evs)
        if (ev) cudaEventDestroy(ev);
  }
  if (e->group) {
    std::lock_guard<std::mutex> lk(e->group->mu);
    if (e->group->eng[size_t(e->tp_rank)] == e) e->group->eng[size_t(e->tp_rank)] = nullptr;
  }
  for (auto ev : e->ev_coll)
    if (ev) cudaEventDestroy(ev);
  if (e->comm && g_nccl.commDestroy) g_nccl.commDestroy(e->comm);
  if (e->own_w) cudaFree(e->w);
  if (e->own_kv) cudaFree(e->kv);
  if (e->own_ws) cudaFree(e->ws);
  if (e->d_tables) cudaFree(e->d_tables);
  if (e->rope_tab) cudaFree(e->rope_tab);
  if (e->dbg) cudaFree(e->dbg);
  for (int i = 0; i < 2; ++i) {
    if (e->h_meta[i]) cudaFreeHost(e->h_meta[i]);
    if (e->meta_free[i]) cudaEventDestroy(e->meta_free[i]);
  }
  for (auto ev : e->ev_pool) cudaEventDestroy(ev);
  if (e->stream) cudaStreamDestroy(e->stream);
  if (e->side) cudaStreamDestroy(e->side);
  if (e->side_lo) cudaStreamDestroy(e->side_lo);
  if (e->ev_fork) cudaEventDestroy(e->ev_fork);
  if (e->ev_join) cudaEventDestroy(e->ev_join);
  if (e->ev_fork2) cudaEventDestroy(e->ev_fork2);
  if (e->ev_join2) cudaEventDestroy(e->ev_join2);
  if (e->ev_step_done) cudaEventDestroy(e->ev_step_done);
  delete e;
  return QOS_OK;
}

int qos_engine_load_synthetic(qos_engine_t* e, uint64_t seed) {
  if (!e) return set_error(QOS_ERR_INVALID_ARG, "engine is NULL");
  QOS_CU(cudaSetDevice(e->device));
  const auto& c = e->cfg;
  const auto& sh = e->sh;
  const int d = c.d_model, hd = c.head_dim;
  cudaStream_t st = internal_stream(e);
  char name[256];
  auto H = [&](const char* s) { return fnv1a64(s); };
  for (int l = 0; l < c.n_layers; ++l) {
    const auto& L = e->wl.layers[l];
    snprintf(name, sizeof name, "model.layers.%d.input_layernorm.weight", l);
    QOS_CU(gen_fill_bf16(W(e, L.ln1), d, 1, d, seed, H(name), 0, 0, d, GEN_NORM, 1, st));
    snprintf(name, sizeof name, "model.layers.%d.post_attention_layernorm.weight", l);
    QOS_CU(gen_fill_bf16(W(e, L.ln2), d, 1, d, seed, H(name), 0, 0, d, GEN_NORM, 1, st));
    // fused QKV [q rows | k rows | v rows] of this rank's heads
    __nv_bfloat16* wqkv = W(e, L.wqkv);
    snprintf(name, sizeof name, "model.layers.%d.self_attn.q_proj.weight", l);
    QOS_CU(gen_fill_bf16(wqkv, d, int64_t(sh.H) * hd, d, seed, H(name), int64_t(sh.h0) * hd, 0, d, GEN_LINEAR, d, st));
    snprintf(name, sizeof name, "model.layers.%d.self_attn.k_proj.weight", l);
    QOS_CU(gen_fill_bf16(wqkv + size_t(sh.H) * hd * d, d, int64_t(sh.Hkv) * hd, d, seed, H(name),
                         int64_t(sh.kv0) * hd, 0, d, GEN_LINEAR, d, st));
    snprintf(name, sizeof name, "model.layers.%d.self_attn.v_proj.weight", l);
    QOS_CU(gen_fill_bf16(wqkv + size_t(sh.H + sh.Hkv) * hd * d, d, int64_t(sh.Hkv) * hd, d, seed, H(name),
                         int64_t(sh.kv0) * hd, 0, d, GEN_LINEAR, d, st));
    if (c.qkv_bias) {
      float* b = reinterpret_cast<float*>(e->w + L.bqkv);
      snprintf(name, sizeof name, "model.layers.%d.self_attn.q_proj.bias", l);
      QOS_CU(gen_fill_f32_bias(b, int64_t(sh.H) * hd, seed, H(name), int64_t(sh.h0) * hd, st));
      snprintf(name, sizeof name, "model.layers.%d.self_attn.k_proj.bias", l);
      QOS_CU(gen_fill_f32_bias(b + sh.H * hd, int64_t(sh.Hkv) * hd, seed, H(name), int64_t(sh.kv0) * hd, st));
      snprintf(name, sizeof name, "model.layers.%d.self_attn.v_proj.bias", l);
      QOS_CU(gen_fill_f32_bias(b + (sh.H + sh.Hkv) * hd, int64_t(sh.Hkv) * hd, seed, H(name), int64_t(sh.kv0) * hd, st));
    }
    // o_proj [d][H*hd]: this rank's columns
    snprintf(name, sizeof name, "model.layers.%d.self_attn.o_proj.weight", l);
    QOS_CU(gen_fill_bf16(W(e, L.wo), int64_t(sh.H) * hd, d, int64_t(sh.H) * hd, seed, H(name), 0, int64_t(sh.h0) * hd,
                         int64_t(c.n_heads) * hd, GEN_LINEAR, c.n_heads * hd, st));
    // gate/up interleaved in groups of 64 rows (QOS_EPI_SILU_GATE layout)
    snprintf(name, sizeof name, "model.layers.%d.mlp.gate_proj.weight", l);
    QOS_CU(gen_fill_bf16_ex(W(e, L.wgu), d, sh.F, d, seed, H(name), sh.f0, 0, d, GEN_LINEAR, d, 0, st));
    snprintf(name, sizeof name, "model.layers.%d.mlp.up_proj.weight", l);
    QOS_CU(gen_fill_bf16_ex(W(e, L.wgu), d, sh.F, d, seed, H(name), sh.f0, 0, d, GEN_LINEAR, d, 1, st));
    // down_proj [d][F]: this rank's columns
    snprintf(name, sizeof name, "model.layers.%d.mlp.down_proj.weight", l);
    QOS_CU(gen_fill_bf16(W(e, L.wd), sh.F, d, sh.F, seed, H(name), 0, sh.f0, c.ffn_dim, GEN_LINEAR, c.ffn_dim, st));
  }
  QOS_CU(gen_fill_bf16(W(e, e->wl.emb), d, c.vocab, d, seed, H("model.embed_tokens.weight"), 0, 0, d, GEN_EMBED, 1, st));
  QOS_CU(gen_fill_bf16(W(e, e->wl.lnf), d, 1, d, seed, H("model.norm.weight"), 0, 0, d, GEN_NORM, 1, st));
  QOS_CU(gen_fill_bf16(W(e, e->wl.head), d, sh.V, d, seed, H("lm_head.weight"), sh.v0, 0, d, GEN_LINEAR, d, st));
  QOS_CU(cudaStreamSynchronize(st));
  return QOS_OK;
}

int qos_engine_read_weight(qos_engine_t* e, const char* name, int64_t row0, int64_t nrows, uint16_t* out) {
  if (!e || !name || !out || row0 < 0 || nrows < 0) return set_error(QOS_ERR_INVALID_ARG, "read_weight args");
  QOS_CU(cudaSetDevice(e->device));
  const auto& c = e->cfg;
  const auto& sh = e->sh;
  const int d = c.d_model, hd = c.head_dim;
  std::string n(name);
  // generic: (device base, rows, cols, row stride, row remap)
  const __nv_bfloat16* base = nullptr;
  int64_t rows = 0, cols = 0, ld = 0;
  int interleave = -1;
  int layer = -1;
  char suffix[128] = {0};
  if (sscanf(name, "model.layers.%d.%127s", &layer, suffix) == 2) {
    if (layer < 0 || layer >= c.n_layers) return set_error(QOS_ERR_INVALID_ARG, "layer");
    const auto& L = e->wl.layers[layer];
    std::string s(suffix);
    if (s == "input_layernorm.weight") { base = W(e, L.ln1); rows = 1; cols = d; ld = d; }
    else if (s == "post_attention_layernorm.weight") { base = W(e, L.ln2); rows = 1; cols = d; ld = d; }
    else if (s == "self_attn.q_proj.weight") { base = W(e, L.wqkv); rows = int64_t(sh.H) * hd; cols = d; ld = d; }
    else if (s == "self_attn.k_proj.weight") { base = W(e, L.wqkv) + size_t(sh.H) * hd * d; rows = int64_t(sh.Hkv) * hd; cols = d; ld = d; }
    else if (s == "self_attn.v_proj.weight") { base = W(e, L.wqkv) + size_t(sh.H + sh.Hkv) * hd * d; rows = int64_t(sh.Hkv) * hd; cols = d; ld = d; }
    else if (s == "self_attn.o_proj.weight") { base = W(e, L.wo); rows = d; cols = int64_t(sh.H) * hd; ld = cols; }
    else if (s == "mlp.gate_proj.weight") { base = W(e, L.wgu); rows = sh.F; cols = d; ld = d; interleave = 0; }
    else if (s == "mlp.up_proj.weight") { base = W(e, L.wgu); rows = sh.F; cols = d; ld = d; interleave = 1; }
    else if (s == "mlp.down_proj.weight") { base = W(e, L.wd); rows = d; cols = sh.F; ld = cols; }
    else return set_error(QOS_ERR_INVALID_ARG, "unknown tensor name");
  } else if (n == "model.embed_tokens.weight") { base = W(e, e->wl.emb); rows = c.vocab; cols = d; ld = d; }
  else if (n == "model.norm.weight") { base = W(e, e->wl.lnf); rows = 1; cols = d; ld = d; }
  else if (n == "lm_head.weight") { base = W(e, e->wl.head); rows = sh.V; cols = d; ld = d; }
  else return set_error(QOS_ERR_INVALID_ARG, "unknown tensor name");
  if (row0 + nrows > rows) return set_error(QOS_ERR_INVALID_ARG, "row range");
  for (int64_t r = 0; r < nrows; ++r) {
    int64_t sr = row0 + r;
    int64_t dr = interleave >= 0 ? (sr / 64) * 128 + interleave * 64 + sr % 64 : sr;
    QOS_CU(cudaMemcpy(out + r * cols, base + dr * ld, size_t(cols) * 2, cudaMemcpyDeviceToHost));
  }
  return QOS_OK;
}

// ------------------------------------------------------------------ KV allocator
int qos_kv_alloc(qos_engine_t* e, int64_t req, int32_t n_tokens_total) {
  if (!e || n_tokens_total < 0) return set_error(QOS_ERR_INVALID_ARG, "kv_alloc args");
  if (n_tokens_total > e->cfg.max_seq_len) return set_error(QOS_ERR_INVALID_ARG, "n_tokens_total > max_seq_len");
  const int need_total = (n_tokens_total + 15) / 16;
  auto it = e->reqs.find(req);
  const int have = it == e->reqs.end() ? 0 : int(it->second.blocks.size());
  const int need = need_total - have;
  if (need > int64_t(e->free_heap.size())) return set_error(QOS_ERR_OOM, "KV pool exhausted");
  if (it == e->reqs.end()) {
    if (e->free_rows.empty()) return set_error(QOS_ERR_OOM, "max_requests reached");
    ReqState rs;
    rs.row = alloc_table_row(e);
    it = e->reqs.emplace(req, std::move(rs)).first;
  }
  ReqState& rs = it->second;
  for (int k = 0; k < need; ++k) {
    std::pop_heap(e->free_heap.begin(), e->free_heap.end(), std::greater<int32_t>());
    const int32_t blk = e->free_heap.back();
    e->free_heap.pop_back();
    const int col = int(rs.blocks.size());
    rs.blocks.push_back(blk);
    e->pending_upd.push_back(rs.row);
    e->pending_upd.push_back(col);
    e->pending_upd.push_back(blk);
  }
  return QOS_OK;
}

int qos_kv_free(qos_engine_t* e, int64_t req) {
  if (!e) return set_error(QOS_ERR_INVALID_ARG, "engine is NULL");
  auto it = e->reqs.find(req);
  if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "unknown request");
  // table updates of this row not yet on the device are obsolete: drop them so a later owner
  // of the row can never be overwritten by them (the update kernel applies triples unordered)
  {
    const int row = it->second.row;
    size_t w = 0;
    for (size_t i = 0; i < e->pending_upd.size(); i += 3)
      if (e->pending_upd[i] != row) {
        e->pending_upd[w] = e->pending_upd[i];
        e->pending_upd[w + 1] = e->pending_upd[i + 1];
        e->pending_upd[w + 2] = e->pending_upd[i + 2];
        w += 3;
      }
    e->pending_upd.resize(w);
  }
  for (int32_t b : it->second.blocks) {
    e->free_heap.push_back(b);
    std::push_heap(e->free_heap.begin(), e->free_heap.end(), std::greater<int32_t>());
  }
  e->free_rows.push_back(it->second.row);
  std::push_heap(e->free_rows.begin(), e->free_rows.end(), std::greater<int>());
  e->reqs.erase(it);
  return QOS_OK;
}

int qos_kv_table(qos_engine_t* e, int64_t req, int32_t* out, int32_t cap, int32_t* n_out) {
  if (!e || !n_out || (cap > 0 && !out)) return set_error(QOS_ERR_INVALID_ARG, "kv_table args");
  auto it = e->reqs.find(req);
  if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "unknown request");
  const auto& b = it->second.blocks;
  *n_out = int32_t(b.size());
  for (int32_t i = 0; i < cap && i < int32_t(b.size()); ++i) out[i] = b[size_t(i)];
  return QOS_OK;
}

int qos_kv_table_device(qos_engine_t* e, int64_t req, int32_t* out, int32_t cap, int32_t* n_out) {
  if (!e || !n_out || (cap > 0 && !out)) return set_error(QOS_ERR_INVALID_ARG, "kv_table_device args");
  auto it = e->reqs.find(req);
  if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "unknown request");
  QOS_CU(cudaSetDevice(e->device));
  QOS_TRY(flush_table_updates(e, internal_stream(e)));
  QOS_CU(cudaStreamSynchronize(e->stream));
  const int n = int(it->second.blocks.size());
  *n_out = n;
  const int k = std::min(n, int(cap));
  if (k > 0) QOS_CU(cudaMemcpy(out, e->d_tables + size_t(it->second.row) * e->table_w, size_t(k) * 4, cudaMemcpyDeviceToHost));
  return QOS_OK;
}

int qos_kv_cached_len(qos_engine_t* e, int64_t req, int32_t* out) {
  if (!e || !out) return set_error(QOS_ERR_INVALID_ARG, "args");
  auto it = e->reqs.find(req);
  if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "unknown request");
  *out = it->second.cached;
  return QOS_OK;
}

int qos_kv_free_blocks(qos_engine_t* e, int64_t* out) {
  if (!e || !out) return set_error(QOS_ERR_INVALID_ARG, "args");
  *out = int64_t(e->free_heap.size());
  return QOS_OK;
}

int qos_kv_fill_synthetic(qos_engine_t* e, int64_t req, int32_t n_tokens, uint64_t seed) {
  if (!e || n_tokens < 0) return set_error(QOS_ERR_INVALID_ARG, "args");
  auto it = e->reqs.find(req);
  if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "unknown request");
  if (int64_t(it->second.blocks.size()) * 16 < n_tokens) return set_error(QOS_ERR_NOT_ALLOCATED, "not allocated");
  QOS_CU(cudaSetDevice(e->device));
  cudaStream_t st = internal_stream(e);
  QOS_TRY(flush_table_updates(e, st));
  const int32_t* trow = e->d_tables + size_t(it->second.row) * e->table_w;
  char name[128];
  for (int l = 0; l < e->cfg.n_layers; ++l)
    for (int kv = 0; kv < 2; ++kv) {
      snprintf(name, sizeof name, "kvfill.%d.%c.%lld", l, kv ? 'v' : 'k', (long long)req);
      void* plane = reinterpret_cast<__nv_bfloat16*>(e->kv) + (size_t(l) * 2 + kv) * e->plane_elems;
      QOS_CU(kvfill_launch(plane, trow, n_tokens, e->sh.Hkv, e->cfg.n_kv_heads, e->sh.kv0, e->cfg.head_dim, seed,
                           fnv1a64(name), kv, st));
    }
  QOS_CU(cudaStreamSynchronize(st));
  it->second.cached = n_tokens;
  return QOS_OK;
}

// ------------------------------------------------------------------ step / profile / timing
int qos_hybrid_step(qos_engine_t* e, const qos_batch* batch, void* logits, int logits_dtype, int32_t* next_tokens,
                    int outputs_on_host, void* stream) {
  if (!e) return set_error(QOS_ERR_INVALID_ARG, "engine is NULL");
  return do_step(e, batch, logits, logits_dtype, next_tokens, outputs_on_host, reinterpret_cast<cudaStream_t>(stream),
                 true);
}

int qos_hybrid_step_ex(qos_engine_t* e, const qos_batch* batch, void* logits, int logits_dtype, int32_t* next_tokens,
                       int outputs_on_host, void* stream, const int32_t* decode_tokens_dev) {
  if (!e) return set_error(QOS_ERR_INVALID_ARG, "engine is NULL");
  return do_step(e, batch, logits, logits_dtype, next_tokens, outputs_on_host, reinterpret_cast<cudaStream_t>(stream),
                 true, decode_tokens_dev);
}

int qos_profile_step_ex(qos_engine_t* e, int32_t chunk_len, int32_t kv_start, int32_t n_decode,
                        const int32_t* ctx_lens, int32_t warmup, int32_t reps, float* ms_median, float* ms_p95) {
  if (warmup < 0) warmup = 3;
  if (!e || chunk_len < 0 || kv_start < 0 || n_decode < 0 || (n_decode && !ctx_lens) || reps < 1 || !ms_median)
    return set_error(QOS_ERR_INVALID_ARG, "profile args");
  if (chunk_len == 0 && n_decode == 0) return set_error(QOS_ERR_INVALID_ARG, "empty profile batch");
  QOS_CU(cudaSetDevice(e->device));
  const int64_t base = INT64_MIN + 1024;  // reserved scratch id range
  std::vector<int64_t> ids;
  auto cleanup = [&]() {
    for (int64_t id : ids) qos_kv_free(e, id);
  };
  std::vector<int32_t> toks(static_cast<size_t>(chunk_len));
  for (int i = 0; i < chunk_len; ++i) toks[size_t(i)] = int32_t((int64_t(i) * 7919 + 13) % e->cfg.vocab);
  qos_prefill_chunk ch{base, kv_start, chunk_len, toks.data()};
  std::vector<qos_decode> dec(static_cast<size_t>(n_decode));
  int r;
  if (chunk_len > 0) {
    if ((r = qos_kv_alloc(e, base, kv_start + chunk_len)) != QOS_OK) return r;
    ids.push_back(base);
    if ((r = qos_kv_fill_synthetic(e, base, kv_start, 2)) != QOS_OK) { cleanup(); return r; }
  }
  for (int j = 0; j < n_decode; ++j) {
    const int64_t id = base + 1 + j;
    if ((r = qos_kv_alloc(e, id, ctx_lens[j] + 1)) != QOS_OK) { cleanup(); return r; }
    ids.push_back(id);
    if ((r = qos_kv_fill_synthetic(e, id, ctx_lens[j], 2)) != QOS_OK) { cleanup(); return r; }
    dec[size_t(j)] = qos_decode{id, ctx_lens[j], int32_t((j * 31 + 7) % e->cfg.vocab)};
  }
  qos_batch b{chunk_len > 0 ? 1 : 0, &ch, n_decode, dec.data()};
  cudaStream_t st = internal_stream(e);
  cudaEvent_t a, z;
  cudaEventCreate(&a);
  cudaEventCreate(&z);
  std::vector<float> ms;
  for (int i = 0; i < warmup + reps; ++i) {
    cudaEventRecord(a, st);
    if ((r = do_step(e, &b, nullptr, QOS_F32, nullptr, 0, st, false)) != QOS_OK) break;
    cudaEventRecord(z, st);
    cudaEventSynchronize(z);
    float t = 0;
    cudaEventElapsedTime(&t, a, z);
    if (i >= warmup) ms.push_back(t);
  }
  cudaEventDestroy(a);
  cudaEventDestroy(z);
  cleanup();
  if (r != QOS_OK) return r;
  std::sort(ms.begin(), ms.end());
  *ms_median = ms[ms.size() / 2];
  if (ms_p95) *ms_p95 = ms[std::min(ms.size() - 1, size_t(std::ceil(0.95 * ms.size())) - 1)];
  return QOS_OK;
}

int qos_profile_step(qos_engine_t* e, int32_t chunk_len, int32_t n_decode, const int32_t* ctx_lens, int32_t reps,
                     float* ms_out) {
  return qos_profile_step_ex(e, chunk_len, 0, n_decode, ctx_lens, -1, reps, ms_out, nullptr);
}

int qos_engine_set_option(qos_engine_t* e, const char* name, int64_t value) {
  if (!e || !name) return set_error(QOS_ERR_INVALID_ARG, "args");
  const std::string n(name);
  if (n == "overlap_attn") e->overlap_attn = value != 0;
  else if (n == "decode_round_split") e->decode_round_split = value != 0;
  else if (n == "decode_split") {
    if (value < 64 || value > 65536 || (value & (value - 1))) return set_error(QOS_ERR_INVALID_ARG, "decode_split must be a power of two in [64, 65536]");
    e->decode_split = int(value);
  }
  else if (n == "gemm_2cta") e->gemm_2cta = value != 0;
  else if (n == "fa_persist") e->fa_persist = value != 0;
  else if (n == "fa_pair") e->fa_pair = value != 0;
  else if (n == "decode_persist") e->decode_persist = value != 0;
  else if (n == "decode_items_per_sm") e->decode_items_per_sm = int(value < 0 ? 0 : value > 64 ? 64 : value);
  else if (n == "fa_item_cost") e->fa_item_cost = int(value < 0 ? 0 : value > 64 ? 64 : value);
  else if (n == "norm_fold") e->norm_fold = value != 0;
  else if (n == "tp_scatter") e->tp_scatter = value != 0;
  else if (n == "attn_order") {
    if (value < 0 || value > 2) return set_error(QOS_ERR_INVALID_ARG, "attn_order must be 0, 1 or 2");
    e->attn_order = int(value);
  }
  else if (n == "tp_twoshot") e->tp_twoshot = value < 0 ? -1 : value > 0 ? 1 : 0;
  else if (n == "decode_stages") {
    if (value != 4 && value != 8) return set_error(QOS_ERR_INVALID_ARG, "decode_stages must be 4 or 8");
    e->decode_stages = int(value);
  }
  else if (n == "fa_qtiles") {
    if (value != 1 && value != 2) return set_error(QOS_ERR_INVALID_ARG, "fa_qtiles must be 1 or 2");
    e->fa_qtiles = int(value);
  }
  else if (n == "gemm_splitk") e->gemm_splitk = value != 0;
  else if (n == "pdl") set_pdl(value != 0);  // process-wide
  else if (n == "fa_poly") set_fa_poly(int(value));  // process-wide
  else if (n == "fa_kvfirst") set_fa_kvfirst(int(value != 0));  // process-wide
  else if (n == "fa_tma5") set_fa_tma5(int(value != 0));  // process-wide
  else if (n == "fa_psplit") set_fa_psplit(int(value != 0));  // process-wide
  else if (n == "gemm2_rel_cluster") set_gemm2_rel_cluster(int(value != 0));  // process-wide (experiment)
  else if (n == "swab_gran") set_swab_gran(int(value));  // process-wide (experiments)
  else if (n == "gemm_swab") e->gemm_swab = int(value < 0 ? 0 : value > 2 ? 2 : value);
  else if (n == "gemm_streamk") e->gemm_streamk = int(value < 0 ? 0 : value > 2 ? 2 : value);
  else if (n == "dual_stream") e->dual_stream = value != 0;
  else if (n == "dual_min_prefill") e->dual_min_prefill = int(value);
  else if (n == "dual_min_decode") e->dual_min_decode = int(value);
  else if (n == "dual_sms_prefill") e->dual_sms_pre = int(value);
  else if (n == "dual_sms_decode") e->dual_sms_dec = int(value);
  else if (n == "add_split") e->add_split = value != 0;
  else if (n == "gemm_bn") e->gemm_bn = (value == 128 || value == 256) ? int(value) : 0;
  else if (n == "shares_device") e->shares_device = value != 0 || (e->group && e->shares_device);
  else if (n == "gemm_sms") e->gemm_sms = int(value < 0 ? 0 : value > e->num_sms ? e->num_sms : value);
  else return set_error(QOS_ERR_INVALID_ARG, "unknown option");
  return QOS_OK;
}

int qos_engine_set_timing(qos_engine_t* e, int enable) {
  if (!e) return set_error(QOS_ERR_INVALID_ARG, "engine is NULL");
  if (cudaDeviceSynchronize() != cudaSuccess) return set_error(QOS_ERR_CUDA, "set_timing sync");
  e->timing = enable != 0;
  e->tev.clear();
  e->ev_used = 0;
  return QOS_OK;
}

int qos_last_step_timing(qos_engine_t* e, float ms[QOS_T_COUNT], int32_t launches[QOS_T_COUNT]) {
  if (!e || !ms) return set_error(QOS_ERR_INVALID_ARG, "args");
  for (int i = 0; i < QOS_T_COUNT; ++i) {
    ms[i] = 0.f;
    if (launches) launches[i] = 0;
  }
  if (!e->tev.empty()) QOS_CU(cudaEventSynchronize(e->tev.back().second.second));
  for (auto& x : e->tev) {
    float t = 0;
    cudaEventElapsedTime(&t, x.second.first, x.second.second);
    ms[x.first] += t;
    if (launches) launches[x.first] += 1;
  }
  e->tev.clear();
  e->ev_used = 0;
  return QOS_OK;
}

int qos_last_step_io(qos_engine_t* e, int64_t* h2d_bytes, int64_t* d2h_bytes) {
  if (!e || !h2d_bytes || !d2h_bytes) return set_error(QOS_ERR_INVALID_ARG, "args");
  *h2d_bytes = e->last_h2d;
  *d2h_bytes = e->last_d2h;
  return QOS_OK;
}

int qos_engine_launch_count(qos_engine_t* e, int64_t* out) {
  if (!out) return set_error(QOS_ERR_INVALID_ARG, "out");
  (void)e;
  *out = g_launches.load();
  return QOS_OK;
}

// ------------------------------------------------------------------ kernel-level ops
static int op_gemm(const void* A, const void* B, void* C, int64_t M, int64_t N, int64_t K, int epi, const float* bias,
                   int ksplit, void* stream) {
  if (!A || !B || !C || (epi == QOS_EPI_BIAS_BF16 && !bias)) return set_error(QOS_ERR_INVALID_ARG, "gemm pointers");
  QOS_TRY(gemm_check_shape(M, N, K, epi));
  int dev = 0, sms = 148;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
  int bn = gemm_pick_bn(M, N, epi, sms);
  static float* part = nullptr;  // process-wide split-K workspace of the op entry point
  static int* cnt = nullptr;
  if (!part) {
    if (cudaMalloc(&part, size_t(kGemmMaxUnits) * 128 * 256 * 4) != cudaSuccess ||
        cudaMalloc(&cnt, size_t(kGemmMaxTiles) * 4) != cudaSuccess || cudaMemset(cnt, 0, size_t(kGemmMaxTiles) * 4))
      return set_error(QOS_ERR_OOM, "gemm split-K workspace");
  }
  static const bool swab_env = !(getenv("QOS_GEMM_SWAB") && atoi(getenv("QOS_GEMM_SWAB")) == 0);
  const int64_t ldc = epi == QOS_EPI_SILU_GATE ? N / 2 : N;
  if (ksplit == -1 || (ksplit == 0 && swab_env && swab_prefer_k(M, N, K, sms))) {
    // weight-streaming swap-AB kernel (gemm_swab.cu)
    const int bnt = swab_pick_bnt(M);
    CUtensorMap tw, tt;
    QOS_TRY(make_tmap_2d_bf16(&tw, B, uint64_t(N), uint64_t(K), uint64_t(K), 128, 64, true));
    QOS_TRY(make_tmap_2d_bf16(&tt, A, uint64_t(M), uint64_t(K), uint64_t(K), uint32_t(bnt), 64, true));
    count_launch();
    return gemm_swab_run(tw, tt, bnt, M, N, K, epi, C, ldc, bias, sms, reinterpret_cast<cudaStream_t>(stream), part,
                         cnt, int64_t(kGemmMaxUnits) * 128 * 256, kGemmMaxTiles, 0, nullptr);
  }
  static const bool g2_env = !(getenv("QOS_GEMM_2CTA") && atoi(getenv("QOS_GEMM_2CTA")) == 0);
  if (ksplit == -3 || (ksplit == 0 && g2_env && gemm2_eligible(M, N, K, sms))) {
    // CTA-pair kernel (256 x 256 tiles)
    if (N % 256) return set_error(QOS_ERR_UNSUPPORTED, "gemm: the CTA-pair kernel needs N % 256 == 0");
    CUtensorMap ta, tb;
    QOS_TRY(make_tmap_2d_bf16(&ta, A, uint64_t(M), uint64_t(K), uint64_t(K), 128, 64, true));
    QOS_TRY(make_tmap_2d_bf16(&tb, B, uint64_t(N), uint64_t(K), uint64_t(K), 128, 64, true));
    count_launch();
    return gemm2_run(ta, tb, M, N, K, epi, C, ldc, bias, sms, reinterpret_cast<cudaStream_t>(stream), 0, 0, nullptr);
  }
  const int sk_mode = ksplit <= -2 ? 2 : 0;
  // automatic = the engine's default: no split-K (QOS_GEMM_SPLITK=1 restores the split heuristic)
  static const bool sk_env = getenv("QOS_GEMM_SPLITK") && atoi(getenv("QOS_GEMM_SPLITK")) != 0;
  int ks = ksplit <= -2 ? 1 : ksplit <= 0 ? (sk_env ? gemm_pick_ksplit(M, N, K, bn, sms, kGemmMaxUnits) : 1) : ksplit;
  static const bool as_env = !(getenv("QOS_ADD_SPLIT") && atoi(getenv("QOS_ADD_SPLIT")) == 0);
  if (ksplit == 0 && !sk_env && as_env && epi == QOS_EPI_ADD_F32) gemm_pick_add_split(M, N, K, sms, kGemmMaxTiles, &bn, &ks);
  if (const char* fb = getenv("QOS_GEMM_BN")) {  // measurement only: force the tile width
    const int v = atoi(fb);
    if (v == 128 || (v == 256 && N % 256 == 0)) bn = v;
  }
  const int64_t tiles = ((M + 127) / 128) * ((N + bn - 1) / bn);
  const bool ordered = epi == QOS_EPI_ADD_F32;  // in-place ordered slices: no partial slots
  if (ks > 1 && (tiles > kGemmMaxTiles || (!ordered && tiles * ks > kGemmMaxUnits) || (K / 64) < ks))
    return set_error(QOS_ERR_INVALID_ARG, "gemm: ksplit too large for the shape / workspace");
  CUtensorMap ta, tb;
  QOS_TRY(make_tmap_2d_bf16(&ta, A, uint64_t(M), uint64_t(K), uint64_t(K), 128, 64, true));
  QOS_TRY(make_tmap_2d_bf16(&tb, B, uint64_t(N), uint64_t(K), uint64_t(K), uint32_t(bn), 64, true));
  count_launch();
  return gemm_run(ta, tb, bn, M, N, K, epi, C, ldc, bias, sms, reinterpret_cast<cudaStream_t>(stream), ks, part, cnt,
                  0, 0, nullptr, sk_mode, true);
}

int qos_op_gemm(const void* A, const void* B, void* C, int64_t M, int64_t N, int64_t K, int epi, const float* bias,
                void* stream) {
  return op_gemm(A, B, C, M, N, K, epi, bias, 0, stream);
}

int qos_op_gemm_ex(const void* A, const void* B, void* C, int64_t M, int64_t N, int64_t K, int epi, const float* bias,
                   int ksplit, void* stream) {
  return op_gemm(A, B, C, M, N, K, epi, bias, ksplit, stream);
}

int qos_op_rmsnorm(const float* x, const void* g, void* out, int32_t T, int32_t d, float eps, void* stream) {
  if (!x || !g || !out || T < 0 || d < 8 || d % 8) return set_error(QOS_ERR_INVALID_ARG, "rmsnorm args");
  QOS_CU(launch_rmsnorm(x, g, out, T, d, eps, reinterpret_cast<cudaStream_t>(stream)));
  return QOS_OK;
}

static int ensure_dbg(qos_engine* e, size_t bytes) {
  if (e->dbg_bytes >= bytes) return QOS_OK;
  if (e->dbg) cudaFree(e->dbg);
  e->dbg = nullptr;
  e->dbg_bytes = 0;
  QOS_CU(cudaMalloc(&e->dbg, bytes));
  e->dbg_bytes = bytes;
  return QOS_OK;
}

static int kv_rw(qos_engine* e, int32_t layer, int64_t req, int32_t pos0, int32_t n, const uint16_t* kin,
                 const uint16_t* vin, uint16_t* kout, uint16_t* vout) {
  if (!e || layer < 0 || layer >= e->cfg.n_layers || pos0 < 0 || n < 0) return set_error(QOS_ERR_INVALID_ARG, "kv args");
  auto it = e->reqs.find(req);
  if (it == e->reqs.end()) return set_error(QOS_ERR_UNKNOWN_REQ, "unknown request");
  if (int64_t(pos0) + n > int64_t(it->second.blocks.size()) * 16) return set_error(QOS_ERR_NOT_ALLOCATED, "range");
  QOS_CU(cudaSetDevice(e->device));
  cudaStream_t st = internal_stream(e);
  QOS_TRY(flush_table_updates(e, st));
  const size_t bytes = size_t(n) * e->sh.Hkv * e->cfg.head_dim * 2;
  QOS_TRY(ensure_dbg(e, bytes));
  const int32_t* trow = e->d_tables + size_t(it->second.row) * e->table_w;
  for (int kv = 0; kv < 2; ++kv) {
    void* plane = reinterpret_cast<__nv_bfloat16*>(e->kv) + (size_t(layer) * 2 + kv) * e->plane_elems;
    if (kin) {
      QOS_CU(cudaMemcpyAsync(e->dbg, kv ? vin : kin, bytes, cudaMemcpyHostToDevice, st));
      QOS_CU(launch_kv_scatter(plane, trow, pos0, n, e->sh.Hkv, e->cfg.head_dim, e->dbg, st));
    } else {
      QOS_CU(launch_kv_gather(plane, trow, pos0, n, e->sh.Hkv, e->cfg.head_dim, e->dbg, st));
      QOS_CU(cudaMemcpyAsync(kv ? vout : kout, e->dbg, bytes, cudaMemcpyDeviceToHost, st));
    }
    QOS_CU(cudaStreamSynchronize(st));
  }
  return QOS_OK;
}

int qos_kv_write(qos_engine_t* e, int32_t layer, int64_t req, int32_t pos0, int32_t n, const uint16_t* k,
                 const uint16_t* v) {
  if (!k || !v) return set_error(QOS_ERR_INVALID_ARG, "kv_write pointers");
  return kv_rw(e, layer, req, pos0, n, k, v, nullptr, nullptr);
}
int qos_kv_read(qos_engine_t* e, int32_t layer, int64_t req, int32_t pos0, int32_t n, uint16_t* k, uint16_t* v) {
  if (!k || !v) return set_error(QOS_ERR_INVALID_ARG, "kv_read pointers");
  return kv_rw(e, layer, req, pos0, n, nullptr, nullptr, k, v);
}

int qos_op_qkv_rope_append(qos_engine_t* e, int32_t layer, const qos_batch* b, const uint16_t* h_in, uint16_t* q_out) {
  if (!e || !h_in || !q_out || layer < 0 || layer >= e->cfg.n_layers) return set_error(QOS_ERR_INVALID_ARG, "args");
  QOS_CU(cudaSetDevice(e->device));
  cudaStream_t st = internal_stream(e);
  QOS_TRY(acquire_staging(e));
  StepMeta m;
  int r = build_step(e, b, false, e->h_meta[e->meta_cur], m);
  if (r != QOS_OK) { e->meta_cur ^= 1; return r; }
  uint8_t* dm;
  QOS_TRY(upload_meta(e, m, st, &dm));
  const int d = e->cfg.d_model, hd = e->cfg.head_dim;
  QOS_CU(cudaMemcpyAsync(e->ws + e->wsl.h, h_in, size_t(m.T) * d * 2, cudaMemcpyHostToDevice, st));
  __nv_bfloat16* kpl = reinterpret_cast<__nv_bfloat16*>(e->kv) + (size_t(layer) * 2 + 0) * e->plane_elems;
  __nv_bfloat16* vpl = reinterpret_cast<__nv_bfloat16*>(e->kv) + (size_t(layer) * 2 + 1) * e->plane_elems;
  const QkvRopeArgs ra{reinterpret_cast<int32_t*>(dm + m.o_pos), reinterpret_cast<int32_t*>(dm + m.o_slot), e->rope_tab,
                       kpl, vpl, e->sh.H, e->sh.Hkv, hd};
  const Seg g{0, m.T, st, false, false, reinterpret_cast<float*>(e->ws + e->wsl.gemm_part),
              reinterpret_cast<int*>(e->ws + e->wsl.gemm_cnt), 0};
  const auto& L = e->wl.layers[layer];
  __nv_bfloat16* qkv = reinterpret_cast<__nv_bfloat16*>(e->ws + e->wsl.qkv);
  QOS_TRY(gemm_seg(e, g, e->a_h, e->lmaps[layer].qkv, e->nqkv, d, EPI_QKV_ROPE, qkv, e->nqkv,
                   e->cfg.qkv_bias ? reinterpret_cast<const float*>(e->w + L.bqkv) : nullptr, &ra));
  const size_t qb = size_t(e->sh.H) * hd * 2;
  QOS_CU(cudaMemcpy2DAsync(q_out, qb, qkv, size_t(e->nqkv) * 2, qb, size_t(m.T), cudaMemcpyDeviceToHost, st));
  QOS_TRY(release_staging(e, st));
  QOS_CU(cudaStreamSynchronize(st));
  return QOS_OK;
}

int qos_op_attention(qos_engine_t* e, int32_t layer, const qos_batch* b, const uint16_t* q_in, float* out) {
  if (!e || !q_in || !out || layer < 0 || layer >= e->cfg.n_layers) return set_error(QOS_ERR_INVALID_ARG, "args");
  QOS_CU(cudaSetDevice(e->device));
  cudaStream_t st = internal_stream(e);
  QOS_TRY(acquire_staging(e));
  StepMeta m;
  int r = build_step(e, b, false, e->h_meta[e->meta_cur], m);
  if (r != QOS_OK) { e->meta_cur ^= 1; return r; }
  uint8_t* dm;
  QOS_TRY(upload_meta(e, m, st, &dm));
  const int hd = e->cfg.head_dim;
  const size_t qrow = size_t(e->sh.H) * hd;
  QOS_TRY(ensure_dbg(e, size_t(m.T) * qrow * (2 + 4)));
  __nv_bfloat16* q = reinterpret_cast<__nv_bfloat16*>(e->dbg);
  float* o = reinterpret_cast<float*>(reinterpret_cast<uint8_t*>(e->dbg) + align_up(size_t(m.T) * qrow * 2, 256));
  QOS_CU(cudaMemcpyAsync(q, q_in, size_t(m.T) * qrow * 2, cudaMemcpyHostToDevice, st));
  AttnLaunch al;
  al.q = q;
  al.q_ld = int(qrow);
  al.out = o;
  al.out_ld = int(qrow);
  al.out_f32 = 1;
  al.kv_tmap = &e->kv_map;
  al.kv_tmap5 = &e->kv_map5;
  al.layer = layer;
  al.H = e->sh.H;
  al.Hkv = e->sh.Hkv;
  al.hd = hd;
  al.num_blocks = int(e->cfg.num_blocks);
  al.tables = e->d_tables;
  al.table_w = e->table_w;
  al.scale_log2 = float(1.4426950408889634 / std::sqrt(double(hd)));
  al.q_tiles = m.fa_qtiles;
  al.cta_off = m.n_pcta ? reinterpret_cast<const int32_t*>(dm + m.o_pcta) : nullptr;
  al.n_cta = m.n_pcta;
  al.pair = m.fa_pair;
  al.q_tmap = nullptr;  // per-launch map over the op's q buffer
  al.q_rows = m.T;
  al.decode_stages = e->decode_stages;
  al.decode_persist = e->decode_persist ? 1 : 0;
  QOS_CU(launch_prefill_attention_tc(al, reinterpret_cast<const PrefillItem*>(dm + m.o_pitems), m.n_pitems, st));
  QOS_CU(launch_decode_attention(al, reinterpret_cast<const DecodeItem*>(dm + m.o_ditems), m.n_ditems,
                                 reinterpret_cast<float*>(e->ws + e->wsl.partials),
                                 reinterpret_cast<int*>(e->ws + e->wsl.counters), st));
  QOS_CU(cudaMemcpyAsync(out, o, size_t(m.T) * qrow * 4, cudaMemcpyDeviceToHost, st));
  QOS_TRY(release_staging(e, st));
  QOS_CU(cudaStreamSynchronize(st));
  return QOS_OK;
}

}  // extern "C"
