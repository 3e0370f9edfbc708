// engine.cu — host side of libckpt.so: the C ABI of include/ckpt.h.
//
// Owns, per handle (one process / GPU): the persistent leaf digests
// Tree(leaf) (Alg.1 l.21, R5), the device record table, the per-stage tree
// scratch, and an arena of consolidated diffs. ckpt_checkpoint enqueues the kernel
// sequence of kernels.h on the caller's stream and synchronises exactly once, to read
// the 128-byte totals record back (the process stops during checkpointing).
// All capacity (record table, diff arena) is reserved before the first kernel, so a
// failure never leaves a half-committed checkpoint (ckpt.h error contract).
#include <cudaTypedefs.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <deque>
#include <new>
#include <vector>

#include "../../include/ckpt.h"
#include "arena.h"
#include "kernels.h"

using namespace ckpt;

namespace {

struct DiffRec {
  ckpt_diff info;
  uint8_t* ptr;
  // restore plan (k_restore.cu), built lazily by the first restore that needs it
  unsigned long long* Flo = nullptr;
  unsigned long long* Foff = nullptr;
  unsigned long long* Slo = nullptr;
  unsigned long long* Soff = nullptr;
  unsigned long long* Ssrc = nullptr;
  unsigned long long* Fseg = nullptr;
  unsigned long long* Sseg = nullptr;
  uint32_t* Cch = nullptr;              // claim list (chunk-major restore)
  unsigned long long* Csrc = nullptr;
  unsigned long long shift_bytes = 0;
  bool planned = false;
  bool collided = false;                // CKPT_ECOLLIDE: committed with a skipped insert (R14)
};

// A checkpoint whose kernels are enqueued and whose statistics the host has not collected
// (ckpt_checkpoint_submit; ckpt_checkpoint collects its own before returning).
struct Inflight {
  uint32_t k = 0;
  uint8_t* out = nullptr;            // the diff's place in arena[arena]
  int arena = 0;
  cudaStream_t wait_st = nullptr;    // queried while waiting (a failed kernel never publishes)
  std::chrono::steady_clock::time_point t_entry, t_pre, t_launched;
};

#ifndef CKPT_PIPE_DEPTH
#define CKPT_PIPE_DEPTH CKPT_PIPELINE_DEPTH   // pipelined calls in flight (include/ckpt.h). A depth-3
                                              // build (3 arenas, 4 counter sets) measured the same as 2
                                              // with SM partitions: the chain's throughput on its SMs, not
                                              // its latency, bounds the step
#endif
constexpr int kDepth = CKPT_PIPE_DEPTH;
static_assert(kDepth >= 2 && kDepth <= 3, "pipeline depth");
#ifndef CKPT_GREEN_CAND_PER_SM
#define CKPT_GREEN_CAND_PER_SM 2600   // candidates per chain SM up to which a pipelined call is partitioned
#endif
#ifndef CKPT_K1_C32_SMEM
#define CKPT_K1_C32_SMEM 49152      // K1 stage budget per CTA when C = 32 (data + digests; 4 CTAs per SM)
#endif
#ifndef CKPT_K1_SMALLC_SMEM
#define CKPT_K1_SMALLC_SMEM 65536   // K1 stage budget per CTA when 32 < C < 128 (3 CTAs per SM)
#endif
#ifndef CKPT_K1_GRAB_BYTES
#define CKPT_K1_GRAB_BYTES 32768
#endif
#ifndef CKPT_TABLE_GROW_LOAD
#define CKPT_TABLE_GROW_LOAD 0.6
#endif
constexpr double kGrowLoad = CKPT_TABLE_GROW_LOAD;   // load factor right after a growth
constexpr double kMaxLoad = kGrowLoad + 0.2;         // reserve so that even a worst-case checkpoint stays below this
constexpr uint64_t kArenaVA[] = {4ull << 40, 1ull << 40, 256ull << 30, 64ull << 30};

}  // namespace

struct ckpt_ctx {
  int device = 0;
  int num_sms = 148;
  bool poisoned = false;
  uint32_t C = 0;
  int mode = kModeTree;          // CKPT_MODE_*
  uint32_t variant = 0;          // CKPT_VARIANT_* (Tree mode; R22, R23)
  uint32_t switch_permille = 1000;
  // geometry (fixed after checkpoint 0, R17)
  bool geo_set = false;
  uint64_t B = 0, n = 0, m = 0;
  int h = 0, t0 = 0;
  int S = 0;
  int Lin[kMaxStages] = {}, gsz[kMaxStages] = {};
  uint64_t ngroups[kMaxStages] = {};
  // device state
  Digest* prev = nullptr;
  uint32_t* cand = nullptr;       // = cand2[k % kDepth] of the current call
  uint32_t* cand2[kDepth] = {};   // candidate bits per call slot (k % kDepth): a pipelined call's K1 writes its own
                                  // while the previous call's tree phases read theirs
  Digest* cdig2[kDepth] = {};          // pipelined calls: the candidates' digests of call k (slot k % kDepth), read
                                  // by its K1b / tree kernels while the next call's K1 updates prev in place
  uint64_t nwords = 0;
  unsigned long long* res_of = nullptr;   // per chunk (candidates only): K1b's resolution
  LevelIO lvl[kMaxStages] = {};
  Digest* tdig[kMaxStages] = {};
  unsigned long long* tsrc[kMaxStages] = {};
  uint32_t* arr2[kMaxStages] = {};
  uint32_t* arr3[kMaxStages] = {};
  uint32_t* arr4[kMaxStages] = {};
  uint32_t* dcnt[kMaxStages] = {};
  uint32_t* gm2[kMaxStages] = {};
  uint32_t* gm3[kMaxStages] = {};
  uint32_t* gm4[kMaxStages] = {};
  uint32_t* wl0 = nullptr;
  uint32_t* dbits = nullptr;     // dirty bit per stage-0 tree tile (inside ctr: zeroed per call)
  uint32_t* tcc = nullptr;       // candidate leaves per stage-0 tree tile (inside ctr)
  // Totals + per-stage counters, triple-buffered: call k uses ctr3[k % 3] and its last kernel
  // zeroes ctr3[(k + 2) % 3] (the previous call's, complete by then) for call k + 2, so no
  // memset precedes K1 and a pipelined call's K1 never meets a buffer still being zeroed.
  uint8_t* ctr3[kDepth + 1] = {};
  size_t ctr_bytes = 0;
  size_t ctr_dbits_off = 0, ctr_tcc_off = 0, ctr_bsum_off = 0, ctr_gsum_off = 0, ctr_stage_off[kMaxStages] = {};
  uint4* scratch = nullptr;
  uint4* tilecnt = nullptr;
  uint32_t* lmask = nullptr;
  uint32_t* defer = nullptr;     // 256-chunk leaf tiles whose inserts go to K1b (= defer2[k % kDepth])
  uint32_t* defer2[kDepth] = {};
  unsigned long long* blocksum = nullptr;
  unsigned long long* gsum = nullptr;
  Totals* tot = nullptr;         // = (Totals*)ctr
  Totals* tot_host2[kDepth] = {};    // pinned + mapped, per call slot: written by the gather kernel
  Slot* tab = nullptr;
  uint64_t cap = 0, live = 0;
  std::vector<void*> retired;    // record tables replaced by a growth (freed by ckpt_destroy)
  DiffArena arena[kDepth];       // diffs; pipelined calls rotate (call k: arena[k % kDepth])
  int arenas_ready = 1;          // arena[0] is set up with the geometry, the others at first use
  std::vector<DiffRec> diffs;
  // pipelining (ckpt_checkpoint_submit): K1 on the caller's stream, K1b .. gather on `cs`
  std::deque<Inflight> inflight;
  bool call_pipe[4] = {};        // call k was submitted pipelined (index k & 3)
  cudaStream_t cs = nullptr;
  cudaEvent_t ev_k1[kDepth] = {}, ev_chain[kDepth] = {};   // after K1(k) / after gather(k), slot k % kDepth
  // SM partitions of pipelined calls (green contexts): K1 on the SMs of one
  // green context (stream k1s), the chain on the other m (stream cs), so that the next K1 and
  // this call's chain run side by side instead of taking turns for the SMs. m is chosen per
  // call from the candidate count of the last collected call; none when the chain is heavy.
  struct Part {
    int m = 0;
    CUgreenCtx g[2] = {};
    cudaStream_t k1s = nullptr, cs = nullptr;
    int sm_k1 = 0, sm_chain = 0;
  };
  static constexpr int kMaxParts = 4;
  static constexpr int kPartSMs[kMaxParts] = {16, 24, 32, 40};   // chain SMs of each partition
  Part parts[kMaxParts];            // created at the first pipelined call of a buffer <= 2 GiB (ensure_pipe_state)
  bool green_ok = false;            // partitions allowed (no CKPT_GREEN=0, no profiling tool, a full GPU)
  int forced_m = 0;                 // CKPT_GREEN=m (m >= 8): every pipelined call on one m-SM partition (tuning)
  int prio_hi = 0;                  // the chain streams' priority
  cudaEvent_t ev_in[kDepth] = {};
  cudaStream_t prev_cs = nullptr;   // chain stream of the previous pipelined call
  uint64_t last_cand = ~0ull;       // non-FIXED leaves of the last collected call (~0: none yet)
  uint8_t* staging = nullptr;
  uint64_t staging_size = 0;
  // restore state (lazy): chunk owners, plan scratch, the chain's plans on device
  unsigned long long* owner = nullptr;   // restore: source address of every chunk (chunk-major form)
  unsigned long long* rs_len = nullptr;
  uint64_t rs_len_cap = 0;
  void* rs_scan = nullptr;
  size_t rs_scan_bytes = 0;
  int* rs_err = nullptr;
  RestoreDiff* rs_chain = nullptr;
  uint64_t rs_chain_cap = 0;
  cudaStream_t internal = nullptr;
  // completion of the latest ckpt_checkpoint's work (its gather kernel finishes writing the
  // diff after the call has returned on the statistics): every later consumer of the lineage
  // on another stream (the next checkpoint, D2H copies, restores, introspection) waits for
  // the stream the call ran on. The event is recorded lazily, when such a consumer comes:
  // an event between the gather and the next call's K1 on the same stream would stop K1's
  // programmatic early launch
  cudaEvent_t done_ev = nullptr;
  cudaStream_t last_stream = nullptr;
  bool pending = false;
  uint64_t launches = 0;         // kernels this handle has enqueued (all calls)
  uint64_t host_syncs = 0;       // host waits on the device this handle has performed (all calls)
  int prof = 0;                  // 0 off, 1 K1 + whole call, 2 every phase
  // per-checkpoint event sets (ring), queried lazily so the call itself never waits on them
  static constexpr int kEvRing = 256;
  cudaEvent_t evr[kEvRing][6] = {};
  int64_t ev_id[kEvRing] = {};
  int ev_level[kEvRing] = {};
  cudaEvent_t* ev = nullptr;     // event set of the current call
  float times[12] = {};          // host times of the latest call ([6..11])
  PFN_cuTensorMapEncodeTiled_v12000 encode = nullptr;
  std::vector<void*> allocs;   // per-geometry allocations
  // diagnostics: CKPT_TRACE=<file prefix> records per-group tree timings of each call
  const char* trace_path = nullptr;
  int dbg = 0;
  ulonglong4* trace = nullptr;
  uint32_t* trace_n = nullptr;
};

#define CK(x)                                                                               \
  do {                                                                                      \
    cudaError_t e_ = (x);                                                                   \
    if (e_ != cudaSuccess) {                                                                \
      fprintf(stderr, "libckpt: CUDA error %s at %s:%d\n", cudaGetErrorString(e_), __FILE__, __LINE__); \
      h->poisoned = true;                                                                   \
      return CKPT_ECUDA;                                                                    \
    }                                                                                       \
  } while (0)

// Any host thread may call the library: each entry point that touches the device makes the
// handle's device (its primary context) current first. A thread that has made no CUDA
// runtime call has no current context, and the driver-API tensor-map encode then fails.
#define BIND(h)                                                                  \
  do {                                                                           \
    if (cudaSetDevice((h)->device) != cudaSuccess) {                             \
      cudaGetLastError();                                                        \
      return CKPT_ECUDA;                                                         \
    }                                                                            \
  } while (0)

namespace {

// Every place the library blocks the host on the device goes through here (counted: the
// one-synchronisation contract of ckpt_checkpoint is tested with ckpt_host_syncs).
cudaError_t sync_stream(ckpt_ctx* h, cudaStream_t st) {
  ++h->host_syncs;
  return cudaStreamSynchronize(st);
}

// Order `st` after the latest checkpoint's kernels (no host wait). On the stream that call
// ran on, stream order does it; elsewhere an event recorded now on that stream (it follows
// the call's kernels, and possibly later work of the caller there: correct, at worst early).
cudaError_t after_last_checkpoint(ckpt_ctx* h, cudaStream_t st) {
  if (!h->pending || st == h->last_stream) return cudaSuccess;
  cudaError_t e = cudaEventRecord(h->done_ev, h->last_stream);
  if (e == cudaSuccess) e = cudaStreamWaitEvent(st, h->done_ev, 0);
  return e;
}

template <class T>
cudaError_t dalloc(ckpt_ctx* h, T** p, size_t count) {
  void* q = nullptr;
  cudaError_t e = cudaMalloc(&q, count * sizeof(T) > 0 ? count * sizeof(T) : 16);
  if (e != cudaSuccess) return e;
  h->allocs.push_back(q);
  *p = static_cast<T*>(q);
  return cudaSuccess;
}

int ceil_log2(uint64_t n) {
  int h = 0;
  while ((1ull << h) < n) ++h;
  return h;
}

// Per-geometry state, allocated by the first checkpoint (or import) of a handle. The
// counter blocks are zeroed on `st`, the stream the call's kernels then run on.
int setup_geometry(ckpt_ctx* h, uint64_t B, cudaStream_t st) {
  h->B = B;
  h->n = (B + h->C - 1) / h->C;
  h->h = ceil_log2(h->n);
  h->m = 2 * h->n - (1ull << h->h);
  h->t0 = std::min(kTileLog, h->h);
  // stage plan: stage 0 covers heights 0..t0 (tiles); then groups of kGroupLog levels
  h->S = 0;
  int L = 0;
  h->Lin[0] = 0;
  h->gsz[0] = h->t0;
  h->S = 1;
  L = h->t0;
  while (L < h->h) {
    if (h->S >= kMaxStages) return CKPT_EINVAL;
    const int g = std::min(kGroupLog, h->h - L);
    h->Lin[h->S] = L;
    h->gsz[h->S] = g;
    ++h->S;
    L += g;
  }
  for (int s = 0; s < h->S; ++s) h->ngroups[s] = 1ull << (h->h - h->Lin[s] - h->gsz[s]);

  const uint64_t n = h->n;
  const uint64_t n_tiles = h->ngroups[0];
  h->nwords = (n + 31) / 32;
  cudaError_t e = cudaSuccess;
#define AL(ptr, cnt)                      \
  do {                                    \
    e = dalloc(h, &(ptr), (cnt));         \
    if (e != cudaSuccess) return CKPT_ENOMEM; \
  } while (0)
  AL(h->prev, n);
  for (int i = 0; i < kDepth; ++i) AL(h->cand2[i], h->nwords + 32);
  h->cand = h->cand2[0];
  AL(h->res_of, n);
  for (int s = 0; s < h->S; ++s) {
    if (s >= 1) {
      const uint64_t P = 1ull << (h->h - h->Lin[s]);
      AL(h->lvl[s].dig, P);
      AL(h->lvl[s].src, P);
    }
    const uint64_t slots = h->ngroups[s] << h->gsz[s];
    AL(h->tdig[s], slots);
    AL(h->tsrc[s], 2 * slots);
  }
  // per-call counters: Totals, then cnt/done2/done3 of every stage s >= 1
  {
    size_t bytes = (sizeof(Totals) + 255) & ~size_t(255);
    const size_t dbits_off = bytes;
    bytes += ((n_tiles + 31) / 32) * sizeof(uint32_t);
    bytes = (bytes + 255) & ~size_t(255);
    const size_t tcc_off = bytes;
    bytes += n_tiles * sizeof(uint32_t);
    bytes = (bytes + 255) & ~size_t(255);
    const size_t bsum_off = bytes;
    bytes += (3 * ((n_tiles + kTilesPerBlock - 1) / kTilesPerBlock) + 3) * sizeof(unsigned long long);
    bytes = (bytes + 255) & ~size_t(255);
    const size_t gsum_off = bytes;
    bytes += 3 * ((n_tiles + 31) / 32) * sizeof(unsigned long long);
    bytes = (bytes + 255) & ~size_t(255);
    size_t off[kMaxStages] = {};
    for (int s = 1; s < h->S; ++s) {
      off[s] = bytes;
      bytes += (4 + 32 + 64 + 32) * h->ngroups[s] * sizeof(uint32_t);   // arr2 arr3 arr4 dcnt, gm2, gm3, gm4
    }
    for (int i = 0; i < kDepth + 1; ++i) {
      AL(h->ctr3[i], bytes);
      if (cudaMemsetAsync(h->ctr3[i], 0, bytes, st) != cudaSuccess) return CKPT_ECUDA;
    }
    h->ctr_bytes = bytes;
    h->ctr_dbits_off = dbits_off;
    h->ctr_tcc_off = tcc_off;
    h->ctr_bsum_off = bsum_off;
    h->ctr_gsum_off = gsum_off;
    for (int s = 1; s < h->S; ++s) h->ctr_stage_off[s] = off[s];
  }
  AL(h->scratch, n_tiles << h->t0);
  AL(h->tilecnt, n_tiles);
  AL(h->wl0, n_tiles);
  AL(h->lmask, n_tiles * kLmWords);
  for (int i = 0; i < kDepth; ++i) AL(h->defer2[i], n / 32 + 16);   // (tile << 3 | round), one per 32 candidates
  h->defer = h->defer2[0];
#undef AL
  if (cudaMemsetAsync(h->tilecnt, 0, n_tiles * sizeof(uint4), st) != cudaSuccess) return CKPT_ECUDA;
  if (h->trace_path) {
    if (dalloc(h, &h->trace, (uint64_t)kTraceLanes * kTraceLaneCap) != cudaSuccess ||
        dalloc(h, &h->trace_n, 8 * kTraceLanes) != cudaSuccess)
      return CKPT_ENOMEM;
  }
  bool reserved = false;
  for (uint64_t va : kArenaVA)
    if (va >= 4 * (h->B + 12 * n + 1024) && h->arena[0].reserve(va)) { reserved = true; break; }
  if (!reserved) return CKPT_ENOMEM;
  h->geo_set = true;
  return CKPT_OK;
}

Geo make_geo(const ckpt_ctx* h, uint32_t k) {
  Geo g;
  g.B = h->B;
  g.n = h->n;
  g.m = h->m;
  g.C = h->C;
  g.h = h->h;
  g.t0 = h->t0;
  g.k = k;
  g.epoch = k + 1;
  return g;
}

int ensure_table(ckpt_ctx* h, cudaStream_t st, bool pipe) {
  // worst case: every node inserted, by this call and, for pipelined calls, by
  // the call that may still be in flight (its inserts are not counted in `live` yet); sized
  // for two from the first pipelined call on, so the growth happens there and not later
  uint64_t need = h->live + (pipe ? kDepth : 1) * (2 * h->n - 1);
  if (h->dbg & 256) need = h->live + h->n / 2;   // diagnostics only: undersized table experiment
  if (h->cap && (double)need <= kMaxLoad * (double)h->cap) return CKPT_OK;
  // geometric growth: at least double, so a lineage whose record keeps growing pays for a
  // (stream-ordered) reallocation and rehash only O(log) times
  uint64_t new_cap = (uint64_t)((double)need / kGrowLoad) + 1;
  if (h->cap && new_cap < 2 * h->cap) new_cap = 2 * h->cap;
  if (new_cap < 4096) new_cap = 4096;
  if (new_cap >= (1ull << 32)) return CKPT_ENOMEM;   // slot ids are u32
  // Growth without a host synchronisation (ckpt.h: one sync per call): the new table is
  // allocated (cudaMalloc: < 1 ms for GBs on B200, where a stream-ordered cudaMallocAsync
  // took 6-23 ms, tools/alloc_probe.cu), filled and rehashed on the caller's stream. The
  // old table is read by that rehash, so it is retired, not freed: cudaFree would
  // synchronise the device. Retired tables (geometric growth: together at most the size of
  // the current one) are released by ckpt_destroy.
  Slot* nt = nullptr;
  if (cudaMalloc(reinterpret_cast<void**>(&nt), new_cap * sizeof(Slot)) != cudaSuccess) {
    cudaGetLastError();
    return CKPT_ENOMEM;
  }
  if (cudaMemsetAsync(nt, 0xFF, new_cap * sizeof(Slot), st) != cudaSuccess) return CKPT_ECUDA;
  if (h->tab) {
    if (launch_rehash(h->tab, h->cap, nt, new_cap, st) != cudaSuccess) return CKPT_ECUDA;
    h->retired.push_back(h->tab);
  }
  h->tab = nt;
  h->cap = new_cap;
  return CKPT_OK;
}

int make_tmap(ckpt_ctx* h, const void* buf, const LeafParams& lp, CUtensorMap* map) {
  cuuint64_t dims[3];
  cuuint64_t strides[2];
  cuuint32_t box[3];
  cuuint32_t es[3] = {1, 1, 1};
  cuuint32_t rank;
  if (lp.mode3d == 2) {   // rows of C bytes; a box past C is zero-filled (not read)
    rank = 2;
    dims[0] = h->C; dims[1] = lp.n_main;
    strides[0] = h->C;
    box[0] = 128; box[1] = kLeafThreads;
  } else if (lp.mode3d) {
    rank = 3;
    dims[0] = 128; dims[1] = h->C / 128; dims[2] = lp.n_main;
    strides[0] = 128; strides[1] = h->C;
    box[0] = 128; box[1] = 1; box[2] = kLeafThreads;
  } else {
    rank = 2;
    dims[0] = 128; dims[1] = lp.n_main * h->C / 128;
    strides[0] = 128;
    box[0] = 128; box[1] = lp.stage_bytes / 128;
  }
  // MODE3D 2: a chunk row starts anywhere in a 128-B line, and 256-B promotion fetched lines of
  // the neighbouring rows early (K1 at C = 176: 0.265 ms/GiB with 256-B, 0.221 with 128-B promotion)
  const CUtensorMapL2promotion promo =
      lp.mode3d == 2 ? CU_TENSOR_MAP_L2_PROMOTION_L2_128B : CU_TENSOR_MAP_L2_PROMOTION_L2_256B;
  CUresult r = h->encode(map, CU_TENSOR_MAP_DATA_TYPE_UINT8, rank, const_cast<void*>(buf), dims, strides, box, es,
                         CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, promo,
                         CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) fprintf(stderr, "libckpt: cuTensorMapEncodeTiled failed (%d)\n", (int)r);
  return r == CUDA_SUCCESS ? CKPT_OK : CKPT_ECUDA;
}

void fill_diff(const ckpt_ctx* h, uint32_t id, const Totals& t, uint8_t* ptr, ckpt_diff* d) {
  std::memset(d, 0, sizeof(*d));
  d->id = id;
  d->chunk_bytes = h->C;
  d->dev_ptr = ptr;
  d->meta_bytes = t.meta_bytes;
  d->data_bytes = t.data_bytes;
  d->bytes = t.meta_bytes + t.data_bytes;
  d->buf_bytes = h->B;
  d->n_leaves = h->n;
  d->n_first_regions = t.nF;
  d->n_shift_regions = t.nS;
  d->n_first = t.n_first;
  d->n_spatial = t.n_spatial;
  d->n_temporal = t.n_temporal;
  d->n_fixed = h->n - t.n_first - t.n_spatial - t.n_temporal;
  d->list_entries = t.n_first + t.n_spatial + t.n_temporal;
  d->record_size = h->live;
  d->record_capacity = h->cap;
  d->phase2_inserts = t.p2_inserts;
  d->phase3_inserts = t.p3_inserts;
}

// ---- host twins of dev.cuh's tree geometry (R3), used only to validate imported diffs
// before any kernel reads them (ckpt_import: a corrupted body must not steer device writes)
struct HostGeo {
  uint64_t B, n, m;
  uint32_t C;
  int h;
};

uint64_t hg_chunk_of_vslot(const HostGeo& g, uint64_t v) { return v <= g.m ? v : g.m + (v - g.m) / 2; }

// chunk range [lo, hi) of heap node `node`; false if the id names no node of the tree
bool hg_node_range(const HostGeo& g, uint64_t node, uint64_t& lo, uint64_t& hi) {
  if (node >= 2 * g.n - 1) return false;
  const int depth = 63 - __builtin_clzll(node + 1);
  if (depth > g.h) return false;
  const int L = g.h - depth;
  const uint64_t j = node + 1 - (1ull << depth);
  lo = hg_chunk_of_vslot(g, j << L);
  hi = hg_chunk_of_vslot(g, (j + 1) << L);
  return lo < hi;
}

uint64_t hg_range_bytes(const HostGeo& g, uint64_t lo, uint64_t hi) {
  const uint64_t e = std::min<uint64_t>(hi * g.C, g.B);
  return e - lo * g.C;
}

// The body of a diff to import: every node id names a tree node; FIRST and
// SHIFT regions are sorted by first chunk and pairwise disjoint; a SHIFT source checkpoint is
// <= id and its source node covers as many bytes as the region; the FIRST regions' bytes
// sum to data_bytes. Basic: the bitmap's popcount is nF, no bit at or past n, and the
// changed chunks' bytes sum to data_bytes. Full form: the root alone, the whole buffer.
bool validate_import_body(const HostGeo& g, const uint8_t* hd, uint32_t id, int mode, bool full, uint64_t nF,
                          uint64_t nS, uint64_t data) {
  auto rd32 = [&](uint64_t o) { uint32_t v; std::memcpy(&v, hd + o, 4); return v; };
  if (mode == kModeBasic) {
    const uint64_t words = (g.n + 31) / 32;
    uint64_t cnt = 0;
    bool last_set = false;
    for (uint64_t w = 0; w < words; ++w) {
      uint32_t x = rd32(64 + 4 * w);
      if (w + 1 == words && (g.n & 31)) {
        if (x >> (g.n & 31)) return false;   // bits past n
      }
      if (w + 1 == words) last_set = (x >> ((g.n - 1) & 31)) & 1u;
      cnt += __builtin_popcount(x);
    }
    if (cnt != nF) return false;
    const uint64_t bytes = nF * g.C - (last_set ? g.n * g.C - g.B : 0);
    return bytes == data;
  }
  if (full) return nF == 1 && nS == 0 && rd32(64) == 0 && data == g.B;
  uint64_t sum = 0, prev_hi = 0;
  std::vector<std::pair<uint64_t, uint64_t>> fr;
  fr.reserve(nF);
  for (uint64_t i = 0; i < nF; ++i) {
    uint64_t lo, hi;
    if (!hg_node_range(g, rd32(64 + 4 * i), lo, hi) || lo < prev_hi) return false;
    prev_hi = hi;
    sum += hg_range_bytes(g, lo, hi);
    fr.emplace_back(lo, hi);
  }
  if (sum != data) return false;
  prev_hi = 0;
  uint64_t f = 0;   // FIRST regions before the current SHIFT region (disjointness by merge)
  for (uint64_t i = 0; i < nS; ++i) {
    const uint64_t e = 64 + 4 * nF + 12 * i;
    uint64_t lo, hi, vlo, vhi;
    if (!hg_node_range(g, rd32(e), lo, hi) || lo < prev_hi) return false;
    if (!hg_node_range(g, rd32(e + 4), vlo, vhi) || rd32(e + 8) > id) return false;
    if (hg_range_bytes(g, lo, hi) != hg_range_bytes(g, vlo, vhi)) return false;
    while (f < fr.size() && fr[f].second <= lo) ++f;
    if (f < fr.size() && fr[f].first < hi) return false;   // overlaps a FIRST region
    prev_hi = hi;
  }
  return true;
}

}  // namespace

// Green contexts (CUDA 12.4+ driver API, through cudaGetDriverEntryPoint): the device's SMs
// split into m for the chain and the rest for K1; one stream in each. The kernels' attributes
// (K1's dynamic shared memory) are set and the modules loaded in both contexts.
template <class F>
static F drv(const char* name) {
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &fn, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess) {
    cudaGetLastError();
    return nullptr;
  }
  return reinterpret_cast<F>(fn);
}

static int make_green(ckpt_ctx* h, ckpt_ctx::Part& P, int m, int prio_hi) {
  auto getres = drv<CUresult (*)(CUdevice, CUdevResource*, CUdevResourceType)>("cuDeviceGetDevResource");
  auto split = drv<CUresult (*)(CUdevResource*, unsigned*, const CUdevResource*, CUdevResource*, unsigned, unsigned)>(
      "cuDevSmResourceSplitByCount");
  auto gendesc = drv<CUresult (*)(CUdevResourceDesc*, CUdevResource*, unsigned)>("cuDevResourceGenerateDesc");
  auto gcreate = drv<CUresult (*)(CUgreenCtx*, CUdevResourceDesc, CUdevice, unsigned)>("cuGreenCtxCreate");
  auto gstream = drv<CUresult (*)(CUstream*, CUgreenCtx, unsigned, int)>("cuGreenCtxStreamCreate");
  auto fromgreen = drv<CUresult (*)(CUcontext*, CUgreenCtx)>("cuCtxFromGreenCtx");
  auto getcur = drv<CUresult (*)(CUcontext*)>("cuCtxGetCurrent");
  auto setcur = drv<CUresult (*)(CUcontext)>("cuCtxSetCurrent");
  if (!getres || !split || !gendesc || !gcreate || !gstream || !fromgreen || !getcur || !setcur) return CKPT_ECUDA;
  const CUdevice dev = (CUdevice)h->device;
  CUdevResource all, grp, rest;
  unsigned ng = 1;
  CUdevResourceDesc dk, dc;
  if (getres(dev, &all, CU_DEV_RESOURCE_TYPE_SM) != CUDA_SUCCESS ||
      split(&grp, &ng, &all, &rest, 0, (unsigned)m) != CUDA_SUCCESS || ng != 1 ||
      gendesc(&dk, &rest, 1) != CUDA_SUCCESS || gendesc(&dc, &grp, 1) != CUDA_SUCCESS ||
      gcreate(&P.g[0], dk, dev, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS ||
      gcreate(&P.g[1], dc, dev, CU_GREEN_CTX_DEFAULT_STREAM) != CUDA_SUCCESS)
    return CKPT_ECUDA;
  CUstream sk, sc;
  if (gstream(&sk, P.g[0], CU_STREAM_NON_BLOCKING, 0) != CUDA_SUCCESS ||
      gstream(&sc, P.g[1], CU_STREAM_NON_BLOCKING, prio_hi) != CUDA_SUCCESS)
    return CKPT_ECUDA;
  P.m = m;
  P.k1s = reinterpret_cast<cudaStream_t>(sk);
  P.cs = reinterpret_cast<cudaStream_t>(sc);
  P.sm_k1 = (int)rest.sm.smCount;
  P.sm_chain = (int)grp.sm.smCount;
  CUcontext prim = nullptr;
  if (getcur(&prim) != CUDA_SUCCESS) return CKPT_ECUDA;
  for (int i = 0; i < 2; ++i) {
    CUcontext c = nullptr;
    if (fromgreen(&c, P.g[i]) != CUDA_SUCCESS || setcur(c) != CUDA_SUCCESS) return CKPT_ECUDA;
    const bool ok = leaf_setup_attributes() == cudaSuccess && tree_setup_attributes() == cudaSuccess &&
                    preload_leaf() == cudaSuccess && preload_tree() == cudaSuccess && preload_compact() == cudaSuccess;
    setcur(prim);
    if (!ok) { cudaGetLastError(); return CKPT_ECUDA; }
  }
  return CKPT_OK;
}

// The partition of a pipelined call: the chain's SMs from the candidate count of the last
// collected call (the chain's work grows with it). Measured on config 2 (1 GiB, C = 128,
// DESIGN.md §1a): ~6 K candidates run best with 16 chain SMs (0.176 ms per step against 0.206
// without a partition), ~59 K with 20-32 (0.207 against 0.222), and ~300 K (p = 5 %) best
// without one (a 32-SM chain took 0.44 ms). Below ~2 600 candidates per chain SM a partition
// of that size keeps the chain within the next K1 (59 K on 24 SMs: 0.2054 ms; on 20: 0.2068;
// on 16, 3 700 per SM, the chain no longer keeps up: 0.277). K1 on 16 SMs fewer streams ~3 % slower,
// which outweighs the hidden chain on long K1 passes (config 3, 4 GiB at C = 4096: 0.715 ->
// 0.733 ms per step), so buffers above 2 GiB are not partitioned.
static const ckpt_ctx::Part* pick_part(const ckpt_ctx* h) {
  if (!h->green_ok) return nullptr;
  int i = -1;
  if (h->forced_m) {
    i = 0;
  } else if (h->last_cand != ~0ull && h->B <= (2ull << 30)) {
    for (int j = 0; j < ckpt_ctx::kMaxParts && i < 0; ++j)
      if (h->last_cand <= (uint64_t)CKPT_GREEN_CAND_PER_SM * (uint64_t)ckpt_ctx::kPartSMs[j]) i = j;
  }
  if (i < 0) return nullptr;
  return &h->parts[i];
}

extern "C" {

static int drain(ckpt_ctx* h);   // collects the calls in flight (ckpt_checkpoint_submit)

const char* ckpt_strerror(int status) {
  switch (status) {
    case CKPT_OK: return "ok";
    case CKPT_EINVAL: return "invalid argument";
    case CKPT_ENOMEM: return "out of device memory";
    case CKPT_ECUDA: return "CUDA error";
    case CKPT_ERANGE: return "checkpoint id out of range";
    case CKPT_ESTATE: return "handle poisoned by an earlier CUDA error";
    case CKPT_ECOLLIDE: return "128-bit digest collision detected";
    default: return "unknown status";
  }
}

int ckpt_create(uint32_t chunk_bytes, ckpt_handle* out) { return ckpt_create_mode(chunk_bytes, CKPT_MODE_TREE, out); }

int ckpt_create_mode(uint32_t chunk_bytes, int mode, ckpt_handle* out) {
  if (!out || chunk_bytes < 32 || chunk_bytes > 65536 || chunk_bytes % 16) return CKPT_EINVAL;
  if (mode != CKPT_MODE_TREE && mode != CKPT_MODE_LIST && mode != CKPT_MODE_BASIC) return CKPT_EINVAL;
  *out = nullptr;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return CKPT_ECUDA; }
  cudaDeviceProp prop;
  if (cudaGetDeviceProperties(&prop, dev) != cudaSuccess) { cudaGetLastError(); return CKPT_ECUDA; }
  if (prop.major != 10) return CKPT_ECUDA;   // built for sm_100a only; no fallback
  ckpt_ctx* h = new (std::nothrow) ckpt_ctx();
  if (!h) return CKPT_ENOMEM;
  h->device = dev;
  h->num_sms = prop.multiProcessorCount;
  h->C = chunk_bytes;
  h->mode = mode;
  h->trace_path = getenv("CKPT_TRACE");
  if (const char* d = getenv("CKPT_DBG")) h->dbg = atoi(d);
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess || !fn) {
    delete h;
    return CKPT_ECUDA;
  }
  h->encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  if (leaf_setup_attributes() != cudaSuccess || tree_setup_attributes() != cudaSuccess ||
      preload_leaf() != cudaSuccess || preload_tree() != cudaSuccess || preload_compact() != cudaSuccess ||
      preload_restore() != cudaSuccess) {
    delete h;
    return CKPT_ECUDA;
  }
  if (!h->arena[0].init(dev)) {
    delete h;
    return CKPT_ECUDA;
  }
  // The internal stream is a BLOCKING stream: work the caller enqueued earlier on the legacy
  // default stream (torch's default) completes before ckpt_restore / ckpt_import /
  // ckpt_leaf_digests touch memory on it (ckpt.h ordering contract).
  if (cudaStreamCreateWithFlags(&h->internal, cudaStreamDefault) != cudaSuccess) { delete h; return CKPT_ECUDA; }
  for (int i = 0; i < kDepth; ++i)
    if (cudaHostAlloc(&h->tot_host2[i], sizeof(Totals), cudaHostAllocMapped) != cudaSuccess) { delete h; return CKPT_ECUDA; }
  if (cudaEventCreateWithFlags(&h->done_ev, cudaEventDisableTiming) != cudaSuccess) { delete h; return CKPT_ECUDA; }
  for (int i = 0; i < kDepth; ++i) std::memset(h->tot_host2[i], 0, sizeof(Totals));   // done = 0: epochs start at 1
  for (int r = 0; r < ckpt_ctx::kEvRing; ++r) {
    h->ev_id[r] = -1;
    for (int i = 0; i < 6; ++i) cudaEventCreate(&h->evr[r][i]);
  }
  *out = h;
  return CKPT_OK;
}

int ckpt_destroy(ckpt_handle h) {
  if (!h) return CKPT_EINVAL;
  cudaSetDevice(h->device);
  cudaDeviceSynchronize();
  for (void* p : h->allocs) cudaFree(p);
  for (int i = 0; i < h->arenas_ready; ++i) h->arena[i].release_all();
  for (auto& d : h->diffs)
    for (void* q : {(void*)d.Flo, (void*)d.Foff, (void*)d.Slo, (void*)d.Soff, (void*)d.Ssrc, (void*)d.Fseg, (void*)d.Sseg,
                    (void*)d.Cch, (void*)d.Csrc})
      if (q) cudaFree(q);
  for (void* q : {(void*)h->owner, (void*)h->rs_len, h->rs_scan, (void*)h->rs_err, (void*)h->rs_chain})
    if (q) cudaFree(q);
  if (h->tab) cudaFree(h->tab);
  for (void* q : h->retired) cudaFree(q);
  for (int i = 0; i < kDepth; ++i)
    if (h->tot_host2[i]) cudaFreeHost(h->tot_host2[i]);
  for (int i = 0; i < kDepth; ++i) {
    if (h->ev_k1[i]) cudaEventDestroy(h->ev_k1[i]);
    if (h->ev_chain[i]) cudaEventDestroy(h->ev_chain[i]);
  }
  if (h->cs) cudaStreamDestroy(h->cs);
  for (int i = 0; i < kDepth; ++i)
    if (h->ev_in[i]) cudaEventDestroy(h->ev_in[i]);
  {
    auto gdestroy = drv<CUresult (*)(CUgreenCtx)>("cuGreenCtxDestroy");
    for (auto& P : h->parts) {
      if (P.k1s) cudaStreamDestroy(P.k1s);
      if (P.cs) cudaStreamDestroy(P.cs);
      for (int i = 0; i < 2; ++i)
        if (P.g[i] && gdestroy) gdestroy(P.g[i]);
    }
  }
  if (h->staging) cudaFree(h->staging);
  for (int r = 0; r < ckpt_ctx::kEvRing; ++r)
    for (int i = 0; i < 6; ++i) if (h->evr[r][i]) cudaEventDestroy(h->evr[r][i]);
  if (h->internal) cudaStreamDestroy(h->internal);
  if (h->done_ev) cudaEventDestroy(h->done_ev);
  cudaGetLastError();
  delete h;
  return CKPT_OK;
}

int ckpt_num_checkpoints(ckpt_handle h, uint32_t* count) {
  if (!h || !count) return CKPT_EINVAL;
  *count = (uint32_t)(h->diffs.size() + h->inflight.size());   // submitted, collected or not
  return CKPT_OK;
}

int ckpt_kernel_launches(ckpt_handle h, uint64_t* count) {
  if (!h || !count) return CKPT_EINVAL;
  *count = h->launches;
  return CKPT_OK;
}

int ckpt_host_syncs(ckpt_handle h, uint64_t* count) {
  if (!h || !count) return CKPT_EINVAL;
  *count = h->host_syncs;
  return CKPT_OK;
}

int ckpt_set_variant(ckpt_handle h, uint32_t flags, uint32_t switch_permille) {
  if (!h) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (h->mode != kModeTree || !h->diffs.empty() || !h->inflight.empty() || (flags & ~7u) || switch_permille > 1000)
    return CKPT_EINVAL;
  h->variant = flags;
  h->switch_permille = switch_permille;
  return CKPT_OK;
}

int ckpt_set_profiling(ckpt_handle h, int enable) {
  if (!h) return CKPT_EINVAL;
  if (enable < 0 || enable > 2) return CKPT_EINVAL;
  h->prof = enable;
  return CKPT_OK;
}

int ckpt_phase_times_of(ckpt_handle h, uint32_t id, float* times, int n) {
  if (!h || !times) return CKPT_EINVAL;
  BIND(h);
  if (const int rd = drain(h)) return rd;
  if (id >= h->diffs.size()) return CKPT_ERANGE;
  const int r = (int)(id % ckpt_ctx::kEvRing);
  float t[12] = {};
  if (h->ev_id[r] == (int64_t)id) {
    cudaEvent_t* e = h->evr[r];
    cudaEventSynchronize(e[5]);   // the call returned on its statistics; its kernels may still run
    if (h->ev_level[r] >= 2) {
      for (int i = 0; i < 5; ++i) cudaEventElapsedTime(&t[i], e[i], e[i + 1]);   // K1, K1b, phase 2, phase 3, compaction
    } else {
      cudaEventElapsedTime(&t[0], e[0], e[1]);   // K1 only
    }
    cudaEventElapsedTime(&t[5], e[0], e[5]);
    cudaGetLastError();
  }
  if (id + 1 == h->diffs.size())
    for (int i = 6; i < 12; ++i) t[i] = h->times[i];
  for (int i = 0; i < n && i < 12; ++i) times[i] = t[i];
  return CKPT_OK;
}

int ckpt_phase_times(ckpt_handle h, float* times, int n) {
  if (!h || !times) return CKPT_EINVAL;
  BIND(h);
  if (const int rd = drain(h)) return rd;
  if (h->diffs.empty()) {
    for (int i = 0; i < n && i < 12; ++i) times[i] = 0.f;
    return CKPT_OK;
  }
  return ckpt_phase_times_of(h, (uint32_t)(h->diffs.size() - 1), times, n);
}

// Adds the kernels enqueued during one API call to the handle's launch counter.
struct LaunchCount {
  ckpt_ctx* h;
  uint64_t start;
  explicit LaunchCount(ckpt_ctx* hh) : h(hh), start(g_kernel_launches) {}
  ~LaunchCount() { h->launches += g_kernel_launches - start; }
};

// Point the per-call views at call k's buffers: counters ctr3[k % 3], candidate bits and
// deferred tiles of slot k % kDepth.
static void select_ctr(ckpt_ctx* h, uint32_t k) {
  h->cand = h->cand2[k % kDepth];
  h->defer = h->defer2[k % kDepth];
  uint8_t* c = h->ctr3[k % (kDepth + 1)];
  h->tot = reinterpret_cast<Totals*>(c);
  h->dbits = reinterpret_cast<uint32_t*>(c + h->ctr_dbits_off);
  h->tcc = reinterpret_cast<uint32_t*>(c + h->ctr_tcc_off);
  h->blocksum = reinterpret_cast<unsigned long long*>(c + h->ctr_bsum_off);
  h->gsum = reinterpret_cast<unsigned long long*>(c + h->ctr_gsum_off);
  for (int s = 1; s < h->S; ++s) {
    h->arr2[s] = reinterpret_cast<uint32_t*>(c + h->ctr_stage_off[s]);
    h->arr3[s] = h->arr2[s] + h->ngroups[s];
    h->arr4[s] = h->arr3[s] + h->ngroups[s];
    h->dcnt[s] = h->arr4[s] + h->ngroups[s];
    h->gm2[s] = h->dcnt[s] + h->ngroups[s];
    h->gm3[s] = h->gm2[s] + 32 * h->ngroups[s];
    h->gm4[s] = h->gm3[s] + 64 * h->ngroups[s];
  }
}

using clk = std::chrono::steady_clock;
static float ms_since(clk::time_point a, clk::time_point b) { return std::chrono::duration<float, std::milli>(b - a).count(); }

// Pipelined calls only: the chain stream, the events and the second arena (created once).
static int ensure_pipe_state(ckpt_ctx* h, uint64_t bytes) {
  if (h->cs) return CKPT_OK;
  // non-blocking: work on the legacy default stream must not serialise against the chain.
  // Highest priority: when K1 of the next call and this chain's kernels both wait for SM
  // resources, the (short, latency-bound) chain kernels are placed first and K1's persistent
  // CTAs fill the rest, growing back as the chain's CTAs exit
  int lo = 0, hi = 0;   // numerically lowest = highest priority
  if (cudaDeviceGetStreamPriorityRange(&lo, &hi) != cudaSuccess) { cudaGetLastError(); return CKPT_ECUDA; }
  // (measured: with default priority, config 2 steps were 0.220 ms when the chain won the
  // race and 0.4-2.4 ms when K1's CTAs starved the chain's statically partitioned K1b and
  // gather; with the highest priority 0.226-0.228 ms, every run)
  if (cudaStreamCreateWithPriority(&h->cs, cudaStreamNonBlocking, hi) != cudaSuccess) { cudaGetLastError(); return CKPT_ECUDA; }
  // SM partitions (CKPT_GREEN=0 disables them): chain sizes 16, 24, 32, 40 SMs. Not under a
  // profiling / injection tool: under ncu 2025.2 a pipelined lineage on green contexts failed
  // at its first partitioned call ("Failed to prepare kernel for profiling")
  const char* gm = getenv("CKPT_GREEN");
  bool tool = false;
  for (const char* v : {"CUDA_INJECTION64_PATH", "NV_COMPUTE_PROFILER_PERFWORKS_DIR", "NVIDIA-PROCESS-TRACKING-CONFIGURATION"})
    if (const char* e = getenv(v)) tool = tool || *e;
  // Created here, at the first pipelined call (host time once: a partition created when the
  // candidate count first calls for it stalled that call by 10-25 ms, inside a timed lineage),
  // and only for buffers that can use them (pick_part: <= 2 GiB)
  const int forced = gm ? atoi(gm) : 0;
  if (!(gm && forced == 0) && !tool && h->num_sms >= 96 && (bytes <= (2ull << 30) || forced >= 8)) {
    h->prio_hi = hi;
    if (forced >= 8 && forced <= h->num_sms - 64) h->forced_m = forced;
    bool ok = true;
    for (int j = 0; j < (h->forced_m ? 1 : ckpt_ctx::kMaxParts) && ok; ++j)
      ok = make_green(h, h->parts[j], h->forced_m ? h->forced_m : ckpt_ctx::kPartSMs[j], hi) == CKPT_OK;
    if (!ok) cudaGetLastError();   // no partitions on this device: the shared form
    h->green_ok = ok;
    for (int i = 0; i < kDepth; ++i)
      if (cudaEventCreateWithFlags(&h->ev_in[i], cudaEventDisableTiming) != cudaSuccess) return CKPT_ECUDA;
  }
  for (int i = 0; i < kDepth; ++i)
    if (cudaEventCreateWithFlags(&h->ev_k1[i], cudaEventDisableTiming) != cudaSuccess ||
        cudaEventCreateWithFlags(&h->ev_chain[i], cudaEventDisableTiming) != cudaSuccess) {
      cudaGetLastError();
      return CKPT_ECUDA;
    }
  return CKPT_OK;
}

// Enqueue checkpoint k = (calls so far) of dev_ptr. Synchronous form: every kernel on `st`,
// PDL-chained. Pipelined form (pipe): K1 (+ K1t) on `st`, then K1b .. gather on the chain
// stream h->cs. There K1(k) waits only for K1(k - 1) (the digests it compares with) and for
// the tree phases of call k - 2 (whose candidate bits, candidate digests, deferred tiles and
// counters it reuses), so it runs while call k - 1's tree phases do.
static int launch_call(ckpt_ctx* h, const void* dev_ptr, uint64_t bytes, cudaStream_t st, bool pipe, Inflight* f) {
  const auto t_entry = clk::now();
  if (!h->geo_set) {
    const int r = setup_geometry(h, bytes, st);
    if (r != CKPT_OK) return r;
  }
  const uint32_t k = (uint32_t)(h->diffs.size() + h->inflight.size());
  int r = CKPT_OK;
  // the stream of the tree phases and the gather; with an SM partition (CKPT_GREEN), K1's
  // stream too, and the SMs each side sizes its grids for
  const ckpt_ctx::Part* part = pipe ? pick_part(h) : nullptr;
  const bool green = part != nullptr;
  const cudaStream_t cst = green ? part->cs : pipe ? h->cs : st;
  const cudaStream_t kst = green ? part->k1s : st;
  const int sms_k1 = green ? part->sm_k1 : h->num_sms, sms_chain = green ? part->sm_chain : h->num_sms;
  if (pipe) {
    if (!h->cdig2[0]) {
      for (int i = 0; i < kDepth; ++i)
        if (dalloc(h, &h->cdig2[i], h->n) != cudaSuccess) return CKPT_ENOMEM;
    }
    const bool prev_pipe = k > 0 && h->call_pipe[(k - 1) & 3];
    if (!prev_pipe) {
      // after a synchronous call (or the first call: the setup memsets on st): both streams
      // follow everything enqueued so far
      if (h->pending || k == 0) {
        const cudaStream_t ls = h->pending ? h->last_stream : st;
        CK(cudaEventRecord(h->done_ev, ls));
        if (st != ls) CK(cudaStreamWaitEvent(st, h->done_ev, 0));
        if (cst != ls) CK(cudaStreamWaitEvent(cst, h->done_ev, 0));
        if (kst != st && kst != ls) CK(cudaStreamWaitEvent(kst, h->done_ev, 0));
      }
    } else {
      // K1(k) after K1(k - 1) (prev digests, possibly another stream) and after the chain of
      // call k - 2 (this parity's buffers); the chain follows call k - 1's on h->cs
      CK(cudaStreamWaitEvent(kst, h->ev_k1[(k - 1) % kDepth], 0));
      // K1(k) reuses the buffers of call k - kDepth (slot k % kDepth): after that call's chain
      if (k >= (uint32_t)kDepth && h->call_pipe[(k - kDepth) & 3])
        CK(cudaStreamWaitEvent(kst, h->ev_chain[k % kDepth], 0));
      // a chain on another stream than the previous call's follows that call's chain
      if (cst != h->prev_cs) CK(cudaStreamWaitEvent(cst, h->ev_chain[(k - 1) % kDepth], 0));
    }
    if (green) {   // K1 after the caller's work on `st` (the input buffer)
      CK(cudaEventRecord(h->ev_in[k % kDepth], st));
      CK(cudaStreamWaitEvent(kst, h->ev_in[k % kDepth], 0));
    }
  }
  const auto t_tab = clk::now();
  // a growth's rehash runs on the chain stream: after the inserts of a call still in flight
  r = h->mode == kModeBasic ? CKPT_OK : ensure_table(h, cst, pipe);   // Basic keeps no record
  if (r != CKPT_OK) return r;
  const auto t_arena = clk::now();
  const uint64_t worst = 64 + 12 * h->n + 16 + h->B;
  // pipelined calls rotate over kDepth arenas, so a call's place is known while the sizes of
  // the calls still in flight are not; that arena's last diff (call k - kDepth) is final
  const int ai = pipe ? (int)(k % kDepth) : 0;
  while (ai >= h->arenas_ready) {
    DiffArena& A = h->arena[h->arenas_ready];
    if (!A.init(h->device)) return CKPT_ECUDA;
    bool reserved = false;
    for (uint64_t va : kArenaVA)
      if (va >= 4 * (h->B + 12 * h->n + 1024) && A.reserve(va)) { reserved = true; break; }
    if (!reserved) return CKPT_ENOMEM;
    ++h->arenas_ready;
  }
  // pipelined: an arena's first mapping covers two diffs' worst case, so that its next
  // physical growth (a host cost of 0.5-2 ms, during which a pipelined lineage starves) comes
  // only after about a buffer's worth of diffs, not at its second call
  const bool first_map = pipe && h->arena[ai].mapped() == 0 && worst <= (8ull << 30);
  if (!h->arena[ai].ensure(first_map ? 2 * worst : worst)) return CKPT_ENOMEM;
  h->times[10] = ms_since(t_tab, t_arena);
  h->times[11] = ms_since(t_arena, clk::now());
  uint8_t* out = h->arena[ai].top_ptr();

  const Geo g = make_geo(h, k);
  const uint8_t* buf = static_cast<const uint8_t*>(dev_ptr);
  select_ctr(h, k);
  // the leaf digests the chain reads: prev itself, or (pipelined) this call's copy of its
  // candidates' digests, since the next call's K1 rewrites prev meanwhile
  Digest* const ldig = pipe ? h->cdig2[k % kDepth] : h->prev;

  // ---- record-insert state (K1's insert warp and K1b)
  InsertParams ip;
  std::memset(&ip, 0, sizeof(ip));
  ip.g = g; ip.prev = ldig; ip.cand = h->cand; ip.nwords = h->nwords;
  ip.tab = h->tab; ip.cap = h->cap; ip.res_of = h->res_of;
  ip.tot = h->tot;
  ip.defer = h->defer;
  ip.dbits = h->dbits;
  ip.tcc = h->tcc;
  ip.n_tiles = h->ngroups[0];
  ip.wl0 = h->wl0;
  ip.S = h->S;
  for (int s = 0; s < kMaxStages; ++s) {
    ip.gsz[s] = h->gsz[s];
    ip.dcnt[s] = h->dcnt[s];
  }
  ip.trace = h->trace; ip.trace_n = h->trace_n;
  ip.mode = h->mode;
  ip.sw_permille = (h->variant & CKPT_VARIANT_FULL_SWITCH) ? (int)h->switch_permille : -1;   // R23
  ip.blocksum = h->blocksum;
  ip.gsum = h->gsum;

  // ---- leaf pass configuration
  LeafParams lp;
  std::memset(&lp, 0, sizeof(lp));
  lp.g = g;
  lp.buf = buf;
  lp.prev = h->prev;
  lp.cdig = pipe ? ldig : nullptr;
  lp.cand = h->cand;
  lp.ins = ip;
  const uint64_t n_full = h->B / h->C;
  if (h->C % 128 == 0) {
    lp.mode3d = 1;
    lp.segs = (int)(h->C / 128);
    lp.stage_bytes = 128 * kLeafThreads;
    lp.nst = kLeafStages3d;
    lp.n_main = (n_full / kLeafThreads) * kLeafThreads;
  } else if (h->C < 128) {
    lp.mode3d = 0;
    lp.segs = 1;
    lp.stage_bytes = kLeafThreads * h->C;
    const uint64_t budget = h->C == 32 ? CKPT_K1_C32_SMEM : CKPT_K1_SMALLC_SMEM;
    lp.nst = (int)std::min<uint64_t>(8, std::max<uint64_t>(2, budget / (lp.stage_bytes + kLeafThreads * 16)));
    lp.n_main = (n_full / kLeafThreads) * kLeafThreads;
  } else if (h->C < 1024 && h->C % 128 >= 32) {
    // C > 128, not a multiple of 128: ceil(C / 128) segments, the last one partial. Not kept
    // when that segment is a single 16-B unit (a pipeline step for 16 bytes: slower than the
    // direct-load pass, e.g. C = 144, 1040) nor at C > 1024 (the direct pass was as fast);
    // DESIGN.md §5, K1 design
    lp.mode3d = 2;
    lp.segs = (int)((h->C + 127) / 128);
    lp.stage_bytes = 128 * kLeafThreads;
    lp.nst = kLeafStages3d;
    lp.n_main = (n_full / kLeafThreads) * kLeafThreads;
  } else {
    lp.n_main = 0;   // the direct-load pass only
  }
  lp.tail_begin = lp.n_main;
  // one cursor grab per >= 32 KB of input (CKPT_K1_GRAB_BYTES): a tile is 256 C bytes
  lp.tpg = (uint32_t)std::max<uint64_t>(1, (uint64_t)CKPT_K1_GRAB_BYTES / (kLeafThreads * (uint64_t)h->C));
  CUtensorMap tmap;
  if (lp.n_main) {
    r = make_tmap(h, buf, lp, &tmap);
    if (r != CKPT_OK) { h->poisoned = true; return r; }
  }

  h->ev = h->evr[k % ckpt_ctx::kEvRing];
  h->ev_id[k % ckpt_ctx::kEvRing] = h->prof ? (int64_t)k : -1;
  h->ev_level[k % ckpt_ctx::kEvRing] = h->prof;
  // an event between two kernels stops the second from launching early (PDL), so level 1
  // keeps only the events around K1 (the first kernel) and at the end of the call
  const bool pe = h->prof >= 2;
  const auto t_pre = clk::now();
  if (!pipe) CK(after_last_checkpoint(h, st));   // the previous call's gather may still be finishing
  if (h->trace) CK(cudaMemsetAsync(h->trace_n, 0, 32 * kTraceLanes, kst));
  if (h->prof) CK(cudaEventRecord(h->ev[0], kst));
  // K1 + K1t: hash, fixed test, candidate bits, digest update (Alg.1 l.1-5, l.21)
  CK(launch_leaf_tail(lp, kst));
  CK(launch_leaf(&tmap, lp, sms_k1, kst));
  if (h->prof) CK(cudaEventRecord(h->ev[1], kst));
  if (pipe) {
    CK(cudaEventRecord(h->ev_k1[k % kDepth], kst));
    CK(cudaStreamWaitEvent(cst, h->ev_k1[k % kDepth], 0));
  }
  // K1b: record insert + tie-break (l.6-19), dirty tiles
  // pipelined: a plain launch (the chain stream's previous kernel is the last call's gather,
  // which triggers early; see launch_insert)
  CK(launch_insert(ip, sms_chain, cst, !pipe));
  if (pe) CK(cudaEventRecord(h->ev[2], cst));

  // ---- phase 2 (all stages, one launch), then phase 3 (all stages, one launch): R11
  TreeParams tp;
  std::memset(&tp, 0, sizeof(tp));
  tp.g = g;
  tp.S = h->S;
  tp.n_tiles = h->ngroups[0];
  tp.wl0 = h->wl0;
  tp.buf = buf;
  tp.tcc = h->tcc;
  tp.cand = h->cand; tp.res_of = h->res_of; tp.prev = ldig;
  tp.tab = h->tab; tp.cap = h->cap;
  tp.scratch = h->scratch; tp.tilecnt = h->tilecnt; tp.lmask = h->lmask; tp.tot = h->tot;
  tp.blocksum = h->blocksum;
  tp.gsum = h->gsum;
  tp.trace = h->trace; tp.trace_n = h->trace_n;
  tp.dbg = h->dbg;

  for (int s = 0; s < h->S; ++s) {
    StageParams& sp = tp.st[s];
    sp.Lin = h->Lin[s];
    sp.gsz = h->gsz[s];
    sp.in = s >= 1 ? h->lvl[s] : LevelIO{};
    sp.tdig = h->tdig[s];
    sp.tsrc = h->tsrc[s];
    sp.arr2 = h->arr2[s];
    sp.arr3 = h->arr3[s];
    sp.arr4 = h->arr4[s];
    sp.dcnt = h->dcnt[s];
    sp.gm2 = h->gm2[s];
    sp.gm3 = h->gm3[s];
    sp.gm4 = h->gm4[s];
  }
  tp.list = h->mode == kModeList;
  tp.shift_insert = h->mode == kModeTree && (h->variant & CKPT_VARIANT_SHIFT_INSERT);
  tp.sw_permille = ip.sw_permille;
  if (h->mode != kModeBasic) {   // Basic: no record, no tree
    CK(launch_tree(tp, 2, sms_chain, cst));
    if (pe) CK(cudaEventRecord(h->ev[3], cst));
    if (tp.shift_insert) CK(launch_tree(tp, 4, sms_chain, cst));   // R24 inserts, before any lookup
    CK(launch_tree(tp, 3, sms_chain, cst));
    if (pe) CK(cudaEventRecord(h->ev[4], cst));
  } else if (pe) {
    CK(cudaEventRecord(h->ev[3], cst));
    CK(cudaEventRecord(h->ev[4], cst));
  }

  // ---- compaction + serialisation
  CompactParams cp;
  cp.g = g;
  cp.n_tiles = h->ngroups[0];
  cp.tilecnt = h->tilecnt; cp.scratch = h->scratch; cp.blocksum = h->blocksum;
  cp.gsum = h->gsum; cp.wl0 = h->wl0; cp.tot = h->tot;
  cp.lmask = h->lmask;
  cp.out = out; cp.buf = buf;
  cp.trace = h->trace; cp.trace_n = h->trace_n;
  cp.tot_host = h->tot_host2[k % kDepth];
  cp.dbg = h->dbg;
  cp.ctr_next = reinterpret_cast<uint4*>(h->ctr3[(k + kDepth) % (kDepth + 1)]);   // call k - 1's: complete
  cp.ctr_next_words = h->ctr_bytes / 16;
  cp.mode = h->mode;
  cp.flags = tp.shift_insert ? CKPT_FLAGS_SHIFT_INSERT : h->mode;
  cp.cand = h->cand;
  cp.nwords = h->nwords;
  cp.tcc = h->tcc;
  cp.parts = gather_parts(h->ngroups[0], h->C, sms_chain);
  cp.sw_permille = ip.sw_permille;
  cp.full_first = (h->variant & CKPT_VARIANT_FULL_FIRST) && k == 0;   // R22
  CK(launch_compact(cp, sms_chain, cst));
  if (h->prof) CK(cudaEventRecord(h->ev[5], cst));
  if (pipe) {
    CK(cudaEventRecord(h->ev_chain[k % kDepth], cst));
    h->prev_cs = cst;
  }
  h->last_stream = cst;
  h->pending = true;
  h->call_pipe[k & 3] = pipe;
  f->k = k;
  f->out = out;
  f->arena = ai;
  f->wait_st = cst;
  f->t_entry = t_entry;
  f->t_pre = t_pre;
  f->t_launched = clk::now();
  return CKPT_OK;
}

// Collect a launched call: the one host synchronisation of a call is a spin on the
// completion epoch the gather kernel writes to mapped memory once the statistics are final
// (measured ~8 us per call sooner than cudaStreamSynchronize). The stream is queried now and
// then, so a failed kernel (which never publishes) surfaces as an error instead of a hang.
static int finish_call(ckpt_ctx* h, const Inflight& f, ckpt_diff* diff) {
  const uint32_t k = f.k;
  const uint32_t epoch = k + 1;
  Totals* const th = h->tot_host2[k % kDepth];
  {
    ++h->host_syncs;
    volatile uint32_t* done = &th->done;
    for (uint32_t it = 1;; ++it) {
      if (*done == epoch) break;
      if ((it & 1023) == 0) {
        const cudaError_t q = cudaStreamQuery(f.wait_st);
        if (q == cudaSuccess) {
          if (*done == epoch) break;
          fprintf(stderr, "libckpt: stream idle without completion\n");
          h->poisoned = true;
          return CKPT_ECUDA;
        }
        if (q != cudaErrorNotReady) CK(q);
      }
    }
  }

  std::atomic_thread_fence(std::memory_order_acquire);   // the totals after the epoch
  const auto t_synced = clk::now();

  const Totals t = *th;   // written by the gather kernel (mapped host memory)
  if (h->trace) {   // diagnostics only: dump {t0, t1, stage<<32|G, phase} records
    CK(sync_stream(h, f.wait_st));
    std::vector<uint32_t> cnt(8 * kTraceLanes);
    cudaMemcpy(cnt.data(), h->trace_n, cnt.size() * 4, cudaMemcpyDeviceToHost);
    std::vector<ulonglong4> tr;
    for (uint32_t l = 0; l < kTraceLanes; ++l) {
      const uint32_t nl = std::min<uint32_t>(cnt[8 * l], kTraceLaneCap);
      const size_t o = tr.size();
      tr.resize(o + nl);
      cudaMemcpy(tr.data() + o, h->trace + (size_t)l * kTraceLaneCap, nl * sizeof(ulonglong4), cudaMemcpyDeviceToHost);
    }
    char path[512];
    snprintf(path, sizeof(path), "%s.%u.bin", h->trace_path, k);
    if (FILE* fp = fopen(path, "wb")) { fwrite(tr.data(), sizeof(ulonglong4), tr.size(), fp); fclose(fp); }
  }
  if (h->mode != kModeBasic && t.full_kind != 2) h->live += t.n_first + t.p2_inserts + t.p3_inserts;   // R23: no record op
  h->last_cand = t.n_first + t.n_spatial + t.n_temporal;   // the next pipelined call's partition
  DiffRec rec;
  rec.ptr = f.out;
  fill_diff(h, k, t, f.out, &rec.info);
  rec.collided = t.collisions != 0;
  h->arena[f.arena].commit(rec.info.bytes);
  h->diffs.push_back(rec);
  if (diff) *diff = rec.info;
  // host-side timings: [6] entry->first enqueue, [7] enqueue of the sequence, [8] sync wait, [9] post
  const auto t_exit = clk::now();
  h->times[6] = ms_since(f.t_entry, f.t_pre);
  h->times[7] = ms_since(f.t_pre, f.t_launched);
  h->times[8] = ms_since(f.t_launched, t_synced);
  h->times[9] = ms_since(t_synced, t_exit);
  return rec.collided ? CKPT_ECOLLIDE : CKPT_OK;
}

// Collect every call still in flight (oldest first). Collisions are committed warnings
// (kept per diff for ckpt_checkpoint_wait), not errors.
static int drain(ckpt_ctx* h) {
  while (!h->inflight.empty()) {
    const Inflight f = h->inflight.front();
    h->inflight.pop_front();
    const int r = finish_call(h, f, nullptr);
    if (r != CKPT_OK && r != CKPT_ECOLLIDE) return r;
  }
  return CKPT_OK;
}

static int check_buffer(ckpt_ctx* h, const void* dev_ptr, uint64_t bytes) {
  if (!dev_ptr || bytes == 0 || (reinterpret_cast<uintptr_t>(dev_ptr) & 15)) return CKPT_EINVAL;
  if ((bytes + h->C - 1) / h->C > (1ull << 31)) return CKPT_EINVAL;
  if (h->geo_set && bytes != h->B) return CKPT_EINVAL;   // R17
  cudaPointerAttributes pa;
  if (cudaPointerGetAttributes(&pa, dev_ptr) != cudaSuccess) { cudaGetLastError(); return CKPT_EINVAL; }
  if (pa.type != cudaMemoryTypeDevice && pa.type != cudaMemoryTypeManaged) return CKPT_EINVAL;
  return CKPT_OK;
}

int ckpt_checkpoint(ckpt_handle h, const void* dev_ptr, uint64_t bytes, void* stream, ckpt_diff* diff) {
  if (!h || !diff) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  LaunchCount lc(h);
  int r = check_buffer(h, dev_ptr, bytes);
  if (r != CKPT_OK) return r;
  if ((r = drain(h)) != CKPT_OK) return r;
  Inflight f;
  if ((r = launch_call(h, dev_ptr, bytes, static_cast<cudaStream_t>(stream), false, &f)) != CKPT_OK) return r;
  return finish_call(h, f, diff);
}

int ckpt_checkpoint_submit(ckpt_handle h, const void* dev_ptr, uint64_t bytes, void* stream, uint32_t* id) {
  if (!h || !id) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  LaunchCount lc(h);
  int r = check_buffer(h, dev_ptr, bytes);
  if (r != CKPT_OK) return r;
  // at most kDepth calls in flight: collect the oldest first
  while (h->inflight.size() >= (size_t)kDepth) {
    const Inflight f = h->inflight.front();
    h->inflight.pop_front();
    r = finish_call(h, f, nullptr);
    if (r != CKPT_OK && r != CKPT_ECOLLIDE) return r;
  }
  if ((r = ensure_pipe_state(h, bytes)) != CKPT_OK) return r;
  Inflight f;
  if ((r = launch_call(h, dev_ptr, bytes, static_cast<cudaStream_t>(stream), true, &f)) != CKPT_OK) return r;
  h->inflight.push_back(f);
  *id = f.k;
  return CKPT_OK;
}

int ckpt_checkpoint_wait(ckpt_handle h, uint32_t id, void* stream, ckpt_diff* diff) {
  if (!h || !diff) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (id >= h->diffs.size() + h->inflight.size()) return CKPT_ERANGE;
  while (h->diffs.size() <= id) {
    const Inflight f = h->inflight.front();
    h->inflight.pop_front();
    const int r = finish_call(h, f, nullptr);
    if (r != CKPT_OK && r != CKPT_ECOLLIDE) return r;
  }
  // the rest of call id (its gather) before the caller's later work on `stream`: the event
  // of this parity follows call id's gather (or a later call's, at worst late)
  const cudaStream_t ws = static_cast<cudaStream_t>(stream);
  if (h->call_pipe[id & 3]) CK(cudaStreamWaitEvent(ws, h->ev_chain[id % kDepth], 0));
  *diff = h->diffs[id].info;
  return h->diffs[id].collided ? CKPT_ECOLLIDE : CKPT_OK;
}

int ckpt_diff_info(ckpt_handle h, uint32_t id, ckpt_diff* diff) {
  if (!h || !diff) return CKPT_EINVAL;
  if (!h->inflight.empty()) {
    BIND(h);
    if (const int rd = drain(h)) return rd;
  }
  if (id >= h->diffs.size()) return CKPT_ERANGE;
  *diff = h->diffs[id].info;
  return CKPT_OK;
}

int ckpt_diff_to_host(ckpt_handle h, uint32_t id, void* host_ptr, uint64_t capacity) {
  if (!h || !host_ptr) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (const int rd = drain(h)) return rd;   // calls in flight are collected first
  if (id >= h->diffs.size()) return CKPT_ERANGE;
  const DiffRec& d = h->diffs[id];
  if (capacity < d.info.bytes) return CKPT_EINVAL;
  CK(after_last_checkpoint(h, h->internal));
  CK(cudaMemcpyAsync(host_ptr, d.ptr, d.info.bytes, cudaMemcpyDeviceToHost, h->internal));   // one D2H
  CK(sync_stream(h, h->internal));
  return CKPT_OK;
}

int ckpt_diff_to_host_async(ckpt_handle h, uint32_t id, void* host_ptr, uint64_t capacity, void* stream) {
  if (!h || !host_ptr) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  // a collected diff is copied without collecting the calls still in flight (a pipelined
  // lineage keeps overlapping); an uncollected one is collected first
  if (id >= h->diffs.size())
    if (const int rd = drain(h)) return rd;
  if (id >= h->diffs.size()) return CKPT_ERANGE;
  const DiffRec& d = h->diffs[id];
  if (capacity < d.info.bytes) return CKPT_EINVAL;
  const cudaStream_t ds = static_cast<cudaStream_t>(stream);
  // after the gather of call id: the event of its parity (re-recorded by a later call of the
  // same parity at most, which is later still), or the latest call for a synchronous one
  if (h->call_pipe[id & 3]) CK(cudaStreamWaitEvent(ds, h->ev_chain[id % kDepth], 0));
  else CK(after_last_checkpoint(h, ds));
  CK(cudaMemcpyAsync(host_ptr, d.ptr, d.info.bytes, cudaMemcpyDeviceToHost, ds));
  return CKPT_OK;
}

int ckpt_checkpoint_host(ckpt_handle h, const void* host_ptr, uint64_t bytes, void* stream, void* host_diff,
                         uint64_t host_diff_cap, ckpt_diff* diff) {
  if (!h || !host_ptr || !diff || bytes == 0) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (const int rd = drain(h)) return rd;   // calls in flight are collected first
  if (h->geo_set && bytes != h->B) return CKPT_EINVAL;
  if (h->staging_size < bytes) {
    if (h->staging) cudaFree(h->staging);
    h->staging = nullptr;
    h->staging_size = 0;
    if (cudaMalloc(&h->staging, bytes) != cudaSuccess) { cudaGetLastError(); return CKPT_ENOMEM; }
    h->staging_size = bytes;
  }
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  CK(after_last_checkpoint(h, st));   // the previous call's kernels may still read the staging buffer
  CK(cudaMemcpyAsync(h->staging, host_ptr, bytes, cudaMemcpyHostToDevice, st));
  int r = ckpt_checkpoint(h, h->staging, bytes, stream, diff);
  if (r != CKPT_OK) return r;
  if (host_diff) {
    if (host_diff_cap < diff->bytes) return CKPT_EINVAL;
    CK(cudaMemcpyAsync(host_diff, diff->dev_ptr, diff->bytes, cudaMemcpyDeviceToHost, st));
    CK(sync_stream(h, st));
  }
  return CKPT_OK;
}

// Restore plans of diffs 0..id (built once per diff, then cached; diffs are immutable).
static int ensure_plans(ckpt_ctx* h, uint32_t id, const Geo& g, cudaStream_t st) {
  uint64_t need_len = 1;
  bool any = false;
  const bool basic = h->mode == kModeBasic;
  for (uint32_t c = 0; c <= id; ++c) {
    const DiffRec& d = h->diffs[c];
    if (d.planned) continue;
    any = true;
    need_len = std::max<uint64_t>(need_len, std::max(d.info.n_first_regions, d.info.n_shift_regions));
  }
  if (basic) need_len = std::max<uint64_t>(need_len, 2 * h->nwords);   // word counts + their scan
  if (!any) return CKPT_OK;
  auto grow = [](void** p, size_t bytes) -> bool {
    if (*p) cudaFree(*p);
    *p = nullptr;
    if (cudaMalloc(p, bytes) != cudaSuccess) { cudaGetLastError(); return false; }
    return true;
  };
  if (h->rs_len_cap < need_len) {
    if (!grow(reinterpret_cast<void**>(&h->rs_len), need_len * 8)) return CKPT_ENOMEM;
    h->rs_len_cap = need_len;
  }
  const size_t sb = scan_tmp_bytes_for(need_len);
  if (h->rs_scan_bytes < sb) {
    if (!grow(&h->rs_scan, sb)) return CKPT_ENOMEM;
    h->rs_scan_bytes = sb;
  }
  if (!h->rs_err && !grow(reinterpret_cast<void**>(&h->rs_err), sizeof(int))) return CKPT_ENOMEM;
  if (h->rs_chain_cap < h->diffs.size()) {
    const uint64_t cap = std::max<uint64_t>(64, 2 * h->diffs.size());
    RestoreDiff* nc = nullptr;
    if (cudaMalloc(&nc, cap * sizeof(RestoreDiff)) != cudaSuccess) { cudaGetLastError(); return CKPT_ENOMEM; }
    if (h->rs_chain) cudaFree(h->rs_chain);
    h->rs_chain = nc;
    h->rs_chain_cap = cap;
  }
  if (cudaMemsetAsync(h->rs_err, 0, sizeof(int), st) != cudaSuccess) return CKPT_ECUDA;
  // FIRST plans first: a SHIFT plan of diff c reads the FIRST plan of its source diff c' <= c
  std::vector<RestoreDiff> rd(id + 1, RestoreDiff{});
  for (uint32_t c = 0; c <= id; ++c) {
    DiffRec& d = h->diffs[c];
    RestoreDiff& r = rd[c];
    r.id = c;
    r.composite = (h->variant & CKPT_VARIANT_SHIFT_INSERT) ? 1u : 0u;   // R25
    r.base = d.ptr;
    r.nF = d.info.n_first_regions;
    r.nS = d.info.n_shift_regions;
    r.meta_bytes = d.info.meta_bytes;
    r.data_bytes = d.info.data_bytes;
    if (!d.planned) {
      if ((r.nF && !d.Flo) || (r.nS && !d.Slo)) {
        if ((r.nF && (cudaMalloc(&d.Flo, r.nF * 8) != cudaSuccess || cudaMalloc(&d.Foff, r.nF * 8) != cudaSuccess)) ||
            (r.nS && (cudaMalloc(&d.Slo, r.nS * 8) != cudaSuccess || cudaMalloc(&d.Soff, (r.nS + 1) * 8) != cudaSuccess ||
                      cudaMalloc(&d.Ssrc, r.nS * 8) != cudaSuccess))) {
          cudaGetLastError();
          return CKPT_ENOMEM;
        }
      }
    }
    r.Flo = d.Flo; r.Foff = d.Foff; r.Slo = d.Slo; r.Soff = d.Soff; r.Ssrc = d.Ssrc;
    r.shift_bytes = d.shift_bytes; r.Fseg = d.Fseg; r.Sseg = d.Sseg;
    r.Cch = d.Cch; r.Csrc = d.Csrc;
    if (!d.planned && r.nF &&
        (basic ? restore_prepare_basic(g, r, h->nwords, h->rs_len, h->rs_scan, h->rs_scan_bytes, st)
               : restore_prepare_first(g, r, h->rs_len, h->rs_scan, h->rs_scan_bytes, st)) != cudaSuccess)
      return CKPT_ECUDA;
  }
  if (cudaMemcpyAsync(h->rs_chain, rd.data(), rd.size() * sizeof(RestoreDiff), cudaMemcpyHostToDevice, st) != cudaSuccess)
    return CKPT_ECUDA;
  for (uint32_t c = 0; c <= id; ++c) {
    DiffRec& d = h->diffs[c];
    if (!d.planned && rd[c].nS &&
        restore_prepare_shift(g, rd[c], h->rs_chain, h->rs_len, h->rs_err, h->rs_scan, h->rs_scan_bytes, st) != cudaSuccess)
      return CKPT_ECUDA;
  }
  // SHIFT stream totals (device scalars) back to the host, then the segment maps
  std::vector<unsigned long long> shb(id + 1, 0);
  for (uint32_t c = 0; c <= id; ++c)
    if (!h->diffs[c].planned && rd[c].nS &&
        cudaMemcpyAsync(&shb[c], rd[c].Soff + rd[c].nS, 8, cudaMemcpyDeviceToHost, st) != cudaSuccess)
      return CKPT_ECUDA;
  int herr = 0;
  if (cudaMemcpyAsync(&herr, h->rs_err, sizeof(int), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
      sync_stream(h, st) != cudaSuccess)
    return CKPT_ECUDA;
  if (herr) return CKPT_EINVAL;   // malformed chain (a source outside any FIRST region)
  for (uint32_t c = 0; c <= id; ++c) {
    DiffRec& d = h->diffs[c];
    if (d.planned) continue;
    d.shift_bytes = shb[c];
    rd[c].shift_bytes = shb[c];
    if ((rd[c].nF && cudaMalloc(&d.Fseg, (restore_segments(rd[c].data_bytes) + 1) * 8) != cudaSuccess) ||
        (rd[c].nS && cudaMalloc(&d.Sseg, (restore_segments(shb[c]) + 1) * 8) != cudaSuccess)) {
      cudaGetLastError();
      return CKPT_ENOMEM;
    }
    rd[c].Fseg = d.Fseg;
    rd[c].Sseg = d.Sseg;
    if (restore_segmaps(rd[c], st) != cudaSuccess) return CKPT_ECUDA;
    const uint64_t ncl = (rd[c].data_bytes + h->C - 1) / h->C + (shb[c] + h->C - 1) / h->C;
    if (ncl && (cudaMalloc(&d.Cch, ncl * 4) != cudaSuccess || cudaMalloc(&d.Csrc, ncl * 8) != cudaSuccess)) {
      cudaGetLastError();
      return CKPT_ENOMEM;
    }
    rd[c].Cch = d.Cch;
    rd[c].Csrc = d.Csrc;
    if (restore_claimlist(g, rd[c], h->num_sms, st) != cudaSuccess) return CKPT_ECUDA;
    if (rd[c].composite && rd[c].nS) {
      // R25: SHIFT chunks whose source lies outside the source diff's FIRST data take the
      // address of that chunk in the source checkpoint (its own claim list, complete for
      // older diffs; for this diff, one level per pass since a source node's bytes are
      // regions of smaller levels)
      if (cudaMemcpyAsync(h->rs_chain + c, &rd[c], sizeof(RestoreDiff), cudaMemcpyHostToDevice, st) != cudaSuccess ||
          restore_resolve(g, rd[c], h->rs_chain, h->h + 2, h->rs_err, h->num_sms, st) != cudaSuccess)
        return CKPT_ECUDA;
    }
  }
  {
    int herr2 = 0;
    if (cudaMemcpyAsync(&herr2, h->rs_err, sizeof(int), cudaMemcpyDeviceToHost, st) != cudaSuccess ||
        sync_stream(h, st) != cudaSuccess)
      return CKPT_ECUDA;
    if (herr2) return CKPT_EINVAL;   // a source chunk no diff covers (malformed chain)
  }
  if (sync_stream(h, st) != cudaSuccess) return CKPT_ECUDA;
  for (uint32_t c = 0; c <= id; ++c) h->diffs[c].planned = true;
  return CKPT_OK;
}

static void free_plan(DiffRec& d) {
  for (unsigned long long** q : {&d.Flo, &d.Foff, &d.Slo, &d.Soff, &d.Ssrc, &d.Fseg, &d.Sseg, &d.Csrc}) {
    if (*q) cudaFree(*q);
    *q = nullptr;
  }
  if (d.Cch) cudaFree(d.Cch);
  d.Cch = nullptr;
  d.planned = false;
}

int ckpt_import(ckpt_handle h, const void* host_diff, uint64_t bytes, void* stream) {
  if (!h || !host_diff || bytes < 64) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (const int rd = drain(h)) return rd;   // calls in flight are collected first
  const uint8_t* hd = static_cast<const uint8_t*>(host_diff);
  auto rd32h = [&](size_t o) { uint32_t v; std::memcpy(&v, hd + o, 4); return v; };
  auto rd64h = [&](size_t o) { uint64_t v; std::memcpy(&v, hd + o, 8); return v; };
  uint16_t ver, flags;
  std::memcpy(&ver, hd + 4, 2);
  std::memcpy(&flags, hd + 6, 2);
  const uint32_t id = (uint32_t)h->diffs.size();
  const uint64_t B = rd64h(16), n = rd64h(24), nF = rd64h(32), nS = rd64h(40), data = rd64h(48);
  const bool full_form = flags == CKPT_FLAGS_FULL && h->mode == kModeTree && (h->variant & 3);   // R22 / R23
  const bool shift_insert = h->mode == kModeTree && (h->variant & CKPT_VARIANT_SHIFT_INSERT);      // R24
  const uint16_t want_flags = shift_insert ? (uint16_t)CKPT_FLAGS_SHIFT_INSERT : (uint16_t)h->mode;
  if (rd32h(0) != 0x44504B43u || ver != 1 || (flags != want_flags && !full_form) || rd32h(8) != id ||
      rd32h(12) != h->C)
    return CKPT_EINVAL;
  if (B == 0 || n != (B + h->C - 1) / h->C || n > (1ull << 31) || (h->geo_set && B != h->B)) return CKPT_EINVAL;
  const uint64_t raw = h->mode == kModeBasic ? 64 + 4 * ((n + 31) / 32) : 64 + 4 * nF + 12 * nS;
  const uint64_t meta = (raw + 15) & ~15ull;
  if (meta + data != bytes || data > B || (h->mode == kModeBasic && nS)) return CKPT_EINVAL;
  {
    HostGeo hg;
    hg.B = B;
    hg.n = n;
    hg.C = h->C;
    hg.h = ceil_log2(n);
    hg.m = 2 * n - (1ull << hg.h);
    if (!validate_import_body(hg, hd, id, h->mode, flags == CKPT_FLAGS_FULL, nF, nS, data)) return CKPT_EINVAL;
  }
  if (!h->geo_set) {
    const int r = setup_geometry(h, B, h->internal);
    if (r != CKPT_OK) return r;
  }
  if (h->staging_size < B) {
    if (h->staging) cudaFree(h->staging);
    h->staging = nullptr;
    h->staging_size = 0;
    if (cudaMalloc(&h->staging, B) != cudaSuccess) { cudaGetLastError(); return CKPT_ENOMEM; }
    h->staging_size = B;
  }
  uint8_t* tmp = nullptr;
  int* flag = nullptr;
  if (cudaMalloc(&tmp, bytes) != cudaSuccess || cudaMalloc(&flag, sizeof(int)) != cudaSuccess) {
    cudaGetLastError();
    cudaFree(tmp);
    return CKPT_ENOMEM;
  }
  auto cleanup = [&]() { cudaFree(tmp); cudaFree(flag); };
  cudaStream_t in = h->internal;
  if (cudaMemcpyAsync(tmp, host_diff, bytes, cudaMemcpyHostToDevice, in) != cudaSuccess ||
      sync_stream(h, in) != cudaSuccess) {
    cleanup();
    h->poisoned = true;
    return CKPT_ECUDA;
  }
  // 1. restore checkpoint `id` from diffs 0..id-1 plus the imported diff
  DiffRec rec;
  std::memset(&rec.info, 0, sizeof(rec.info));
  rec.info.id = id;
  rec.info.n_first_regions = nF;
  rec.info.n_shift_regions = nS;
  rec.info.meta_bytes = meta;
  rec.info.data_bytes = data;
  rec.info.bytes = bytes;
  rec.ptr = tmp;
  h->diffs.push_back(rec);
  int rc = ckpt_restore(h, id, h->staging);
  free_plan(h->diffs.back());
  h->diffs.pop_back();
  if (rc != CKPT_OK) { cleanup(); return rc == CKPT_EINVAL ? CKPT_EINVAL : rc; }
  // 2. de-duplicate it again: rebuilds the record and the leaf digests exactly
  ckpt_diff d;
  rc = ckpt_checkpoint(h, h->staging, B, stream, &d);
  if (rc != CKPT_OK && rc != CKPT_ECOLLIDE) { cleanup(); return rc; }
  // 3. the regenerated diff must be the imported one
  int mismatch = d.bytes != bytes;
  if (!mismatch) {
    int hf = 0;
    if (after_last_checkpoint(h, in) != cudaSuccess || cudaMemsetAsync(flag, 0, sizeof(int), in) != cudaSuccess ||
        device_compare(d.dev_ptr, tmp, bytes, flag, h->num_sms, in) != cudaSuccess ||
        cudaMemcpyAsync(&hf, flag, sizeof(int), cudaMemcpyDeviceToHost, in) != cudaSuccess ||
        sync_stream(h, in) != cudaSuccess) {
      cleanup();
      h->poisoned = true;
      return CKPT_ECUDA;
    }
    mismatch = hf;
  }
  cleanup();
  if (mismatch) {
    h->poisoned = true;   // the lineage no longer matches the imported diffs
    return CKPT_EINVAL;
  }
  return CKPT_OK;
}

int ckpt_restore(ckpt_handle h, uint32_t id, void* dev_ptr) {
  if (!h) return CKPT_EINVAL;
  return ckpt_restore_stream(h, id, dev_ptr, h->internal);
}

int ckpt_restore_stream(ckpt_handle h, uint32_t id, void* dev_ptr, void* stream) {
  if (!h || !dev_ptr || (reinterpret_cast<uintptr_t>(dev_ptr) & 15)) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (const int rd = drain(h)) return rd;   // calls in flight are collected first
  if (id >= h->diffs.size()) return CKPT_ERANGE;
  LaunchCount lc(h);
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  CK(after_last_checkpoint(h, st));
  const Geo g = make_geo(h, id);
  int rc = ensure_plans(h, id, g, st);
  if (rc != CKPT_OK) {
    if (rc == CKPT_ECUDA) h->poisoned = true;
    return rc;
  }
  // chunk owners (8 B per chunk) followed by the bitmap of claimed chunks (claim_kernel)
  const size_t owner_bytes = h->n * sizeof(unsigned long long) + (h->n + 31) / 32 * sizeof(uint32_t);
  if (!h->owner) {
    if (cudaMalloc(&h->owner, owner_bytes) != cudaSuccess) { cudaGetLastError(); return CKPT_ENOMEM; }
  }
  CK(cudaMemsetAsync(h->owner, 0, owner_bytes, st));
  uint8_t* outp = static_cast<uint8_t*>(dev_ptr);
  // claims by bitmap when the newer diffs cover more than the buffer's chunks in total (a
  // long lineage of heavily rewritten checkpoints: config 4 restores 11-20 % faster, config 2
  // 3 % slower with it, restore)
  uint64_t newer = 0;
  for (uint32_t c = 1; c <= id; ++c)
    newer += (h->diffs[c].info.data_bytes + h->diffs[c].shift_bytes + h->C - 1) / h->C;
  const bool bitmap = newer > h->n;
  for (int64_t c = id; c >= 0; --c) {
    const DiffRec& d = h->diffs[c];
    RestoreDiff r = {};
    r.id = (uint32_t)c;
    r.base = d.ptr;
    r.nF = d.info.n_first_regions;
    r.nS = d.info.n_shift_regions;
    r.meta_bytes = d.info.meta_bytes;
    r.data_bytes = d.info.data_bytes;
    r.Flo = d.Flo; r.Foff = d.Foff; r.Slo = d.Slo; r.Soff = d.Soff; r.Ssrc = d.Ssrc;
    r.shift_bytes = d.shift_bytes; r.Fseg = d.Fseg; r.Sseg = d.Sseg;
    r.Cch = d.Cch; r.Csrc = d.Csrc;
    CK(restore_claim(g, r, h->owner, bitmap, h->num_sms, st));
  }
  CK(restore_copy(g, h->owner, outp, h->num_sms, st));
  CK(sync_stream(h, st));
  return CKPT_OK;
}

int ckpt_leaf_digests(ckpt_handle h, void* dev_out) {
  if (!h || !dev_out) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (const int rd = drain(h)) return rd;   // calls in flight are collected first
  if (!h->geo_set) return CKPT_ERANGE;
  CK(after_last_checkpoint(h, h->internal));
  CK(cudaMemcpyAsync(dev_out, h->prev, h->n * 16, cudaMemcpyDeviceToDevice, h->internal));
  CK(sync_stream(h, h->internal));
  return CKPT_OK;
}

int ckpt_record_dump(ckpt_handle h, uint8_t* host_keys, uint32_t* host_nodes, uint32_t* host_ckpts, uint64_t cap,
                     uint64_t* count) {
  if (!h || !count) return CKPT_EINVAL;
  if (h->poisoned) return CKPT_ESTATE;
  BIND(h);
  if (const int rd = drain(h)) return rd;   // calls in flight are collected first
  *count = h->live;
  if (!h->tab || cap == 0) return CKPT_OK;
  std::vector<Slot> all(h->cap);
  CK(after_last_checkpoint(h, h->internal));
  CK(cudaMemcpyAsync(all.data(), h->tab, h->cap * sizeof(Slot), cudaMemcpyDeviceToHost, h->internal));
  CK(sync_stream(h, h->internal));
  uint64_t i = 0;
  for (const Slot& s : all) {
    if (s.klo == kEmpty && s.khi == kEmpty) continue;
    if (i < cap) {
      if (host_keys) {
        std::memcpy(host_keys + 16 * i, &s.klo, 8);
        std::memcpy(host_keys + 16 * i + 8, &s.khi, 8);
      }
      if (host_nodes) host_nodes[i] = (uint32_t)(s.val & 0xffffffffu);
      if (host_ckpts) host_ckpts[i] = (uint32_t)(s.val >> 32);
    }
    ++i;
  }
  *count = i;
  return CKPT_OK;
}

}  // extern "C"
