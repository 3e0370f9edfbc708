// kernels.h — parameter blocks and host launchers of the sm_100a kernels (internal).
//
// Launch order per checkpoint:
//   K1  leaf hash + fixed test (TMA-staged, persistent)      Alg.1 l.1-5, l.21
//   K1t leaf pass for the ragged tail (direct loads)           same
//   K1b record inserts of the candidate chunks                 Alg.1 l.6-19 (R6)
//   P2  phase 2, all stages in one launch (warp per group)     Alg.1 l.24-32
//   P3  phase 3 + emission, all stages in one launch           Alg.1 l.33-46 (R7-R10)
//   KG  gather: offsets, header, entries and data in one launch
#pragma once
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "dev.cuh"

namespace ckpt {

constexpr int kMaxStages = 8;
constexpr int kTileLog = 10;    // stage-0 tile: 1024 virtual leaf slots
constexpr int kGroupLog = 10;   // upper stages: 1024 positions per group
constexpr int kLeafThreads = 256;
#ifndef CKPT_TREE_THREADS
#define CKPT_TREE_THREADS 256   // tree-kernel CTA size (experiments: 128 lets a tree CTA sit beside K1's)
#endif
constexpr int kTreeThreads = CKPT_TREE_THREADS;
constexpr int kTilesPerBlock = 1024;  // compaction: tiles per reduce/offsets CTA
constexpr unsigned long long kResPending = 1ull << 63;   // res_of: value not final after K1b
constexpr int kModeTree = 0, kModeList = 1, kModeBasic = 2;   // = CKPT_MODE_* (include/ckpt.h)
#ifdef CKPT_K1_STAGES
constexpr int kLeafStages3d = CKPT_K1_STAGES;   // experiment builds
#else
constexpr int kLeafStages3d = 3;      // K1 TMA stages of 32 KB (+ 4 KB digests) when C % 128 == 0
#endif

struct Totals {                      // per-checkpoint device counters (zeroed each call)
  unsigned long long nF, nS, data_bytes, meta_bytes;
  unsigned long long n_first, n_spatial, n_temporal, p2_inserts;
  unsigned long long collisions, n_cand;
  unsigned long long p3_inserts;     // CKPT_VARIANT_SHIFT_INSERT: new potential shifted regions (R24)
  unsigned long long full_kind;      // 0, or the difference is stored in full: 1 = full first
                                     // checkpoint, 2 = switched (gather kernel, R22 / R23)
  unsigned long long n_nonfixed;     // non-FIXED leaves (K1/K1t, counted only for the switch)
  uint32_t wl_count[kMaxStages];
  uint32_t tree_next[3];             // work-stealing cursors of the phase-2 / phase-3 / phase-3a kernels
  uint32_t gather_next;              // work-stealing cursor of the gather kernel
  uint32_t k1_next;                  // K1 tile cursor (tiles handed out beyond the first wave)
  uint32_t defer_count;              // 256-chunk leaf tiles whose inserts K1 left to K1b
  uint32_t insert_next;              // work-stealing cursor of K1b
  uint32_t spare;
  uint32_t done;                     // host copy: epoch of the last completed call (spin-wait target)
};

struct InsertParams {
  Geo g;
  const Digest* prev;
  const uint32_t* cand;
  uint64_t nwords;
  Slot* tab;
  uint64_t cap;
  unsigned long long* res_of;    // per candidate: final record value, or kResPending | slot
  Totals* tot;
  uint32_t* defer;               // (tile << 3 | round) entries left for K1b
  // tree work discovery (K1/K1t mark, K1b block 0 compacts)
  uint32_t* dbits;               // dirty bit per stage-0 tree tile
  uint32_t* tcc;                 // candidate leaves per stage-0 tree tile (full-tile test)
  uint64_t n_tiles;
  uint32_t* wl0;                 // out: dirty stage-0 tiles
  int S;
  int gsz[kMaxStages];
  uint32_t* dcnt[kMaxStages];    // out: s >= 1, FULL children per group (the climb target)
  ulonglong4* trace;             // diagnostics (CKPT_TRACE)
  uint32_t* trace_n;
  int mode;                      // CKPT_MODE_*: Basic accumulates the gather's prefix inputs in K1
  unsigned long long* blocksum;  // Basic: per 1024 tree tiles (#changed, 0, changed bytes)
  unsigned long long* gsum;      // Basic: per 32 tree tiles, the same
  int sw_permille;               // full-change switch threshold (R23), -1 = off
};

struct LeafParams {
  Geo g;
  const uint8_t* buf;
  uint64_t n_main;       // chunks handled by the TMA pipeline (multiple of 256)
  uint64_t tail_begin;   // first chunk of the direct-load tail pass
  int segs;              // 128-B rows per chunk (C >= 128) or 1
  int mode3d;            // 1: C % 128 == 0 (3-D map: row r of 256 chunks); 2: other C > 128 (2-D map of
                         // chunk rows, 128-B boxes, zero-filled past C); 0: C < 128 (2-D rows)
  uint32_t stage_bytes;  // TMA bytes per pipeline stage
  int nst;               // pipeline stages
  uint32_t tpg;          // tiles per cursor grab (>= 1; more at small C, see the K1 producer)
  Digest* prev;          // persistent leaf digests Tree(leaf), 16 n bytes
  Digest* cdig;          // pipelined calls: this call's candidate digests (also written here), or null
  uint32_t* cand;        // candidate (non-FIXED) bit per chunk
  InsertParams ins;      // record insert state (K1's producer warp marks/defers, K1b inserts)
};

struct LevelIO {               // per-position arrays at one height (stage boundary)
  Digest* dig;                 // digest of FIRST (phase 2) or SHIFT (phase 3) positions
  unsigned long long* src;     // packed (ckpt<<32|node) source of SHIFT positions
};

struct StageParams {
  int Lin;                     // input height
  int gsz;                     // log2 positions per group (levels processed)
  LevelIO in;                  // s >= 1: input arrays (written by stage s-1)
  Digest* tdig;                // per group: digests of internal nodes (2^gsz entries)
  unsigned long long* tsrc;    // per group: sources of SHIFT nodes (2 * 2^gsz entries)
  uint32_t* arr2;              // s >= 1: arrivals of dirty children, phase 2
  uint32_t* arr3;              //                                     phase 3
  uint32_t* arr4;              //                                     phase 3a (R24 inserts)
  const uint32_t* dcnt;        // s >= 1: full children per group (K1b)
  uint32_t* gm2;               // s >= 1: per group, 32 words: FIRST children (bit-reversed), phase 2
  uint32_t* gm3;               // s >= 1: per group, 64 words: FIRST / SHIFT children, phase 3
  uint32_t* gm4;               // s >= 1: per group, 32 words: all-SHIFT children, phase 3a
};

struct TreeParams {
  Geo g;
  int S;
  uint64_t n_tiles;
  const uint32_t* wl0;         // dirty stage-0 tiles (K1b)
  const uint8_t* buf;          // checkpoint buffer (phase 3 prefetches FIRST bytes into L2)
  const uint32_t* tcc;         // candidate leaves per stage-0 tile (K1/K1t)
  const uint32_t* cand;
  const unsigned long long* res_of;   // per candidate (K1b): final value or kResPending | slot
  const Digest* prev;
  Slot* tab;
  uint64_t cap;
  uint4* scratch;              // per tile: up to 2^t0 region records {node, src_node, src_ckpt, kind}
  uint4* tilecnt;              // per tile: {nF, nS, data_bytes, epoch}
  uint32_t* lmask;             // per tile: resolved leaf masks (phase 2 -> phase 3)
  unsigned long long* blocksum;  // per 1024 tiles: (#FIRST, #SHIFT, FIRST bytes), zeroed per call
  unsigned long long* gsum;      // per 32 tiles: the same sums
  Totals* tot;
  int dbg;                     // diagnostics only (CKPT_DBG bits; 0 in production)
  int list;                    // CKPT_MODE_LIST: no compaction, every FIRST/SHIFT leaf is an entry
  int shift_insert;            // CKPT_VARIANT_SHIFT_INSERT (R24): a lookup finding its own entry is a miss
  int sw_permille;             // full-change switch threshold (R23), -1 = off
  ulonglong4* trace;           // optional diagnostics (CKPT_TRACE): {t_start, t_end, stage|G, phase}
  uint32_t* trace_n;
  StageParams st[kMaxStages];
};

struct CompactParams {
  Geo g;
  uint64_t n_tiles;
  const uint4* tilecnt;
  const uint4* scratch;
  const unsigned long long* blocksum;  // per 1024 tiles: (#FIRST, #SHIFT, FIRST bytes) (phase 3)
  const unsigned long long* gsum;      // per 32 tiles: the same sums (phase 3)
  const uint32_t* wl0;           // dirty stage-0 tiles
  Totals* tot;
  const uint32_t* lmask;         // per tile (phase 2): FIRST-chunk mask at kLmFirstChunks
  uint8_t* out;                  // diff destination (device arena)
  const uint8_t* buf;            // checkpoint buffer (source of first-occurrence data)
  ulonglong4* trace;             // diagnostics (CKPT_TRACE)
  uint32_t* trace_n;
  Totals* tot_host;              // mapped pinned host copy of the final totals (no D2H op)
  int dbg;                       // diagnostics only (CKPT_DBG bits; 0 in production)
  uint4* ctr_next;               // the next call's counter block, zeroed by the gather kernel
  uint64_t ctr_next_words;
  int mode;                      // CKPT_MODE_*: header flags; Basic writes the bitmap instead of entries
  int flags;                     // header flags of a Tree / List / Basic difference (= mode, or 4, R24)
  const uint32_t* cand;          // Basic: the changed-chunk bitmap (K1)
  uint64_t nwords;               // Basic: its u32 words
  const uint32_t* tcc;           // Basic: changed chunks per tree tile (K1)
  uint32_t parts;                // warps per dirty tile (gather_parts)
  int sw_permille;               // full-change switch threshold (R23), -1 = off
  int full_first;                // checkpoint 0 of a full-first lineage (R22): stored in full
};

// R23: checkpoint k >= 1 is stored in full, with no record operation, when at least
// sw_permille / 1000 of its leaves are not FIXED. K1/K1t count them; every later kernel of
// the call reads the final count after its pdl_wait() and takes the same decision.
__device__ __forceinline__ bool switched_full(const Totals* tot, int sw_permille, const Geo& g) {
  if (sw_permille < 0 || g.k == 0) return false;
  const unsigned long long c = *reinterpret_cast<const volatile unsigned long long*>(&tot->n_nonfixed);
  return 1000ull * c >= (unsigned long long)sw_permille * g.n;
}

// Per stage-0 tile, written by phase 2: the resolved leaf masks for phase 3 (F0 S0 X0 F1 S1
// leaf1, bit-reversed, 32 words each) and the tile's FIRST chunks in chunk order (32
// words, bit i = chunk lo + i) for the gather kernel.
constexpr int kLmWords = 224;
constexpr int kLmFirstChunks = 192;

// CKPT_TRACE diagnostics buffer: kTraceLanes regions of kTraceLaneCap 32-B records.
constexpr uint32_t kTraceLanes = 64, kTraceLaneCap = 16384;

// Kernel launches issued by this thread (every launch site calls note_launch once per
// kernel it enqueues); the engine adds the per-call difference to the handle's counter.
inline thread_local uint64_t g_kernel_launches = 0;
inline void note_launch() { ++g_kernel_launches; }

// Launch with programmatic stream serialization (PDL): the kernel may be scheduled while
// its predecessor drains; it must call pdl_wait() before touching the predecessor's output.
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), unsigned grid, unsigned block, size_t smem, cudaStream_t st,
                              Args... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(block);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  note_launch();
  return cudaLaunchKernelEx(&cfg, kernel, args...);
}

// ---- launchers (return cudaGetLastError())
cudaError_t leaf_setup_attributes();
cudaError_t tree_setup_attributes();
cudaError_t preload_leaf();
cudaError_t preload_tree();
cudaError_t preload_compact();
cudaError_t preload_restore();
cudaError_t launch_leaf(const CUtensorMap* tmap, const LeafParams& p, int num_sms, cudaStream_t st);
int leaf_ctas_per_sm(int mode3d, uint32_t C);   // resident K1 CTAs per SM for chunk size C
cudaError_t launch_leaf_tail(const LeafParams& p, cudaStream_t st);
// pdl: launched with programmatic stream serialization. Only after K1 / K1t, which never
// trigger their dependents early: after a gather (the chain stream of pipelined calls) an
// early launch would let the next call's chain start, and its gather zero the previous
// call's counters (pre-wait), while that call's phase 3 and gather still run.
cudaError_t launch_insert(const InsertParams& p, int num_sms, cudaStream_t st, bool pdl);
cudaError_t launch_tree(const TreeParams& p, int phase, int num_sms, cudaStream_t st);
cudaError_t launch_compact(const CompactParams& p, int num_sms, cudaStream_t st);
uint32_t gather_parts(uint64_t n_tiles, uint32_t C, int num_sms);
cudaError_t launch_rehash(const Slot* old_tab, uint64_t old_cap, Slot* new_tab, uint64_t new_cap, cudaStream_t st);
cudaError_t leaf_smem_config(const LeafParams& p, size_t* smem_bytes);

// ---- restore (k_restore.cu)
struct RestoreDiff {           // one diff of the chain, as the restore kernels see it (cached plan)
  uint32_t id;                 // its checkpoint id (a SHIFT source must be <= id)
  uint32_t composite;          // R25: a SHIFT source may lie outside its diff's FIRST regions
  const uint8_t* base;         // diff bytes (device)
  uint64_t nF, nS, meta_bytes, data_bytes;
  unsigned long long* Flo;     // per FIRST region: first chunk (sorted)
  unsigned long long* Foff;    // per FIRST region: offset in the data section
  unsigned long long* Slo;     // per SHIFT region: first chunk
  unsigned long long* Soff;    // per SHIFT region: exclusive scan of byte lengths; [nS] = total
  unsigned long long* Ssrc;    // per SHIFT region: device address of its source bytes
  unsigned long long shift_bytes;  // = Soff[nS]
  unsigned long long* Fseg;    // per 2-KB segment of the FIRST stream: region of its first byte (+1 entry)
  unsigned long long* Sseg;     // same for the SHIFT stream
  uint32_t* Cch;               // claim list: per C-byte step of the FIRST then SHIFT stream, its
  unsigned long long* Csrc;    //   chunk and the device address of its bytes (chunk-major restore)
};
cudaError_t restore_prepare_first(const Geo& g, RestoreDiff& d, unsigned long long* tmp_len, void* scan_tmp,
                                  size_t scan_tmp_bytes, cudaStream_t st);
cudaError_t restore_prepare_shift(const Geo& g, RestoreDiff& d, const RestoreDiff* chain_dev, unsigned long long* tmp_len,
                                  int* err, void* scan_tmp, size_t scan_tmp_bytes, cudaStream_t st);
cudaError_t restore_prepare_basic(const Geo& g, RestoreDiff& d, uint64_t nwords, unsigned long long* tmp_cnt,
                                  void* scan_tmp, size_t scan_tmp_bytes, cudaStream_t st);
cudaError_t restore_segmaps(RestoreDiff& d, cudaStream_t st);
cudaError_t device_compare(const void* a, const void* b, uint64_t bytes, int* diff, int num_sms, cudaStream_t st);
uint64_t restore_segments(uint64_t bytes);
cudaError_t restore_claimlist(const Geo& g, const RestoreDiff& d, int num_sms, cudaStream_t st);
cudaError_t restore_resolve(const Geo& g, const RestoreDiff& d, const RestoreDiff* chain_dev, int passes, int* err,
                            int num_sms, cudaStream_t st);
cudaError_t restore_claim(const Geo& g, const RestoreDiff& d, unsigned long long* owner, bool bitmap, int num_sms,
                          cudaStream_t st);
cudaError_t restore_copy(const Geo& g, const unsigned long long* owner, uint8_t* out, int num_sms, cudaStream_t st);
size_t scan_tmp_bytes_for(uint64_t count);
cudaError_t scan_u64_exclusive(const unsigned long long* in, unsigned long long* out, uint64_t count, void* tmp,
                               size_t tmp_bytes, cudaStream_t st);

}  // namespace ckpt
