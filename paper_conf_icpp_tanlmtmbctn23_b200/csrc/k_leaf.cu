// k_leaf.cu — leaf pass of Algorithm 1 on sm_100a.
//
// K1  (leaf_hash_kernel): "successive threads compute hashes for successive chunks"
//     (P:174). Persistent CTAs (2 per SM) stream 256-chunk tiles through a TMA +
//     mbarrier pipeline into 128B-swizzled shared memory, so thread t reads chunk t's
//     16-byte blocks conflict-free while the global reads stay fully coalesced. Each
//     thread runs MurmurHash3_x64_128 over its chunk (Alg.1 l.2), compares with the
//     persistent digest Tree(leaf) of checkpoint k-1 (l.3, R5; bulk-copied into smem in
//     the same pipeline stage), writes one candidate bit per chunk (warp ballot) and
//     stores the new digest of non-FIXED chunks (l.21). No atomics: the insert (which
//     has long dependent latency) runs in K1b so the streaming loop never waits on it.
// K1t (leaf_tail_kernel): the same for the ragged tail (< 256 chunks + a partial last
//     chunk hashed at its true length, R4) with direct loads.
// K1b (insert_kernel): Map.insert(digest, (leaf, chkptID)) for every candidate
//     (Alg.1 l.6-19) with the R6 tie-break (atomicMin over ckpt<<32|node), one warp per
//     round of 32 candidates of a 256-chunk tile, warp-level de-duplication of equal
//     digests (__match_any) so a hot key (e.g. all-zero chunks) costs one atomic per warp.
#include "kernels.h"
#include "tma.cuh"

namespace ckpt {

// ------------------------------------------------------------------ shared epilogue
// Fixed test (Alg.1 l.3-4) and digest update (l.21) for chunk c with digest d.
__device__ __forceinline__ bool leaf_is_candidate(const Geo& g, const Digest& d, const Digest& prevd) {
  return !(g.k > 0 && d == prevd);
}

// ------------------------------------------------------------------ record insert
constexpr uint32_t kDenseTile = 64;
#ifndef CKPT_K1B_DEDUP_ALL
#define CKPT_K1B_DEDUP_ALL 0   // 1: warp-level key de-duplication at every checkpoint (A/B)
#endif
#ifndef CKPT_K1B_BPS
#define CKPT_K1B_BPS 4   // K1b launch bound: 4 resident blocks per SM (<= 64 registers)
#endif   // candidates per 256-chunk tile above which inserts read first
// Map.insert(digest, (leaf, chkptID)) for the candidates of one 256-chunk leaf tile
// (Alg.1 l.6-19), by one warp: lane i < 8 holds candidate word i. The candidates are
// spread evenly over the lanes (prefix over popcounts, __fns), identical digests within a
// round are collapsed (__match_any) so a hot key costs one record operation per warp, the
// R6 tie-break is atomicMin over (ckpt << 32 | node).
__device__ __forceinline__ void insert_tile(const InsertParams& p, uint32_t tile, uint32_t word, uint32_t* s_word,
                                            uint32_t* s_excl, unsigned long long& ncand, int only_round = -1) {
  const int lane = threadIdx.x & 31;
  const uint32_t cnt = __popc(word);
  uint32_t incl = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  if (total == 0) return;
  s_word[lane] = word;
  s_excl[lane] = incl - cnt;
  __syncwarp();
  const uint64_t c0 = (uint64_t)tile * 256;
  const uint64_t pol = policy_evict_last();
  const uint32_t b_begin = only_round < 0 ? 0u : 32u * (uint32_t)only_round;
  const uint32_t b_end = only_round < 0 ? total : (b_begin + 32 < total ? b_begin + 32 : total);
  for (uint32_t base = b_begin; base < b_end; base += 32) {
    const uint32_t j = base + lane;
    const bool has = j < b_end;
    const unsigned active = __ballot_sync(0xffffffffu, has);
    if (has) {
      int lo = 0;   // source word: last w < 8 with excl[w] <= j
#pragma unroll
      for (int step = 4; step > 0; step >>= 1)
        if (lo + step < 8 && s_excl[lo + step] <= j) lo += step;
      const uint32_t b = __fns(s_word[lo], 0, (int)(j - s_excl[lo]) + 1);
      const uint64_t c = c0 + (uint64_t)lo * 32 + b;
      const ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2*>(p.prev) + c);
      const Digest d{v.x, v.y};
      const uint32_t node = node_of_chunk(p.g, c);
      // Warp-level de-duplication of equal digests (one record operation per distinct key)
      // at checkpoint 0, where hot keys (e.g. all-zero chunks) would otherwise serialise
      // thousands of atomics on one slot. Later checkpoints skip it: every lane inserts its
      // own candidate; equal keys then meet in the table, where the R6 atomicMin gives the
      // same result, and older keys cost one read.
      const bool dedup = CKPT_K1B_DEDUP_ALL || p.g.k == 0;
      const unsigned grp = dedup ? (__match_any_sync(active, d.lo) & __match_any_sync(active, d.hi)) : (1u << lane);
      const int leader = __ffs(grp) - 1;
      // minimum node id of the group (every active lane shuffles). Measured on config 4: a
      // vote that skips this loop for rounds of distinct digests made K1b 14 % slower, and
      // __reduce_min_sync over the (non-uniform) group masks 30 % slower.
      uint32_t minnode = node;
      for (unsigned a = dedup ? active : 0u; a; a &= a - 1) {
        const int sl = __ffs(a) - 1;
        const uint32_t vv = __shfl_sync(active, node, sl);
        if ((grp >> sl) & 1u) minnode = vv < minnode ? vv : minnode;
      }
      unsigned long long res = 0;
      if (lane == leader) {
        bool claimed;
        unsigned long long seen;
        // Sparse candidates after checkpoint 0 are mostly new keys (CAS first: one round trip).
        // Checkpoint 0 and dense tiles (moved or repeated content) mostly hit existing keys:
        // read key + value first, no atomic when the entry is older (one round trip).
        const uint32_t slot = (uint32_t)table_insert_min(p.tab, p.cap, d, pack_entry(p.g.k, minnode), &claimed,
                                                         p.g.k > 0 && total < kDenseTile, &seen);
        // an entry of an earlier checkpoint never changes again (R6): the leaf is resolved
        // here (SHIFT to it); otherwise phase 2 reads the final value from the slot
        res = seen < ((unsigned long long)p.g.k << 32) ? seen : (kResPending | slot);
      }
      res = __shfl_sync(active, res, leader);
      st_evict_last_u64(p.res_of + c, res, pol);
    }
  }
  ncand += b_end - b_begin;
  __syncwarp();
}

// Mark the stage-0 tree tile(s) holding 256-chunk leaf tile `tile` dirty (fire-and-forget;
// a tree tile marked without candidates is processed as all-FIXED, which is harmless).
// bits [a, b) of a 256-bit word array
__device__ __forceinline__ uint32_t popc_range(const uint32_t* w, uint32_t a, uint32_t b) {
  uint32_t n = 0;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const uint32_t lo = 32u * i, hi = lo + 32u;
    const uint32_t x = a > lo ? a : lo, y = b < hi ? b : hi;
    if (x < y) n += __popc(w[i] & (((y - lo) == 32 ? 0xFFFFFFFFu : ((1u << (y - lo)) - 1u)) & ~((1u << (x - lo)) - 1u)));
  }
  return n;
}

// A 256-chunk leaf tile with candidates: mark the stage-0 tree tile(s) it overlaps dirty and
// add its candidates to their counts (a leaf tile can straddle two tree tiles where the
// leaves sit at height 1, R3).
__device__ __forceinline__ void mark_tree_dirty(const InsertParams& p, uint32_t tile, const uint32_t* w) {
  const uint64_t c0 = (uint64_t)tile * 256;
  uint64_t c1 = c0 + 255;
  if (c1 >= p.g.n) c1 = p.g.n - 1;
  const uint64_t t0 = vpos_of_chunk(p.g, c0) >> p.g.t0, t1 = vpos_of_chunk(p.g, c1) >> p.g.t0;
  for (uint64_t t = t0; t <= t1; ++t) {
    atomicOr(p.dbits + (t >> 5), 1u << (t & 31));
    uint64_t lo, hi;
    chunk_range(p.g, p.g.t0, t, lo, hi);
    const uint64_t a = lo > c0 ? lo : c0, b = hi < c1 + 1 ? hi : c1 + 1;
    const uint32_t cnt = a < b ? popc_range(w, (uint32_t)(a - c0), (uint32_t)(b - c0)) : 0u;
    if (cnt) {
      atomicAdd(p.tcc + t, cnt);
      if (p.mode == kModeBasic) {
        // Basic: the gather's prefix inputs are the changed chunks and their bytes (the
        // buffer's last chunk may be short)
        unsigned long long bytes = (unsigned long long)cnt * p.g.C;
        const uint64_t last = p.g.n - 1;
        if (a <= last && last < b && ((w[(last - c0) >> 5] >> ((last - c0) & 31)) & 1u))
          bytes -= (unsigned long long)p.g.n * p.g.C - p.g.B;
        atomicAdd(p.blocksum + 3 * (t / kTilesPerBlock), (unsigned long long)cnt);
        atomicAdd(p.blocksum + 3 * (t / kTilesPerBlock) + 2, bytes);
        atomicAdd(p.gsum + 3 * (t / 32), (unsigned long long)cnt);
        atomicAdd(p.gsum + 3 * (t / 32) + 2, bytes);
      }
    }
  }
}

// Defer a tile's inserts to K1b as one entry (tile << 3 | round) per 32 candidates, so
// the rounds of a dense tile run on different warps.
__device__ __forceinline__ void defer_tile(const InsertParams& p, uint32_t tile, uint32_t ncand_tile) {
  const uint32_t rounds = (ncand_tile + 31) / 32;
  if (p.sw_permille >= 0) atomicAdd(&p.tot->n_nonfixed, (unsigned long long)ncand_tile);   // R23
  const uint32_t i = atomicAdd(&p.tot->defer_count, rounds);
  for (uint32_t r = 0; r < rounds; ++r) p.defer[i + r] = (tile << 3) | r;
}

// ------------------------------------------------------------------ K1
// 8 hashing (consumer) warps + 1 producer warp. The producer streams the stages with TMA
// (full barriers, complete_tx) and re-fills a stage as soon as all 8 consumer warps have
// released it (empty barriers, one arrive per warp): fast warps never wait for slow ones
// at a CTA barrier, they run ahead into the next filled stage. Tiles are handed out
// dynamically (first wave = blockIdx, then a global cursor, fetched one tile ahead): the
// SMs do not stream at the same rate (measured: with a static tile stride the first CTA
// finished 20 % before the last), so a static split leaves the tail waiting on the slowest.
// At the end of a 256-chunk tile each consumer warp leaves its candidate ballot word in
// the stage's slot; the producer, on the stage's release, marks the tree tile(s) dirty and
// defers the tile's inserts to K1b, so that bookkeeping is off the hashing warps' path.
constexpr int kK1Threads = kLeafThreads + 32;
constexpr int kMaxStagesK1 = 8;
#ifndef CKPT_K1_CTAS
#define CKPT_K1_CTAS 2   // resident K1 CTAs per SM when C % 128 == 0 (3 stages of 36 KB each)
#endif
#ifndef CKPT_K1_PDL
#define CKPT_K1_PDL 1           // K1 launched with programmatic stream serialization (see pdl_wait)
#endif
#ifndef CKPT_K1_CTAS_C32
#define CKPT_K1_CTAS_C32 4      // C = 32: 4 CTAs per SM with 48 KB of stages each (issue-bound: one
#endif                          // more CTA of hashing warps, 274 -> 255 us per GiB; neutral at C = 64)
#ifndef CKPT_K1_CTAS_SMALLC
#define CKPT_K1_CTAS_SMALLC 3   // C < 128: a tile is only 256 C bytes and one producer thread per
#endif                          // CTA bounds the rate (C = 32: 2 CTAs 320 us, 3 CTAs 288 us / GiB)
constexpr uint32_t kNoTile = 0xFFFFFFFFu;

struct K1Shared {
  uint64_t full[kMaxStagesK1];
  uint64_t empty[kMaxStagesK1];
  uint32_t tile[kMaxStagesK1];       // tile streamed into the stage (kNoTile: stop)
  uint32_t tile_end[kMaxStagesK1];   // 1 if the stage holds the tile's last segment
  uint32_t words[kMaxStagesK1][8];   // candidate ballot words of the tile ending in the stage
};

__device__ __forceinline__ void mbar_arrive(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}

// MODE3D: 1 = C % 128 == 0 (3-D map: 128-B row r of 256 chunks per stage); 2 = C > 128 not a
// multiple of 128 (2-D map of C-byte rows, the same 128-B boxes; the last one runs past the
// chunk's end, which TMA fills with zeros without reading, and hashes only its C mod 128 bytes);
// 0 = C < 128 (whole chunks in 2-D rows).
// UNITS: the 16-byte blocks of a thread's chunk per stage as a compile-time constant (8 for
// C >= 128; C / 16 for the small chunk sizes C = 32 and 64), 0 = read from p at run time.
// With it known, each thread's swizzled shared-memory offsets are computed once, outside
// the stage loop (at C = 32 the per-stage address arithmetic and the generic unit loop were
// as many instructions as a block of the hash, and K1 is issue-bound there).
template <int MODE3D, int UNITS>
__global__ void __launch_bounds__(kK1Threads, MODE3D ? CKPT_K1_CTAS : (UNITS == 2 ? CKPT_K1_CTAS_C32 : CKPT_K1_CTAS_SMALLC)) leaf_hash_kernel(const __grid_constant__ CUtensorMap tmap, LeafParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-B alignment for the 128B swizzle atom, kept as a shared-space pointer (LDS, not LD)
  const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
  uint8_t* const data = smem_raw + pad;                                    // nst * stage_bytes
  const int nst = p.nst;
  const uint32_t stage_bytes = p.stage_bytes;
  Digest* const prevbuf = reinterpret_cast<Digest*>(data + nst * stage_bytes);   // nst * 256 digests
  K1Shared& sh = *reinterpret_cast<K1Shared*>(prevbuf + nst * kLeafThreads);

  const unsigned long long bt0 = p.ins.trace ? gtime_ns() : 0;
  const int tid = threadIdx.x;
  const uint32_t n_tiles = (uint32_t)(p.n_main / kLeafThreads);
  const int segs = p.segs;
  const bool use_prev = p.g.k > 0;

  if (tid == 0) {
    prefetch_tmap(&tmap);
    for (int s = 0; s < nst; ++s) {
      mbar_init(&sh.full[s], 1);
      mbar_init(&sh.empty[s], kLeafThreads / 32);
    }
    fence_mbar_init();
  }
  __syncthreads();
  // K1 is launched with programmatic stream serialization: its CTAs may be set up while the
  // previous call's gather kernel drains (that call has already returned on its statistics);
  // nothing of the previous call's memory is touched before this wait
  pdl_wait();

  if (tid >= kLeafThreads) {
    // ---------------- producer warp (lane 0)
    if (tid != kLeafThreads) return;
    const uint64_t pol_stream = policy_evict_first();
    uint32_t* cursor = &p.ins.tot->k1_next;
    // the tile epilogue of the step last consumed from stage s: dirty marks + deferral
    auto epilogue = [&](int s) {
      if (!sh.tile_end[s]) return;
      const uint32_t tile = sh.tile[s];
      uint32_t w[8], any = 0, pc = 0;
#pragma unroll
      for (int q = 0; q < 8; ++q) { w[q] = sh.words[s][q]; any |= w[q]; pc += __popc(w[q]); }
      if (any) {
        mark_tree_dirty(p.ins, tile, w);
        if (p.ins.mode != kModeBasic) defer_tile(p.ins, tile, pc);   // Basic keeps no record
      }
    };
    // tiles are handed out in groups of tpg consecutive tiles (one cursor atomic per group:
    // at small C a tile is only 256 C bytes, and one atomic per tile on one address
    // throttled the producers)
    const uint32_t tpg = p.tpg;
    uint32_t grp = blockIdx.x, ing = 0;
    uint32_t tile = grp * tpg, seg = 0, i = 0;
    uint32_t nxt = tile < n_tiles ? gridDim.x + atomicAdd(cursor, 1u) : kNoTile;   // one group ahead
    for (;; ++i) {
      const int s = (int)(i % (uint32_t)nst);
      if (i >= (uint32_t)nst) {
        mbar_wait(&sh.empty[s], ((i / nst) - 1) & 1u);   // all consumer warps released step i - nst
        epilogue(s);
      }
      if (tile >= n_tiles) {   // stop marker: wakes the consumers without data
        sh.tile[s] = kNoTile;
        sh.tile_end[s] = 0;
        mbar_arrive(&sh.full[s]);
        break;
      }
      const bool with_prev = use_prev && (int)seg == segs - 1;
      sh.tile[s] = tile;
      sh.tile_end[s] = (int)seg == segs - 1;
      mbar_arrive_expect_tx(&sh.full[s], stage_bytes + (with_prev ? kLeafThreads * 16u : 0u));
      if (MODE3D == 1)
        tma_load_3d(data + (size_t)s * stage_bytes, &tmap, &sh.full[s], 0, (int)seg, (int)(tile * kLeafThreads), pol_stream);
      else if (MODE3D == 2)   // box (128 B, 256 chunks) at byte seg * 128 of each chunk row; past C: zero fill
        tma_load_2d(data + (size_t)s * stage_bytes, &tmap, &sh.full[s], (int)(seg * 128), (int)(tile * kLeafThreads),
                    pol_stream);
      else
        tma_load_2d(data + (size_t)s * stage_bytes, &tmap, &sh.full[s], 0, (int)(tile * (stage_bytes / 128)), pol_stream);
      if (with_prev)
        bulk_load(prevbuf + s * kLeafThreads, p.prev + (uint64_t)tile * kLeafThreads, kLeafThreads * 16u, &sh.full[s],
                  pol_stream);
      if ((int)++seg == segs) {
        seg = 0;
        if (++ing < tpg && tile + 1 < n_tiles) {
          ++tile;
        } else {
          ing = 0;
          grp = nxt;
          tile = grp < (n_tiles + tpg - 1) / tpg ? grp * tpg : n_tiles;
          if (tile < n_tiles) nxt = gridDim.x + atomicAdd(cursor, 1u);
        }
      }
    }
    // drain: the real steps after the last one handled above (i - nst + 1 .. i - 1)
    for (uint32_t j = i + 1 > (uint32_t)nst ? i + 1 - nst : 0; j < i; ++j) {
      mbar_wait(&sh.empty[j % nst], (j / nst) & 1u);
      epilogue((int)(j % (uint32_t)nst));
    }
    return;
  }

  // ---------------- consumer (hashing) warps
  const uint64_t pol_keep = policy_evict_last();
  const int units = UNITS ? UNITS : (int)(p.g.C / 16);   // 16-byte blocks of this thread per stage
  const uint32_t ubase = (uint32_t)tid * (uint32_t)units;
  const int lane = tid & 31, wid = tid >> 5;
  constexpr int kOffs = UNITS ? UNITS : 1;
  uint32_t offs[kOffs];   // SWIZZLE_128B offsets of this thread's units within a stage
#pragma unroll
  for (int j = 0; j < kOffs; ++j) {
    const uint32_t u = ubase + j, row = u >> 3;
    offs[j] = (row << 7) | ((((u & 7) ^ (row & 7))) << 4);
  }
  uint64_t h1 = 0, h2 = 0;
  int st = 0, seg = 0;
  uint32_t phase = 0;
  for (;;) {
    mbar_wait(&sh.full[st], phase);
    const uint32_t tile = sh.tile[st];
    if (tile == kNoTile) break;
    if (!MODE3D || seg == 0) { h1 = 0; h2 = 0; }   // seed 0 (R1); C < 128: one stage per chunk
    const uint8_t* sd = data + (size_t)st * stage_bytes;
    if (UNITS) {
      // MODE3D 2: the chunk's last segment holds (C mod 128) / 16 units
      const int nu = (MODE3D == 2 && seg == segs - 1) ? (int)((p.g.C & 127u) >> 4) : kOffs;
#pragma unroll
      for (int j = 0; j < kOffs; ++j) {
        if (MODE3D == 2 && j >= nu) break;
        const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(sd + offs[j]);
#ifdef CKPT_K1_NOHASH   // timing experiment only: data movement without the hash
        h1 ^= v.x; h2 ^= v.y;
#else
        mm::block(h1, h2, v.x, v.y);
#endif
      }
    } else {
#pragma unroll 8
      for (int j = 0; j < units; ++j) {
        const uint32_t u = ubase + j;
        const uint32_t row = u >> 3;
        const uint32_t off = (row << 7) | ((((u & 7) ^ (row & 7))) << 4);   // SWIZZLE_128B
        const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(sd + off);
#ifdef CKPT_K1_NOHASH
        h1 ^= v.x; h2 ^= v.y;
#else
        mm::block(h1, h2, v.x, v.y);
#endif
      }
    }
    if (!MODE3D || seg == segs - 1) {
      const Digest d = mm::finish(h1, h2, p.g.C);
      const uint64_t c = (uint64_t)tile * kLeafThreads + tid;
      Digest pd{0, 0};
      if (use_prev) pd = prevbuf[st * kLeafThreads + tid];
      const bool cand = leaf_is_candidate(p.g, d, pd);
      const unsigned mask = __ballot_sync(0xffffffffu, cand);
      if (lane == 0) {
        st_evict_last_u32(p.cand + (c >> 5), mask, pol_keep);
        sh.words[st][wid] = mask;
      }
      if (cand) {
        // (raising the L2 priority of the candidate chunk's own lines for the gather kernel
        // was measured neutral on configs 2 and 4 and is not done)
        st_evict_last_v2(p.prev + c, d.lo, d.hi, pol_keep);   // K1b / the tree kernels re-read it
        if (p.cdig) st_evict_last_v2(p.cdig + c, d.lo, d.hi, pol_keep);   // pipelined: the chain reads this copy
      }
    }
    __syncwarp();
    if (lane == 0) mbar_arrive(&sh.empty[st]);   // this warp is done with stage st
    if (++st == nst) { st = 0; phase ^= 1u; }
    if (++seg == segs) seg = 0;
  }
  trace_block(p.ins.trace, p.ins.trace_n, bt0, bt0, 0);
}

// ------------------------------------------------------------------ K1t
// The ragged tail (direct loads): one block = one 256-chunk tile; its inserts are deferred.
__global__ void __launch_bounds__(256) leaf_tail_kernel(LeafParams p) {
  const uint64_t c = p.tail_begin + (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  const bool valid = c < p.g.n;
  bool cand = false;
  Digest d{0, 0};
  if (valid) {
    const uint64_t off = c * p.g.C;
    uint64_t len = p.g.B - off;
    if (len > p.g.C) len = p.g.C;
    const uint8_t* src = p.buf + off;
    uint64_t h1 = 0, h2 = 0;
    const uint64_t nb = len / 16;
    for (uint64_t b = 0; b < nb; ++b) {
      const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(src + 16 * b);
      mm::block(h1, h2, v.x, v.y);
    }
    const unsigned rem = (unsigned)(len & 15);
    if (rem) {
      uint64_t t1 = 0, t2 = 0;
      const uint8_t* t = src + 16 * nb;
      for (unsigned i = 0; i < rem; ++i) {
        if (i < 8) t1 |= (uint64_t)t[i] << (8 * i);
        else t2 |= (uint64_t)t[i] << (8 * (i - 8));
      }
      mm::tail(h1, h2, t1, t2, rem);
    }
    d = mm::finish(h1, h2, len);
    Digest pd{0, 0};
    if (p.g.k > 0) {
      const ulonglong2 v = reinterpret_cast<const ulonglong2*>(p.prev)[c];
      pd = Digest{v.x, v.y};
    }
    cand = leaf_is_candidate(p.g, d, pd);
  }
  __shared__ uint32_t s_w[8];
  const unsigned mask = __ballot_sync(0xffffffffu, cand);
  if ((threadIdx.x & 31) == 0) {
    s_w[threadIdx.x >> 5] = mask;
    if (c < p.g.n) p.cand[c >> 5] = mask;
  }
  if (cand) {
    reinterpret_cast<ulonglong2*>(p.prev)[c] = make_ulonglong2(d.lo, d.hi);
    if (p.cdig) reinterpret_cast<ulonglong2*>(p.cdig)[c] = make_ulonglong2(d.lo, d.hi);
  }
  const int pc = __syncthreads_count(cand);
  if (pc && threadIdx.x == 0) {
    const uint32_t tile = (uint32_t)((p.tail_begin >> 8) + blockIdx.x);
    mark_tree_dirty(p.ins, tile, s_w);
    if (p.ins.mode != kModeBasic) defer_tile(p.ins, tile, (uint32_t)pc);
  }
}

// ------------------------------------------------------------------ K1b
// Record inserts of every 256-chunk tile with candidates (K1 and K1t defer them here, so
// the streaming loop never waits on an atomic): one warp per (tile, round of 32 candidates).
// Block 0 of K1b turns the dirty-tile bitmap into the tree kernels' work description: the
// compact list of dirty stage-0 tiles (block scan) and, per upper group, the number of
// dirty children (the climb target of the tree kernels).
__device__ void build_tree_work(const InsertParams& p) {
  __shared__ uint32_t s_ws[8], s_carry;
  const unsigned long long tw0 = p.trace ? gtime_ns() : 0;
  const int tid = threadIdx.x, lane = tid & 31, wid = tid >> 5;
  const uint64_t nw = (p.n_tiles + 31) / 32;
  if (tid == 0) s_carry = 0;
  __syncthreads();
  for (uint64_t base = 0; base < nw; base += 256) {
    const uint64_t wi = base + tid;
    uint32_t bits = wi < nw ? __ldcg(p.dbits + wi) : 0u;
    if (wi == nw - 1 && (p.n_tiles & 31)) bits &= (1u << (p.n_tiles & 31)) - 1u;
    const uint32_t pc = __popc(bits);
    uint32_t incl = pc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += v;
    }
    if (lane == 31) s_ws[wid] = incl;
    __syncthreads();
    uint32_t off = s_carry, tot = 0;
    for (int i = 0; i < 8; ++i) {
      if (i < wid) off += s_ws[i];
      tot += s_ws[i];
    }
    off += incl - pc;
    for (uint32_t m = bits; m; m &= m - 1) p.wl0[off++] = (uint32_t)(wi * 32 + (__ffs(m) - 1));
    __syncthreads();
    if (tid == 0) s_carry += tot;
    __syncthreads();
  }
  if (tid == 0) p.tot->wl_count[0] = s_carry;
  const unsigned long long tw1 = p.trace ? gtime_ns() : 0;
  // dirty children per group, stage by stage
  for (int s = 1; s < p.S; ++s) {
    // groups of stage s: children are positions of stage s-1 (tiles for s == 1)
    uint64_t nchild = p.n_tiles;
    for (int t = 1; t < s; ++t) nchild >>= p.gsz[t];
    const uint64_t ngroups = nchild >> p.gsz[s];
    const uint32_t per = 1u << p.gsz[s];
    // FULL children per group, one warp per group: only a full child can have a FIRST or
    // SHIFT root, so only full children climb to their parent in the tree kernels
    for (uint64_t G = wid; G < ngroups; G += blockDim.x >> 5) {
      uint32_t cnt = 0;
      if (s == 1) {
        const uint32_t q = per / 32;   // tiles per lane
        if (q >= 4) {
          // a lane's q consecutive tile counts as 16-byte vectors, up to 8 in flight (one
          // round trip for a 1024-tile group); only tiles with candidates need their size
          const uint64_t T0 = G * per + (uint64_t)lane * q;
          const uint4* src = reinterpret_cast<const uint4*>(p.tcc + T0);
          for (uint32_t b = 0; b < q / 4; b += 8) {
            uint4 v[8];
#pragma unroll
            for (int u = 0; u < 8; ++u) v[u] = b + u < q / 4 ? __ldcg(src + b + u) : make_uint4(0, 0, 0, 0);
#pragma unroll
            for (int u = 0; u < 8; ++u) {
              const uint32_t c4[4] = {v[u].x, v[u].y, v[u].z, v[u].w};
#pragma unroll
              for (int j = 0; j < 4; ++j) {   // branch-free: a tile without candidates never matches
                uint64_t lo, hi;
                chunk_range(p.g, p.g.t0, T0 + 4 * (b + u) + j, lo, hi);
                cnt += (uint64_t)c4[j] == hi - lo;
              }
            }
          }
        } else {
          for (uint64_t T = G * per + lane; T < (G + 1) * per; T += 32) cnt += tile_full(p.g, p.tcc, T);
        }
      } else {
        const uint32_t full = 1u << p.gsz[s - 1];
        for (uint64_t ch = G * per + lane; ch < (G + 1) * per; ch += 32) cnt += __ldcg(p.dcnt[s - 1] + ch) == full;
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) cnt += __shfl_xor_sync(0xffffffffu, cnt, o);
      if (lane == 0) p.dcnt[s][G] = cnt;
    }
    __syncthreads();
  }
  if (p.trace && tid == 0)
    if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 1)) *r = make_ulonglong4(tw0, tw1, gtime_ns(), 12);
}

__global__ void __launch_bounds__(256, CKPT_K1B_BPS) insert_kernel(InsertParams p) {
  const unsigned long long bt0 = p.trace ? gtime_ns() : 0;
  pdl_launch_dependents();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  __shared__ uint32_t s_word[8][32], s_excl[8][32];
  pdl_wait();
  const unsigned long long bt1 = p.trace ? gtime_ns() : 0;
  if (blockIdx.x == 0) {
    build_tree_work(p);
    __syncthreads();
    trace_block(p.trace, p.trace_n, bt0, bt1, 11);
    return;
  }
  unsigned long long tk0 = 0;
  if (p.trace) asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tk0));
  // a switched checkpoint (R23) has no record operation
  const uint32_t count = switched_full(p.tot, p.sw_permille, p.g) ? 0u : *(volatile uint32_t*)&p.tot->defer_count;
  const uint32_t nwarps = (gridDim.x - 1) * (blockDim.x >> 5);
  unsigned long long ncand = 0;
  for (uint32_t w = (blockIdx.x - 1) * (blockDim.x >> 5) + wid; w < count; w += nwarps) {
    unsigned long long t1 = 0, t2 = 0, t3 = 0;
    if (p.trace) asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t1));
    const uint32_t e = p.defer[w];
    const uint32_t tile = e >> 3;
    const uint64_t wi = (uint64_t)tile * 8 + lane;
    const uint32_t word = (lane < 8 && wi < p.nwords) ? __ldcg(p.cand + wi) : 0u;
    if (p.trace) { __syncwarp(); asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t2)); }
    insert_tile(p, tile, word, s_word[wid], s_excl[wid], ncand, (int)(e & 7));
    if (p.trace) {
      asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t3));
      if (lane == 0) {
        if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 1)) *r = make_ulonglong4(tk0, t1, t2, t3);
      }
    }
  }
  if (lane == 0 && ncand) atomicAdd(&p.tot->n_cand, ncand);
  __syncthreads();
  trace_block(p.trace, p.trace_n, bt0, bt1, 1);
}

// ------------------------------------------------------------------ rehash
__global__ void rehash_kernel(const Slot* old_tab, uint64_t old_cap, Slot* new_tab, uint64_t new_cap) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < old_cap; i += (uint64_t)gridDim.x * blockDim.x) {
    const Slot s = old_tab[i];
    if (s.klo == kEmpty && s.khi == kEmpty) continue;
    bool claimed;
    const uint64_t j = table_find_or_claim(new_tab, new_cap, Digest{s.klo, s.khi}, &claimed);
    new_tab[j].val = s.val;
  }
}

// ------------------------------------------------------------------ launchers
int leaf_ctas_per_sm(int mode3d, uint32_t C) {
  return mode3d ? CKPT_K1_CTAS : (C == 32 ? CKPT_K1_CTAS_C32 : CKPT_K1_CTAS_SMALLC);
}

cudaError_t leaf_smem_config(const LeafParams& p, size_t* smem_bytes) {
  *smem_bytes = 1008 + (size_t)p.nst * p.stage_bytes + (size_t)p.nst * kLeafThreads * 16 + sizeof(K1Shared);
  return cudaSuccess;
}

cudaError_t launch_leaf(const CUtensorMap* tmap, const LeafParams& p, int num_sms, cudaStream_t st) {
  if (p.n_main == 0) return cudaSuccess;
  size_t smem;
  leaf_smem_config(p, &smem);
  const uint64_t n_tiles = p.n_main / kLeafThreads;
  uint64_t grid = (uint64_t)num_sms * leaf_ctas_per_sm(p.mode3d, p.g.C);
  const uint64_t groups = (n_tiles + p.tpg - 1) / p.tpg;
  if (grid > groups) grid = groups;
#if CKPT_K1_PDL
  const CUtensorMap tm = *tmap;
  if (p.mode3d == 2) return launch_pdl(leaf_hash_kernel<2, 8>, (unsigned)grid, kK1Threads, smem, st, tm, p);
  if (p.mode3d) return launch_pdl(leaf_hash_kernel<1, 8>, (unsigned)grid, kK1Threads, smem, st, tm, p);
  if (p.g.C == 32) return launch_pdl(leaf_hash_kernel<0, 2>, (unsigned)grid, kK1Threads, smem, st, tm, p);
  if (p.g.C == 64) return launch_pdl(leaf_hash_kernel<0, 4>, (unsigned)grid, kK1Threads, smem, st, tm, p);
  return launch_pdl(leaf_hash_kernel<0, 0>, (unsigned)grid, kK1Threads, smem, st, tm, p);
#else
  if (p.mode3d == 2) leaf_hash_kernel<2, 8><<<(unsigned)grid, kK1Threads, smem, st>>>(*tmap, p);
  else if (p.mode3d) leaf_hash_kernel<1, 8><<<(unsigned)grid, kK1Threads, smem, st>>>(*tmap, p);
  else if (p.g.C == 32) leaf_hash_kernel<0, 2><<<(unsigned)grid, kK1Threads, smem, st>>>(*tmap, p);
  else if (p.g.C == 64) leaf_hash_kernel<0, 4><<<(unsigned)grid, kK1Threads, smem, st>>>(*tmap, p);
  else leaf_hash_kernel<0, 0><<<(unsigned)grid, kK1Threads, smem, st>>>(*tmap, p);
  note_launch();
  return cudaGetLastError();
#endif
}

cudaError_t launch_leaf_tail(const LeafParams& p, cudaStream_t st) {
  if (p.tail_begin >= p.g.n) return cudaSuccess;
  const uint64_t cnt = p.g.n - p.tail_begin;
  leaf_tail_kernel<<<(unsigned)((cnt + 255) / 256), 256, 0, st>>>(p);
  note_launch();
  return cudaGetLastError();
}

static int g_insert_blocks_per_sm = 0;

cudaError_t launch_insert(const InsertParams& p, int num_sms, cudaStream_t st, bool pdl) {
  const uint64_t tiles = (p.nwords + 7) / 8;
  uint64_t blocks = (tiles + 7) / 8 + 1;   // + block 0: tree work description
  if (p.mode == kModeBasic) blocks = 1;    // Basic: no record; only the dirty-tile worklist
  // one resident wave: the deferred work is strided statically over the warps
  const uint64_t wave = (uint64_t)num_sms * (g_insert_blocks_per_sm > 0 ? g_insert_blocks_per_sm : 4);
  if (blocks > wave) blocks = wave;
  if (!blocks) return cudaSuccess;
  if (pdl) return launch_pdl(insert_kernel, (unsigned)blocks, 256, 0, st, p);
  insert_kernel<<<(unsigned)blocks, 256, 0, st>>>(p);
  note_launch();
  return cudaGetLastError();
}

cudaError_t leaf_setup_attributes() {
  // the largest dynamic smem any leaf configuration asks for (C >= 128: 3 x 36 KB; C < 128: <= 96 KB)
  // the largest leaf configuration: kLeafStages3d x (32 KB + 4 KB) when C % 128 == 0, <= 96 KB of stages below
  const int stages = kLeafStages3d * (32768 + 4096) > 98304 + 8 * 4096 ? kLeafStages3d * (32768 + 4096) : 98304 + 8 * 4096;
  const int smem = 1008 + stages + (int)sizeof(K1Shared);
  cudaError_t e = cudaFuncSetAttribute(leaf_hash_kernel<1, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(leaf_hash_kernel<2, 8>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(leaf_hash_kernel<0, 2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(leaf_hash_kernel<0, 4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(leaf_hash_kernel<0, 0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  return e;
}

cudaError_t launch_rehash(const Slot* old_tab, uint64_t old_cap, Slot* new_tab, uint64_t new_cap, cudaStream_t st) {
  uint64_t blocks = (old_cap + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks) {
    rehash_kernel<<<(unsigned)blocks, 256, 0, st>>>(old_tab, old_cap, new_tab, new_cap);
    note_launch();
  }
  return cudaGetLastError();
}


// Load this file's kernels now (CUDA lazy module loading would otherwise stall the first
// launch of each kernel inside the first checkpoint).
cudaError_t preload_leaf() {
  cudaFuncAttributes a;
  cudaError_t e = cudaSuccess;
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, leaf_hash_kernel<0, 2>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, leaf_hash_kernel<0, 4>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, leaf_hash_kernel<0, 0>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, leaf_hash_kernel<1, 8>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, leaf_hash_kernel<2, 8>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, leaf_tail_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, insert_kernel);
  if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_insert_blocks_per_sm, insert_kernel, 256, 0);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, rehash_kernel);
  return e;
}

}  // namespace ckpt
