// k_tree.cu — Merkle level reduction: phase 2 (Alg.1 l.24-32) and phase 3 (l.33-46).
//
// The paper parallelises Algorithm 1 "level-by-level" in two stages: first the
// sub-trees of first-time occurrences, then those of shifted duplicates. Here
// each stage is ONE kernel launch (all of phase 2 finishes before any phase-3 lookup,
// R11, because the phase-3 kernel is launched after the phase-2 kernel on one stream).
//
// Work unit: one WARP per group of up to 1024 positions of one height (a stage-0 tile
// of the virtual leaf level, R3 geometry in dev.cuh, or 1024 roots of the stage below).
// Labels are bitmasks (FIRST, SHIFT, FIXED), one bit per position, 32 positions per
// lane. Each level is kept in BIT-REVERSED position order, so the two children of the
// node at index r sit at indices r and r + N/2 of the level below: a level step is one
// shuffle and an AND (parent FIRST iff both children FIRST; FIXED iff both FIXED, R7;
// "SHIFT pair" iff both SHIFT; otherwise DONE), with no bit compression. Leaf masks enter
// that order once per group through a 32-ballot bit transpose.
//
// Digest work is batched per group instead of per level: pass 1 computes every digest
// the group needs bottom-up from on-chip data (phase 2: FIRST pairs, Alg.1 l.28; phase 3:
// every POTENTIAL shifted pair, l.38 — a superset of the pairs Alg.1 looks up); pass 2
// issues all record operations at once (phase 2: insert, l.29; phase 3: lookup, l.39);
// pass 3 (phase 3) replays the labels with the lookup results and emits the regions.
// Only dirty groups are visited: K1/K1t mark the tree tiles holding a non-FIXED leaf in a
// bitmap, K1b compacts it into a worklist and counts the dirty children of every upper
// group; the warp finishing the LAST dirty child of a group climbs and processes that
// group too, so every stage runs in this launch.
//
// Phase-3 emission ("save roots", R8/R10): a FIRST/SHIFT child of a DONE parent (or the
// FIRST/SHIFT root) becomes a region. Stage 0 records its regions per tile in leaf
// order (FIRST list, then SHIFT list); an upper-stage region starts at a tile boundary
// and is recorded in the tile holding its first leaf, so the per-tile lists in tile
// order are the regions sorted by first chunk (R13) — k_compact.cu relies on it.
//
// PHASE 4 (CKPT_VARIANT_SHIFT_INSERT, reading R24 of P:89) runs between the two: pass 1 as
// phase 3 (the hashes of every POTENTIAL shifted node, i.e. every node whose leaves are all
// SHIFT), pass 2 inserts them (find-or-claim, then atomicMin over ckpt<<32|node: the
// minimum node id wins among equal new hashes, an existing entry is never changed, R6).
// Phase 3 then finds every SHIFT-SHIFT parent; one that finds its own entry is a miss.
#include "kernels.h"
#include "tma.cuh"

namespace ckpt {

namespace {

constexpr int kWarps = kTreeThreads / 32;
#ifndef CKPT_TREE_BPS
#define CKPT_TREE_BPS (512 / CKPT_TREE_THREADS)   // launch bound: 512 threads per SM (<= 128 registers)
#endif
#ifndef CKPT_TREE_KB2
#define CKPT_TREE_KB2 2   // pass-2 record operations per lane in flight (3 and 4 spill: config 4 phase 3 +40-55 %)
#endif
#ifndef CKPT_SIBLING_SHORTCUT
#define CKPT_SIBLING_SHORTCUT 1   // phase 3: level-1 pairs whose sources are siblings need no lookup
#endif
#ifndef CKPT_TREE_CURSOR
#define CKPT_TREE_CURSOR 1   // worklist entries beyond the first per warp from a cursor (0: static stride)
#endif
#ifndef CKPT_DIGCAP
#define CKPT_DIGCAP 256   // on-chip digests per warp (4 KB); dense groups spill to global
#endif
constexpr int kDigCap = CKPT_DIGCAP;

__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %globaltimer;" : "=l"(t));
  return t;
}

// ------------------------------------------------------------------ bit helpers
__device__ __forceinline__ uint32_t low_mask(uint64_t nbits) { return nbits >= 32 ? 0xFFFFFFFFu : ((1u << nbits) - 1u); }
__device__ __forceinline__ uint32_t rev_n(uint32_t x, int n) { return n ? (__brev(x) >> (32 - n)) : 0u; }

// 32 bits of the candidate bitmap starting at chunk c (c may be unaligned)
__device__ __forceinline__ uint32_t cand_bits(const uint32_t* cand, uint64_t c) {
  const uint64_t i = c >> 5;
  const uint32_t sh = (uint32_t)(c & 31);
  const uint32_t a = __ldg(cand + i);
  if (sh == 0) return a;
  const uint32_t b = __ldg(cand + i + 1);
  return (a >> sh) | (b << (32 - sh));
}

struct WarpSmem {
  uint32_t hitF[32];    // result bits written by work items (resolve: FIRST)
  uint32_t hitS[32];    // result bits (resolve: SHIFT)
  uint32_t T[32];       // scatter-transpose scratch
  uint32_t stF[32];     // stage-0 emission: FIRST region start slots (natural order)
  uint32_t stS[32];     //                   SHIFT region start slots
  uint32_t W[32];       // pass-1 nodes of all levels (layout below)
  uint32_t WP[32];      // exclusive prefix of popc(W): a pass-1 node's rank = its compact digest index
  uint32_t H[32];       // pass-2 lookup hits (same layout)
  uint32_t K[32];       // phase 3: level-1 pairs resolved without a lookup (same layout)
  uint16_t items[1 << kTileLog];   // the set bits of the current work mask as a list (word << 5 | bit)
  uint32_t dense;                  // list_bits: the set bits were exactly 0 .. total-1 (no list written)
  Digest dig[kDigCap];  // compact on-chip digests of pass-1 nodes (rank < kDigCap; others: global)
  uint8_t lvl[1 << kTileLog];   // level of the region starting at each slot
  unsigned long long tp[8];     // diagnostics: intra-group timestamps
};

// One 32-word layout holding a bit for every internal node of a 1024-slot group:
// level 1 -> words 0..15, level 2 -> 16..23, level 3 -> 24..27, level 4 -> 28..29,
// level 5 -> word 30, levels 6..10 packed in word 31 at bits 0, 16, 24, 28, 30.
__device__ __forceinline__ int lay_base(int lv) {
  return lv == 1 ? 0 : lv == 2 ? 16 : lv == 3 ? 24 : lv == 4 ? 28 : lv == 5 ? 30 : 31;
}
__device__ __forceinline__ int lay_shift(int lv) {
  return lv <= 6 ? 0 : lv == 7 ? 16 : lv == 8 ? 24 : lv == 9 ? 28 : 30;
}
__device__ __forceinline__ void lay_decode(uint32_t w, uint32_t b, int& lv, uint32_t& q) {
  if (w < 16) { lv = 1; q = 32 * w + b; }
  else if (w < 24) { lv = 2; q = 32 * (w - 16) + b; }
  else if (w < 28) { lv = 3; q = 32 * (w - 24) + b; }
  else if (w < 30) { lv = 4; q = 32 * (w - 28) + b; }
  else if (w == 30) { lv = 5; q = b; }
  else if (b < 16) { lv = 6; q = b; }
  else if (b < 24) { lv = 7; q = b - 16; }
  else if (b < 28) { lv = 8; q = b - 24; }
  else if (b < 30) { lv = 9; q = b - 28; }
  else { lv = 10; q = b - 30; }
}
__device__ __forceinline__ void lay_pos(int lv, uint32_t q, uint32_t& w, uint32_t& b) {
  if (lv <= 5) { w = lay_base(lv) + (q >> 5); b = q & 31; }
  else { w = 31; b = lay_shift(lv) + q; }
}
__device__ __forceinline__ uint32_t lay_rank(const WarpSmem& ws, int lv, uint32_t q) {
  uint32_t w, b;
  lay_pos(lv, q, w, b);
  return ws.WP[w] + __popc(ws.W[w] & ((1u << b) - 1u));
}
__device__ __forceinline__ Digest dig_load(const WarpSmem& ws, const Digest* spill, uint32_t idx) {
  if (idx < kDigCap) return ws.dig[idx];
  const ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2*>(spill) + idx);
  return Digest{v.x, v.y};
}
__device__ __forceinline__ void dig_store(WarpSmem& ws, Digest* spill, uint32_t idx, const Digest& d) {
  if (idx < kDigCap) ws.dig[idx] = d;
  else reinterpret_cast<ulonglong2*>(spill)[idx] = make_ulonglong2(d.lo, d.hi);
}

__device__ __forceinline__ uint64_t lvl_off(uint64_t P0, int lv) { return P0 - (P0 >> (lv - 1)); }  // lv >= 1

// The set bits of per-lane words `m` (word index = lane) as a list in shared memory: each
// lane writes its word's bit positions at its exclusive prefix. Items j are then spread
// evenly over the lanes with no per-item search (a binary search over the prefixes plus a
// find-n-th-set-bit per item was 30 % of the phase-3 instructions on dense tiles).
__device__ __forceinline__ uint32_t list_bits(WarpSmem& ws, uint32_t m) {
  const int lane = threadIdx.x & 31;
  const uint32_t cnt = __popc(m);
  uint32_t incl = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  // dense masks (every position 0 .. total-1 set, e.g. every level of a fully changed
  // tile): item j is position j, and the serial per-bit list (12 % of phase 3's
  // instructions on the duplicate-heavy config) is skipped
  const uint32_t q0 = (uint32_t)lane * 32;
  const uint32_t want = q0 < total ? low_mask(total - q0) : 0u;
  const bool dense = __all_sync(0xffffffffu, m == want);
  if (!dense) {
    uint32_t r = incl - cnt;
    for (uint32_t x = m; x; x &= x - 1) ws.items[r++] = (uint16_t)(lane * 32 + (__ffs(x) - 1));
  }
  if (lane == 0) ws.dense = dense ? 1u : 0u;
  __syncwarp();
  return total;
}

// Balanced distribution of the set bits of per-lane words `m` over the 32 lanes: calls
// f(word, bit, index) once per set bit.
template <class F>
__device__ __forceinline__ void for_each_bit_balanced(WarpSmem& ws, uint32_t m, F&& f) {
  const int lane = threadIdx.x & 31;
  if (!__any_sync(0xffffffffu, m != 0)) return;   // most levels have no work: one vote, no scan
  const uint32_t total = list_bits(ws, m);
  for (uint32_t j = lane; j < total; j += 32) {
    const uint32_t q = ws.dense ? j : ws.items[j];
    f(q >> 5, q & 31u, q);
  }
  __syncwarp();
}

// Batched form: lane takes items j = base + 32 t + lane (t < K) of the balanced order, so
// it can issue the memory operations of K items before waiting on any of them.
constexpr int kB = 4;
__device__ __forceinline__ uint32_t batch_begin(WarpSmem& ws, uint32_t m) {
  if (!__any_sync(0xffffffffu, m != 0)) return 0;
  return list_bits(ws, m);
}
// item j (< total) -> (word, bit)
__device__ __forceinline__ void batch_item(const WarpSmem& ws, uint32_t j, uint32_t& w, uint32_t& b) {
  const uint32_t q = ws.dense ? j : ws.items[j];
  w = q >> 5;
  b = q & 31u;
}

// ---- natural order -> bit-reversed order for a level of N = 2^n positions.
// n == 10: 32-ballot transpose (lane w first fetches natural word rev5(w)); smaller
// levels: scatter through shared memory (small groups only).
__device__ __forceinline__ void to_rev3(WarpSmem& ws, int n, uint32_t a, uint32_t b, uint32_t c, uint32_t& ra,
                                        uint32_t& rb, uint32_t& rc) {
  const int lane = threadIdx.x & 31;
  if (n == 10) {
    const int src = (int)rev_n((uint32_t)lane, 5);
    a = __shfl_sync(0xffffffffu, a, src);
    b = __shfl_sync(0xffffffffu, b, src);
    c = __shfl_sync(0xffffffffu, c, src);
    ra = rb = rc = 0;
#pragma unroll
    for (int bit = 0; bit < 32; ++bit) {
      const uint32_t ma = __ballot_sync(0xffffffffu, (a >> bit) & 1u);
      const uint32_t mb = __ballot_sync(0xffffffffu, (b >> bit) & 1u);
      const uint32_t mc = __ballot_sync(0xffffffffu, (c >> bit) & 1u);
      if (src == bit) { ra = ma; rb = mb; rc = mc; }   // rev5 is an involution: lane == rev5(bit)
    }
    return;
  }
  uint32_t* out[3] = {&ra, &rb, &rc};
  const uint32_t in[3] = {a, b, c};
#pragma unroll
  for (int k = 0; k < 3; ++k) {
    ws.T[lane] = 0;
    __syncwarp();
    for (uint32_t m = in[k]; m; m &= m - 1) {
      const uint32_t q = lane * 32 + (__ffs(m) - 1);
      const uint32_t r = rev_n(q, n);
      atomicOr(&ws.T[r >> 5], 1u << (r & 31));
    }
    __syncwarp();
    *out[k] = ws.T[lane];
    __syncwarp();
  }
}

// Children masks of this lane's parent word: left children (index r) and right children
// (index r + Np) of a level with Nc positions in bit-reversed order.
__device__ __forceinline__ void lr(uint32_t M, uint64_t Nc, uint32_t& l, uint32_t& r) {
  const int lane = threadIdx.x & 31;
  const uint64_t Np = Nc >> 1;
  if (Np >= 32) {
    const int wp = (int)(Np >> 5);
    l = M;
    r = __shfl_sync(0xffffffffu, M, (lane + wp) & 31);
  } else {
    const uint32_t x = __shfl_sync(0xffffffffu, M, 0);
    l = x & low_mask(Np);
    r = (x >> Np) & low_mask(Np);
  }
}

// Parent bits (this level, Np positions) seen from the children words of the level below.
__device__ __forceinline__ uint32_t to_children(uint32_t D, uint64_t Nc) {
  const int lane = threadIdx.x & 31;
  const uint64_t Np = Nc >> 1;
  if (Np >= 32) {
    const int wp = (int)(Np >> 5);
    return __shfl_sync(0xffffffffu, D, lane % wp);
  }
  const uint32_t d = __shfl_sync(0xffffffffu, D, 0) & low_mask(Np);
  return lane == 0 ? (d | (d << Np)) : 0u;
}

__device__ __forceinline__ uint32_t valid_word(uint64_t N) {
  const uint64_t q0 = (uint64_t)(threadIdx.x & 31) * 32;
  return q0 < N ? low_mask(N - q0) : 0u;
}

struct Ctx {
  const TreeParams* p;
  int s;             // stage
  uint64_t G;        // group index
  int Lin, gsz;
  uint64_t P0;       // positions at the input height
  bool leaf;         // stage 0
  Digest* tdig;      // this group's spilled digests (P0 entries)
  unsigned long long* tsrc;   // this group's sources (2 P0 entries, bit-reversed indices)
  bool pub;          // the group published a FIRST/SHIFT root to its parent (needs a release)
};

// digest of the node at (lv, rev index r) of the current group: leaves / inputs from
// global memory, internal pass-1 nodes from the warp's compact store
__device__ __forceinline__ Digest child_digest(const Ctx& c, const WarpSmem& ws, int lv, uint32_t r) {
  const TreeParams& p = *c.p;
  if (lv == 0) {
    const uint64_t q = rev_n(r, c.gsz);
    const ulonglong2* base =
        c.leaf ? reinterpret_cast<const ulonglong2*>(p.prev) : reinterpret_cast<const ulonglong2*>(p.st[c.s].in.dig);
    const ulonglong2 v = c.leaf ? __ldg(base + ((c.G << c.gsz) + q)) : __ldcg(base + ((c.G << c.gsz) + q));
    return Digest{v.x, v.y};
  }
  if (lv == 1 && c.leaf) {
    const uint64_t gq = (c.G << (c.gsz - 1)) + rev_n(r, c.gsz - 1);
    if (2 * gq >= p.g.m) {
      const ulonglong2 v = __ldg(reinterpret_cast<const ulonglong2*>(p.prev) + (gq + p.g.m / 2));
      return Digest{v.x, v.y};
    }
  }
  return dig_load(ws, c.tdig, lay_rank(ws, lv, r));
}

__device__ __forceinline__ unsigned long long child_src(const Ctx& c, int lv, uint32_t r) {
  const TreeParams& p = *c.p;
  if (lv == 0) {
    if (c.leaf) return __ldcg(c.tsrc + r);
    return __ldcg(p.st[c.s].in.src + ((c.G << c.gsz) + rev_n(r, c.gsz)));
  }
  return __ldcg(c.tsrc + c.P0 + lvl_off(c.P0, lv) + r);
}

// Leaf labels of a chunk range (stage 0, phase 2): every candidate is resolved against
// the record (R6: FIRST iff the record's entry is this leaf; otherwise SHIFT with that
// entry as its source), the rest are FIXED. Returns NATURAL-order masks for positions
// [0, npos) (word = lane); the SHIFT sources go to tsrc[src_base + rev_n(pos0 + pos)].
// The leaf classes (first / spatial / temporal) are counted here.
struct LeafCount {
  uint32_t f, s, t;
};

__device__ __forceinline__ void resolve_leaves(const Ctx& c, WarpSmem& ws, uint64_t chunk0, uint64_t npos,
                                               uint64_t src_base, uint32_t pos0, int nrev, uint32_t& F, uint32_t& S,
                                               uint32_t& X, LeafCount& lc) {
  const TreeParams& p = *c.p;
  const int lane = threadIdx.x & 31;
  uint32_t valid = 0, cand = 0;
  const uint64_t q0 = (uint64_t)lane * 32;
  if (q0 < npos) {
    valid = low_mask(npos - q0);
    cand = cand_bits(p.cand, chunk0 + q0) & valid;
  }
  ws.hitF[lane] = 0;
  ws.hitS[lane] = 0;
  __syncwarp();
  const uint32_t k = p.g.k;
  const uint32_t total = batch_begin(ws, cand);
  for (uint32_t base = 0; base < total; base += 32 * kB) {
    uint64_t ch[kB];
    uint32_t iw[kB], ib[kB];
    unsigned long long val[kB];
#pragma unroll
    for (int t = 0; t < kB; ++t) {
      const uint32_t j = base + 32 * t + lane;
      ch[t] = ~0ull;
      if (j < total) {
        batch_item(ws, j, iw[t], ib[t]);
        ch[t] = chunk0 + iw[t] * 32 + ib[t];
      }
    }
#pragma unroll
    for (int t = 0; t < kB; ++t)
      if (ch[t] != ~0ull) val[t] = __ldg(p.res_of + ch[t]);
    // leaves K1b could not resolve (their key was claimed or lowered in this checkpoint):
    // the final value after every insert
#pragma unroll
    for (int t = 0; t < kB; ++t)
      if (ch[t] != ~0ull && (val[t] & kResPending)) val[t] = __ldcg(&p.tab[(uint32_t)val[t]].val);
#pragma unroll
    for (int t = 0; t < kB; ++t) {
      if (ch[t] == ~0ull) continue;
      const uint32_t pos = iw[t] * 32 + ib[t];
      if (val[t] == pack_entry(k, node_of_chunk(p.g, ch[t]))) {
        atomicOr(&ws.hitF[iw[t]], 1u << ib[t]);
        ++lc.f;
      } else {
        atomicOr(&ws.hitS[iw[t]], 1u << ib[t]);
        c.tsrc[src_base + rev_n(pos0 + pos, nrev)] = val[t];
        if ((uint32_t)(val[t] >> 32) == k) ++lc.s; else ++lc.t;
      }
    }
  }
  __syncwarp();
  F = ws.hitF[lane];
  S = ws.hitS[lane];
  X = valid & ~cand;
}

__device__ __forceinline__ bool insert_new_from(Slot* tab, uint64_t cap, const Digest& d, unsigned long long packed,
                                                uint64_t s) {
  for (;;) {
    unsigned long long olo, ohi;
    cas128(tab + s, kEmpty, kEmpty, d.lo, d.hi, olo, ohi);
    if (olo == kEmpty && ohi == kEmpty) {
      tab[s].val = packed;
      return true;
    }
    if (olo == d.lo && ohi == d.hi) return false;
    if (++s == cap) s = 0;
  }
}

// Emit the region (lv, rev index r) of the current group (phase 3).
__device__ __forceinline__ void emit_region(const Ctx& c, WarpSmem& ws, int lv, uint32_t r, bool first,
                                           unsigned long long src) {
  const TreeParams& p = *c.p;
  const uint32_t q = rev_n(r, c.gsz - lv);   // natural position
  if (c.leaf) {
    const uint32_t slot = q << lv;
    atomicOr(first ? &ws.stF[slot >> 5] : &ws.stS[slot >> 5], 1u << (slot & 31));
    ws.lvl[slot] = (uint8_t)lv;
    return;
  }
  const int Lc = c.Lin + lv;
  const uint64_t gpos = (c.G << (c.gsz - lv)) + q;
  const uint32_t node = node_id(p.g, Lc, gpos);
  const uint64_t tile = (gpos << Lc) >> p.g.t0;
  p.scratch[tile << p.g.t0] = make_uint4(node, (uint32_t)(src & 0xffffffffu), (uint32_t)(src >> 32),
                                         first ? L_FIRST : L_SHIFT);
  // region counts of the region's first tile (its FIRST bytes were counted by phase 2)
  reinterpret_cast<uint2*>(p.tilecnt + tile)[0] = make_uint2(first ? 1u : 0u, first ? 0u : 1u);
  // the tile had no region of its own (it lies inside this one): add the region to the
  // sums of its 1024-tile block and 32-tile group (the gather kernel's prefix inputs)
  unsigned long long* bs = p.blocksum + 3 * (tile / kTilesPerBlock);
  unsigned long long* gs = p.gsum + 3 * (tile / 32);
  atomicAdd(bs + (first ? 0 : 1), 1ull);
  atomicAdd(gs + (first ? 0 : 1), 1ull);
}

// Natural-order bit words (lane i = bits 32i..32i+31) shifted up by s bits across the warp.
__device__ __forceinline__ uint32_t shift_up_bits(uint32_t w, uint32_t s) {
  const int lane = threadIdx.x & 31;
  const int q = (int)(s >> 5);
  const uint32_t r = s & 31;
  const uint32_t cur = __shfl_sync(0xffffffffu, w, (lane - q) & 31);
  const uint32_t prv = __shfl_sync(0xffffffffu, w, (lane - q - 1) & 31);
  uint32_t o = 0;
  if (lane >= q) o = cur << r;
  if (lane >= q + 1 && r) o |= prv >> (32 - r);
  return o;
}

// Process one group through its gsz levels. PHASE 2 or 3.
template <int PHASE>
__device__ void process_group(Ctx& c, WarpSmem& ws, unsigned long long& ins_cnt, unsigned long long& coll_cnt,
                              LeafCount& lc) {
  const TreeParams& p = *c.p;
  const Geo& g = p.g;
  const int lane = threadIdx.x & 31;
  const uint64_t P0 = c.P0;
  const int gsz = c.gsz;
  uint32_t F = 0, S = 0, X = 0;                      // current level (bit-reversed order)
  uint32_t leafm1 = 0, lF1 = 0, lS1 = 0, lX1 = 0;   // level-1 leaves of depth h-1 (R3)
  uint32_t* lm = c.leaf ? p.lmask + c.G * kLmWords : nullptr;

  // ---- input level
  if (c.leaf) {
    const uint64_t base = c.G << gsz;
    const uint64_t npos0 = base < g.m ? (g.m - base < P0 ? g.m - base : P0) : 0;   // real leaves at height 0
    const uint64_t Np1 = P0 >> 1;
    const uint64_t pbase1 = c.G << (gsz - 1);
    const uint64_t first_leaf = gsz >= 1 ? ((g.m / 2 > pbase1) ? g.m / 2 - pbase1 : 0) : Np1;   // local, level 1
    const bool has_l1 = gsz >= 1 && first_leaf < Np1;
    if (PHASE == 2) {
      uint32_t nF, nS, nX;
      resolve_leaves(c, ws, base, npos0, 0, 0, gsz, nF, nS, nX, lc);
      uint32_t fchunks = nF;   // the tile's FIRST chunks, chunk order (height-0 chunks first)
      to_rev3(ws, gsz, nF, nS, nX, F, S, X);
      lm[lane] = F;
      lm[32 + lane] = S;
      lm[64 + lane] = X;
      if (has_l1) {
        // chunks gq + m/2 for level-1 local positions [first_leaf, Np1)
        uint32_t tF, tS, tX;
        resolve_leaves(c, ws, pbase1 + first_leaf + g.m / 2, Np1 - first_leaf, P0 + lvl_off(P0, 1),
                       (uint32_t)first_leaf, gsz - 1, tF, tS, tX, lc);
        // natural words relative to first_leaf -> natural words of level 1
        const uint32_t sh = (uint32_t)(first_leaf & 31);
        const int wsrc = (int)(first_leaf >> 5);
        auto realign = [&](uint32_t m) {
          const int a = lane - wsrc;
          const uint32_t cur = __shfl_sync(0xffffffffu, m, a < 0 ? 0 : (a & 31));
          const uint32_t prv = __shfl_sync(0xffffffffu, m, (a - 1) < 0 ? 0 : ((a - 1) & 31));
          uint32_t r = 0;
          if (a >= 0) r = cur << sh;
          if (a >= 1 && sh) r |= prv >> (32 - sh);
          return r;
        };
        const uint32_t v1 = valid_word(Np1);
        const uint32_t q0 = lane * 32;
        const uint32_t lmn = (q0 + 32 > first_leaf) ? (v1 & ~low_mask(first_leaf > q0 ? first_leaf - q0 : 0)) : 0u;
        to_rev3(ws, gsz - 1, realign(tF) & lmn, realign(tS) & lmn, lmn, lF1, lS1, leafm1);
        lm[96 + lane] = lF1;
        lm[128 + lane] = lS1;
        lm[160 + lane] = leafm1;
        fchunks |= shift_up_bits(tF, (uint32_t)npos0);   // height-1 chunks follow at offset npos0
      }
      // The data section is the FIRST chunks in chunk order (every FIRST leaf lies in exactly
      // one FIRST region and those regions hold only FIRST leaves), so the gather kernel
      // needs just this mask and the tile's FIRST bytes (the last chunk may be short).
      lm[kLmFirstChunks + lane] = fchunks;
      uint32_t nfc = __popc(fchunks);
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) nfc += __shfl_xor_sync(0xffffffffu, nfc, o);
      uint64_t lo, hi;
      chunk_range(g, g.t0, c.G, lo, hi);
      unsigned long long fb = (unsigned long long)nfc * g.C;
      if (hi == g.n) {   // the tile holds the buffer's last chunk, possibly short
        const uint32_t b = (uint32_t)(g.n - 1 - lo);
        const uint32_t wlast = __shfl_sync(0xffffffffu, fchunks, (int)(b >> 5));
        if ((wlast >> (b & 31)) & 1u) fb -= (unsigned long long)g.n * g.C - g.B;
      }
      if (lane == 0) {
        reinterpret_cast<uint2*>(p.tilecnt + c.G)[1] = make_uint2((uint32_t)fb, g.epoch);
        if (fb) {
          atomicAdd(p.blocksum + 3 * (c.G / kTilesPerBlock) + 2, fb);
          atomicAdd(p.gsum + 3 * (c.G / 32) + 2, fb);
        }
      }
    } else {
      F = __ldcg(lm + lane);
      S = __ldcg(lm + 32 + lane);
      X = __ldcg(lm + 64 + lane);
      if (has_l1) {
        lF1 = __ldcg(lm + 96 + lane);
        lS1 = __ldcg(lm + 128 + lane);
        leafm1 = __ldcg(lm + 160 + lane);
      }
      ws.stF[lane] = 0;
      ws.stS[lane] = 0;
    }
    lX1 = leafm1 & ~(lF1 | lS1);
  } else {
    // the children ORed their FIRST / SHIFT root labels into this group's masks
    // (bit-reversed order). Every other child is FIXED or DONE; the two behave alike from
    // here up (neither is emitted, and a parent with a FIRST/SHIFT child and a FIXED or
    // DONE child is DONE either way), so both are carried as X.
    const StageParams& sp = p.st[c.s];
    if (PHASE == 2) {
      F = __ldcg(sp.gm2 + c.G * 32 + lane);
      S = 0;
    } else if (PHASE == 4) {
      F = 0;
      S = __ldcg(sp.gm4 + c.G * 32 + lane);
    } else {
      const uint32_t* gm = sp.gm3 + c.G * 64;
      F = __ldcg(gm + lane);
      S = __ldcg(gm + 32 + lane);
    }
    X = valid_word(P0) & ~(F | S);
  }
  __syncwarp();
  if (p.trace && lane == 0) ws.tp[0] = gtimer();

  // An upper group none of whose children has a FIRST or SHIFT root (the steady state:
  // updates are far smaller than a tile) hashes, inserts and emits nothing; its root is
  // FIXED iff every child is, else DONE.
  const bool trivial = !c.leaf && !__any_sync(0xffffffffu, (F | S) != 0);
  if (p.list) {
    // List: no compaction — no internal node is hashed, inserted or looked up;
    // phase 3 emits every FIRST / SHIFT leaf as an entry of its own (R13 order follows
    // from the stage-0 compaction below), and nothing climbs.
    if (PHASE == 3) {
      for (uint32_t m = F | S; m; m &= m - 1) {
        const uint32_t b = __ffs(m) - 1;
        emit_region(c, ws, 0, (uint32_t)lane * 32 + b, (F >> b) & 1u, 0ull);
      }
      for (uint32_t m = lF1 | lS1; m; m &= m - 1) {   // leaves at height 1 (R3, n != 2^h)
        const uint32_t b = __ffs(m) - 1;
        emit_region(c, ws, 1, (uint32_t)lane * 32 + b, (lF1 >> b) & 1u, 0ull);
      }
      __syncwarp();
    }
    F = 0; S = 0; X = 0;
  } else if (trivial) {
    const bool allX = __all_sync(0xffffffffu, X == valid_word(P0));
    X = (lane == 0 && allX) ? 1u : 0u;
  } else {
  // ---- pass 1: digests bottom-up, no record traffic (see file header)
  ws.W[lane] = 0;
  ws.K[lane] = 0;
  __syncwarp();
  uint32_t Ptop = 0;   // PHASE 4: potential shifted nodes at the group's top level
  if (__any_sync(0xffffffffu, ((PHASE == 2 ? F : S) | (PHASE == 2 ? lF1 : lS1)) != 0)) {
    uint32_t P = PHASE == 2 ? F : S;
    for (int lv = 1; lv <= gsz; ++lv) {
      const uint64_t Nc = P0 >> (lv - 1), Np = Nc >> 1;
      uint32_t l, r;
      lr(P, Nc, l, r);
      const uint32_t work = l & r & valid_word(Np) & (lv == 1 ? ~leafm1 : 0xFFFFFFFFu);
      const uint32_t inj = lv == 1 ? (PHASE == 2 ? lF1 : lS1) : 0u;
      if (!__any_sync(0xffffffffu, work != 0)) {
        P = inj;
        continue;
      }
      if (lv <= 5) {
        if ((uint64_t)lane * 32 < Np) ws.W[lay_base(lv) + lane] = work;
      } else if (lane == 0) {
        ws.W[31] |= work << lay_shift(lv);
      }
      __syncwarp();
      {   // ranks: exclusive prefix of the layout popcounts
        const uint32_t cnt = __popc(ws.W[lane]);
        uint32_t incl = cnt;
#pragma unroll
        for (int o2 = 1; o2 < 32; o2 <<= 1) {
          const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o2);
          if (lane >= o2) incl += v;
        }
        ws.WP[lane] = incl - cnt;
      }
      __syncwarp();
      for_each_bit_balanced(ws, work, [&](uint32_t, uint32_t, uint32_t q) {
        if (PHASE == 3 && lv == 1 && CKPT_SIBLING_SHORTCUT) {
          // Both children are SHIFT with known sources. If they are the two children of one
          // node v of checkpoint c (left = 2v+1, right = 2v+2), both were FIRST in c, so
          // phase 2 of c inserted (v, c) for exactly this digest (the record never replaces
          // an entry, R6): the lookup of Alg.1 l.39 would return it, and is skipped.
          // (Applying the same rule at higher levels, from children resolved this way,
          // measured slower: config 4 phase 3 425 -> 434 us.)
          const unsigned long long sL = child_src(c, 0, q), sR = child_src(c, 0, q + (uint32_t)Np);
          const uint32_t nl = (uint32_t)sL, nr = (uint32_t)sR;
          if ((sL >> 32) == (sR >> 32) && (nl & 1u) && nr == nl + 1) {
            atomicOr(&ws.K[q >> 5], 1u << (q & 31));
            c.tsrc[P0 + lvl_off(P0, 1) + q] = (sL & 0xFFFFFFFF00000000ull) | ((nl - 1) >> 1);
          }
        }
        const Digest d = mm::node(child_digest(c, ws, lv - 1, q), child_digest(c, ws, lv - 1, q + (uint32_t)Np));
        dig_store(ws, c.tdig, lay_rank(ws, lv, q), d);
      });
      P = work | inj;
    }
    Ptop = P;
  }
  __syncwarp();
  if (p.trace && lane == 0) ws.tp[1] = gtimer();

  // ---- pass 2: record operations for all pass-1 nodes at once (phase 3: but the pairs
  // pass 1 resolved from their children's sources)
  ws.H[lane] = PHASE == 3 ? ws.K[lane] : 0u;
  __syncwarp();
  if (PHASE == 4) {
    // R24: every potential shifted node's hash enters the record unless present; the
    // minimum node id wins among equal new hashes (read first: hot repeated keys, e.g. the
    // all-zero subtrees of a first checkpoint, meet on one slot)
    const uint32_t total = batch_begin(ws, ws.W[lane]);
    for (uint32_t j = lane; j < total; j += 32) {
      uint32_t iw, ib;
      batch_item(ws, j, iw, ib);
      int lv;
      uint32_t r;
      lay_decode(iw, ib, lv, r);
      const Digest d = dig_load(ws, c.tdig, ws.WP[iw] + __popc(ws.W[iw] & ((1u << ib) - 1u)));
      const uint64_t gpos = (c.G << (gsz - lv)) + rev_n(r, gsz - lv);
      bool claimed;
      unsigned long long seen;
      table_insert_min(p.tab, p.cap, d, pack_entry(g.k, node_id(g, c.Lin + lv, gpos)), &claimed, false, &seen);
      if (claimed) ++ins_cnt;
    }
    __syncwarp();
  } else {
    constexpr int kB2 = CKPT_TREE_KB2;
    const uint32_t total = batch_begin(ws, PHASE == 3 ? (ws.W[lane] & ~ws.K[lane]) : ws.W[lane]);
    for (uint32_t base = 0; base < total; base += 32 * kB2) {
      uint32_t iw[kB2], ib[kB2];
      int lvs[kB2];
      uint32_t rs[kB2];
      Digest d[kB2];
      uint64_t sl[kB2];
      unsigned long long olo[kB2], ohi[kB2], oval[kB2];
      bool has[kB2];
#pragma unroll
      for (int t = 0; t < kB2; ++t) {
        const uint32_t j = base + 32 * t + lane;
        has[t] = j < total;
        if (has[t]) {
          batch_item(ws, j, iw[t], ib[t]);
          lay_decode(iw[t], ib[t], lvs[t], rs[t]);
          d[t] = dig_load(ws, c.tdig, ws.WP[iw[t]] + __popc(ws.W[iw[t]] & ((1u << ib[t]) - 1u)));
          sl[t] = slot_home(d[t].lo, p.cap);
        }
      }
      // first probe of every item in flight at once
#pragma unroll
      for (int t = 0; t < kB2; ++t) {
        if (!has[t]) continue;
        if (PHASE == 2) {
          cas128(p.tab + sl[t], kEmpty, kEmpty, d[t].lo, d[t].hi, olo[t], ohi[t]);   // Alg.1 l.29 (new key)
        } else {
          ld_slot_cg(p.tab + sl[t], olo[t], ohi[t], oval[t]);   // Alg.1 l.39: key and value, one load
        }
      }
#pragma unroll
      for (int t = 0; t < kB2; ++t) {
        if (!has[t]) continue;
        const int lv = lvs[t];
        const uint32_t r = rs[t];
        if (PHASE == 2) {
          const uint64_t gpos = (c.G << (gsz - lv)) + rev_n(r, gsz - lv);
          const unsigned long long packed = pack_entry(g.k, node_id(g, c.Lin + lv, gpos));
          bool ok;
          if (olo[t] == kEmpty && ohi[t] == kEmpty) {
            p.tab[sl[t]].val = packed;
            ok = true;
          } else if (olo[t] == d[t].lo && ohi[t] == d[t].hi) {
            ok = false;
          } else {
            uint64_t s2 = sl[t] + 1 == p.cap ? 0 : sl[t] + 1;
            (void)s2;
            ok = insert_new_from(p.tab, p.cap, d[t], packed, s2);
          }
          if (ok) ++ins_cnt;
          else ++coll_cnt;   // R14: a FIRST-FIRST digest already in the record = 128-bit collision
        } else {
          unsigned long long v;
          if (olo[t] == d[t].lo && ohi[t] == d[t].hi) v = oval[t];
          else if (olo[t] == kEmpty && ohi[t] == kEmpty) v = kEmpty;
          else v = table_lookup_from(p.tab, p.cap, d[t], sl[t] + 1 == p.cap ? 0 : sl[t] + 1);
          // R24: a node that finds its own entry is the first occurrence of its content
          if (v != kEmpty && p.shift_insert &&
              v == pack_entry(g.k, node_id(g, c.Lin + lv, (c.G << (gsz - lv)) + rev_n(r, gsz - lv))))
            v = kEmpty;
          if (v != kEmpty) {
            atomicOr(&ws.H[iw[t]], 1u << ib[t]);
            c.tsrc[P0 + lvl_off(P0, lv) + r] = v;
          }
        }
      }
    }
    __syncwarp();
  }
  if (p.trace && lane == 0) ws.tp[2] = gtimer();

  if (PHASE == 4) {
    F = 0;
    S = Ptop;   // the group root is a potential shifted node iff bit 0 of lane 0 is set
  } else if (PHASE == 2) {
    // the FIRST label chain up to the group root (stops once no FIRST node is left)
    for (int lv = 1; lv <= gsz; ++lv) {
      const uint64_t Nc = P0 >> (lv - 1), Np = Nc >> 1;
      uint32_t l, r;
      lr(F, Nc, l, r);
      F = (l & r & valid_word(Np) & (lv == 1 ? ~leafm1 : 0xFFFFFFFFu)) | (lv == 1 ? lF1 : 0u);
      if (!__any_sync(0xffffffffu, F != 0)) break;
    }
  } else {
    // ---- pass 3: Alg.1 l.33-46 with the lookup results; emission of "roots" (R8)
    for (int lv = 1; lv <= gsz; ++lv) {
      const uint64_t Nc = P0 >> (lv - 1), Np = Nc >> 1;
      uint32_t lF, rF, lS, rS, lX, rX;
      lr(F, Nc, lF, rF);
      lr(S, Nc, lS, rS);
      lr(X, Nc, lX, rX);
      const uint32_t leafm = lv == 1 ? leafm1 : 0u;
      const uint32_t valid = valid_word(Np) & ~leafm;
      uint32_t hw;
      if (lv <= 5) hw = ((uint64_t)lane * 32 < Np) ? ws.H[lay_base(lv) + lane] : 0u;
      else hw = lane == 0 ? (ws.H[31] >> lay_shift(lv)) & low_mask(Np) : 0u;
      const uint32_t bothF = lF & rF & valid;
      const uint32_t bothX = lX & rX & valid;
      const uint32_t hitS = lS & rS & valid & hw;        // both children SHIFT and found
      const uint32_t nD = valid & ~bothF & ~bothX & ~hitS;
      // the FIRST/SHIFT children of DONE parents are regions
      const uint32_t dchild = to_children(nD, Nc);
      const uint32_t emF = dchild & F, emS = dchild & S;
      // emissions spread evenly over the lanes (a dense word would serialise one lane)
      ws.T[lane] = emF;
      const uint32_t ne = batch_begin(ws, emF | emS);
      for (uint32_t j = lane; j < ne; j += 32) {
        uint32_t w, b;
        batch_item(ws, j, w, b);
        const bool isF = (ws.T[w] >> b) & 1u;
        const uint32_t rr = w * 32 + b;
        emit_region(c, ws, lv - 1, rr, isF, (isF || c.leaf) ? 0ull : child_src(c, lv - 1, rr));
      }
      __syncwarp();
      F = bothF | (lv == 1 ? lF1 : 0u);
      X = bothX | (lv == 1 ? lX1 : 0u);
      S = hitS | (lv == 1 ? lS1 : 0u);
      if (lv < gsz && !__any_sync(0xffffffffu, (F | S) != 0)) {
        // no FIRST/SHIFT node left: the levels above hold only FIXED and DONE nodes and
        // emit nothing; the root is FIXED iff every node of this level is FIXED
        const bool allX = __all_sync(0xffffffffu, X == valid_word(Np));
        X = (lane == 0 && allX) ? 1u : 0u;
        break;
      }
    }
  }

  }   // !trivial
  if (p.trace && lane == 0) ws.tp[3] = gtimer();
  // ---- group root (single position at level gsz: lane 0 bit 0)
  const uint32_t rF = __shfl_sync(0xffffffffu, F, 0) & 1u;
  const uint32_t rS = __shfl_sync(0xffffffffu, S, 0) & 1u;
  const bool last = (c.s == p.S - 1);
  c.pub = !last && (rF || (PHASE != 2 && rS));
  if (last) {
    if (PHASE == 3 && lane == 0 && (rF | rS))
      emit_region(c, ws, gsz, 0, rF != 0, rS ? child_src(c, gsz, 0) : 0ull);   // R10
  } else if (lane == 0) {
    const StageParams& nx = p.st[c.s + 1];
    const uint32_t qn = (uint32_t)(c.G & ((1ull << nx.gsz) - 1));   // natural position in the parent group
    const uint32_t rr = rev_n(qn, nx.gsz);
    const uint64_t Pg = c.G >> nx.gsz;
    if (PHASE == 2) {
      if (rF) {
        const Digest d = child_digest(c, ws, gsz, 0);
        reinterpret_cast<ulonglong2*>(nx.in.dig)[c.G] = make_ulonglong2(d.lo, d.hi);
        atomicOr(nx.gm2 + Pg * 32 + (rr >> 5), 1u << (rr & 31));
      }
    } else if (PHASE == 4) {
      if (rS) {
        const Digest d = child_digest(c, ws, gsz, 0);
        reinterpret_cast<ulonglong2*>(nx.in.dig)[c.G] = make_ulonglong2(d.lo, d.hi);
        atomicOr(nx.gm4 + Pg * 32 + (rr >> 5), 1u << (rr & 31));
      }
    } else {
      if (rS) {
        const Digest d = child_digest(c, ws, gsz, 0);
        reinterpret_cast<ulonglong2*>(nx.in.dig)[c.G] = make_ulonglong2(d.lo, d.hi);
        nx.in.src[c.G] = child_src(c, gsz, 0);
      }
      if (rF | rS) atomicOr(nx.gm3 + Pg * 64 + (rF ? 0 : 32) + (rr >> 5), 1u << (rr & 31));
    }
  }
  __syncwarp();

  if (p.trace && lane == 0) ws.tp[4] = gtimer();
  // ---- stage-0 compaction of this tile's regions (leaf order; FIRST list then SHIFT list)
  if (PHASE == 3 && c.leaf) {
    const uint32_t wF = ws.stF[lane], wS = ws.stS[lane];
    uint32_t iF = __popc(wF), iS = __popc(wS);
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t a = __shfl_up_sync(0xffffffffu, iF, o), b = __shfl_up_sync(0xffffffffu, iS, o);
      if (lane >= o) { iF += a; iS += b; }
    }
    const uint32_t nFt = __shfl_sync(0xffffffffu, iF, 31), nSt = __shfl_sync(0xffffffffu, iS, 31);
    // Records j = 0 .. nFt + nSt - 1 spread evenly over the lanes (j = base + 32 t + lane):
    // record j is the j-th FIRST region start (chunk order) or the (j - nFt)-th SHIFT one,
    // listed in shared memory (each lane writes its words' starts at their prefixes); the
    // source loads of a lane's SHIFT records are all issued before any record is written.
    {
      uint32_t r = iF - __popc(wF);
      for (uint32_t x = wF; x; x &= x - 1) ws.items[r++] = (uint16_t)(lane * 32 + (__ffs(x) - 1));
      r = nFt + iS - __popc(wS);
      for (uint32_t x = wS; x; x &= x - 1) ws.items[r++] = (uint16_t)(lane * 32 + (__ffs(x) - 1));
    }
    __syncwarp();
    uint4* out = p.scratch + (c.G << g.t0);
    const uint32_t R = nFt + nSt;
    constexpr int kE = 4;
    for (uint32_t base = 0; base < R; base += 32 * kE) {
      uint32_t slot[kE];
      int lv[kE];
      unsigned long long src[kE];
#pragma unroll
      for (int t = 0; t < kE; ++t) {
        const uint32_t j = base + 32 * t + lane;
        slot[t] = ~0u;
        if (j < R) {
          const bool isF = j < nFt;
          slot[t] = ws.items[j];
          lv[t] = ws.lvl[slot[t]];
          src[t] = isF ? 0ull : child_src(c, lv[t], rev_n(slot[t] >> lv[t], gsz - lv[t]));
        }
      }
#pragma unroll
      for (int t = 0; t < kE; ++t) {
        const uint32_t j = base + 32 * t + lane;
        if (slot[t] == ~0u) continue;
        const uint64_t gpos = (c.G << (gsz - lv[t])) + (slot[t] >> lv[t]);
        out[j] = make_uint4(node_id(g, lv[t], gpos), (uint32_t)(src[t] & 0xffffffffu), (uint32_t)(src[t] >> 32),
                            j < nFt ? L_FIRST : L_SHIFT);
      }
    }
    if (lane == 0) {
      reinterpret_cast<uint2*>(p.tilecnt + c.G)[0] = make_uint2(nFt, nSt);   // bytes: phase 2
      unsigned long long* bs = p.blocksum + 3 * (c.G / kTilesPerBlock);
      unsigned long long* gs = p.gsum + 3 * (c.G / 32);
      if (nFt) { atomicAdd(bs, (unsigned long long)nFt); atomicAdd(gs, (unsigned long long)nFt); }
      if (nSt) { atomicAdd(bs + 1, (unsigned long long)nSt); atomicAdd(gs + 1, (unsigned long long)nSt); }
    }
    __syncwarp();
  }
}

}  // namespace

// ================================================================= kernel
template <int PHASE>
__global__ void __launch_bounds__(kTreeThreads, CKPT_TREE_BPS) tree_kernel(const __grid_constant__ TreeParams p) {
  extern __shared__ __align__(16) uint8_t tree_smem[];
  WarpSmem* sm = reinterpret_cast<WarpSmem*>(tree_smem);
  __shared__ unsigned long long s_cnt[4];
  LeafCount lc{0, 0, 0};
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  WarpSmem& ws = sm[wid];
  const unsigned long long bt0 = p.trace ? gtime_ns() : 0;
  pdl_launch_dependents();
  if (threadIdx.x < 4) s_cnt[threadIdx.x] = 0;
  __syncthreads();
  pdl_wait();
  const unsigned long long bt1 = p.trace ? gtime_ns() : 0;
  unsigned long long ins = 0, coll = 0;

  // Climb from (stage s, group G) after it is finished. Only a FULL group (every leaf below
  // it a candidate) can have a FIRST or SHIFT root, and a parent has work only through
  // such children, so only full groups arrive at their parent; the warp of the last full
  // arrival (K1b counted them) processes the parent. In the steady state no tile is full
  // and nothing climbs.
  auto climb = [&](Ctx& c) {
    if (p.list) return;   // List: no tree above the leaves
    while (c.s < p.S - 1) {
      const bool full = c.s == 0 ? tile_full(p.g, p.tcc, c.G) : __ldcg(p.st[c.s].dcnt + c.G) == (1u << c.gsz);
      if (!full) return;
      const StageParams& up = p.st[c.s + 1];
      const uint64_t P = c.G >> up.gsz;
      const uint32_t target = __ldcg(up.dcnt + P);
      uint32_t old = 0;
      // release: only a group that published a root label / digest to the parent has
      // writes the parent's processor reads (nothing else it wrote is read in this kernel)
      if (c.pub) __threadfence();
      if (lane == 0) old = atomicAdd((PHASE == 2 ? up.arr2 : PHASE == 3 ? up.arr3 : up.arr4) + P, 1u);
      old = __shfl_sync(0xffffffffu, old, 0);
      if (old + 1 != target) return;   // not the last full child
      __threadfence();
      c.s += 1;
      c.G = P;
      c.Lin = up.Lin;
      c.gsz = up.gsz;
      c.P0 = 1ull << c.gsz;
      c.leaf = false;
      c.tdig = up.tdig + (P << c.gsz);
      c.tsrc = up.tsrc + ((P << c.gsz) << 1);
      unsigned long long t0 = p.trace ? gtimer() : 0;
      process_group<PHASE>(c, ws, ins, coll, lc);
      if (p.trace && lane == 0) {
        if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 3)) {
          r[0] = make_ulonglong4(t0, gtimer(), ((unsigned long long)c.s << 32) | c.G, PHASE);
          r[1] = make_ulonglong4(ws.tp[0], ws.tp[1], ws.tp[2], 40 + PHASE);
          r[2] = make_ulonglong4(ws.tp[3], ws.tp[4], 0, 50 + PHASE);
        }
      }
    }
  };

  auto run_tile = [&](uint64_t T) {
    Ctx c;
    c.p = &p;
    c.s = 0;
    c.G = T;
    c.Lin = 0;
    c.gsz = p.st[0].gsz;
    c.P0 = 1ull << c.gsz;
    c.leaf = true;
    c.tdig = p.st[0].tdig + (c.G << c.gsz);
    c.tsrc = p.st[0].tsrc + ((c.G << c.gsz) << 1);
    unsigned long long t0 = p.trace ? gtimer() : 0;
    process_group<PHASE>(c, ws, ins, coll, lc);
    if (p.trace && lane == 0) {
      if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 3)) {
        r[0] = make_ulonglong4(t0, gtimer(), (unsigned long long)c.G, PHASE);
        r[1] = make_ulonglong4(ws.tp[0], ws.tp[1], ws.tp[2], 10 + PHASE);
        r[2] = make_ulonglong4(ws.tp[3], ws.tp[4], 0, 20 + PHASE);
      }
    }
    return c;
  };

  // dirty stage-0 tiles (K1b's list); climb on the last DIRTY child of each group
  // a switched checkpoint (R23) has no tree work
  const uint32_t count = switched_full(p.tot, p.sw_permille, p.g) ? 0u : *(volatile uint32_t*)&p.tot->wl_count[0];
  const uint64_t nwarps = (uint64_t)gridDim.x * kWarps;
  // First entry per warp: w -> block w mod grid, warp w / grid (dirty tiles spread over all
  // SMs; with at most one tile per warp, as in the sparse steady state, no atomic at all).
  // Later entries come from a cursor, fetched one tile ahead so its latency overlaps the
  // current tile: dense checkpoints give tiles (and climbs) of very different cost, and a
  // static stride left warps idle at the end of the kernel.
  uint32_t* cursor = &p.tot->tree_next[PHASE - 2];
  uint64_t w = (uint64_t)wid * gridDim.x + blockIdx.x;
  while (w < count) {
    uint32_t nx = 0;
    if (CKPT_TREE_CURSOR && lane == 0 && nwarps < count) nx = atomicAdd(cursor, 1u);
    const uint64_t T = __ldcg(p.wl0 + w);
    Ctx c = run_tile(T);
    climb(c);
    w = !CKPT_TREE_CURSOR ? w + nwarps : nwarps < count ? nwarps + __shfl_sync(0xffffffffu, nx, 0) : count;
  }
  const unsigned long long ta = p.trace ? gtime_ns() : 0;
  if (PHASE == 4) {
    unsigned long long v = ins;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0 && v) atomicAdd(&s_cnt[3], v);
  }
  if (PHASE == 2) {
    // warp sums first: 64-bit shared atomics are CAS loops, 256 contending threads serialise
    unsigned long long v[5] = {ins, coll, lc.f, lc.s, lc.t};
#pragma unroll
    for (int i = 0; i < 5; ++i)
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) v[i] += __shfl_xor_sync(0xffffffffu, v[i], o);
    if (lane == 0) {
      if (v[0]) atomicAdd(&s_cnt[3], v[0]);
      if (v[1]) atomicAdd(&p.tot->collisions, v[1]);
      if (v[2]) atomicAdd(&s_cnt[0], v[2]);
      if (v[3]) atomicAdd(&s_cnt[1], v[3]);
      if (v[4]) atomicAdd(&s_cnt[2], v[4]);
    }
  }
  __syncthreads();
  const unsigned long long tb = p.trace ? gtime_ns() : 0;
  if (threadIdx.x == 0 && PHASE == 4 && s_cnt[3]) atomicAdd(&p.tot->p3_inserts, s_cnt[3]);
  if (threadIdx.x == 0 && PHASE == 2) {
    if (s_cnt[3]) atomicAdd(&p.tot->p2_inserts, s_cnt[3]);
    if (s_cnt[0]) atomicAdd(&p.tot->n_first, s_cnt[0]);
    if (s_cnt[1]) atomicAdd(&p.tot->n_spatial, s_cnt[1]);
    if (s_cnt[2]) atomicAdd(&p.tot->n_temporal, s_cnt[2]);
  }
  if (p.trace && threadIdx.x == 0)
    if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 1)) *r = make_ulonglong4(ta, tb, gtime_ns(), 90 + PHASE);
  trace_block(p.trace, p.trace_n, bt0, bt1, PHASE);
}

static int g_tree_blocks_per_sm[3] = {0, 0, 0};

cudaError_t launch_tree(const TreeParams& p, int phase, int num_sms, cudaStream_t st) {
  // all CTAs resident at once (static tile striding relies on it): occupancy-sized grid
  const int bps = g_tree_blocks_per_sm[phase - 2] > 0 ? g_tree_blocks_per_sm[phase - 2] : 2;
  uint64_t grid = (uint64_t)num_sms * bps;
  if (grid > p.n_tiles) grid = p.n_tiles ? p.n_tiles : 1;   // worklist spread over blocks first
  const size_t smem = kWarps * sizeof(WarpSmem);
  if (phase == 2) return launch_pdl(tree_kernel<2>, (unsigned)grid, kTreeThreads, smem, st, p);
  if (phase == 4) return launch_pdl(tree_kernel<4>, (unsigned)grid, kTreeThreads, smem, st, p);
  return launch_pdl(tree_kernel<3>, (unsigned)grid, kTreeThreads, smem, st, p);
}

cudaError_t tree_setup_attributes() {
  const int smem = (int)(kWarps * sizeof(WarpSmem));
  cudaError_t e = cudaFuncSetAttribute(tree_kernel<2>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(tree_kernel<3>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(tree_kernel<4>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_tree_blocks_per_sm[0], tree_kernel<2>, kTreeThreads, smem);
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_tree_blocks_per_sm[1], tree_kernel<3>, kTreeThreads, smem);
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_tree_blocks_per_sm[2], tree_kernel<4>, kTreeThreads, smem);
  return e;
}

size_t tree_lmask_words() { return (size_t)kLmWords; }


// Load this file's kernels now (CUDA lazy module loading would otherwise stall the first
// launch of each kernel inside the first checkpoint).
cudaError_t preload_tree() {
  cudaFuncAttributes a;
  cudaError_t e = cudaSuccess;
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, tree_kernel<2>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, tree_kernel<3>);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, tree_kernel<4>);
  return e;
}

}  // namespace ckpt
