// k_tree.cu — Merkle level reduction: phase 2 (Alg.1 l.24-32) and phase 3 (l.33-46).
//
// The paper parallelises Algorithm 1 "level-by-level" in two stages: first the
// sub-trees of first-time occurrences, then those of shifted duplicates. Here
// each stage is ONE kernel launch (all of phase 2 finishes before any phase-3 lookup,
// R11, because the phase-3 kernel is launched after the phase-2 kernel on one stream).
//
// Work unit: one WARP per group of up to 1024 positions of one height (a stage-0 tile
// of the virtual leaf level, R3 geometry in dev.cuh, or 1024 roots of the stage below).
// The labels of a level are bitmasks — lane w holds positions 32w..32w+31 of each class
// (FIRST, SHIFT, FIXED) — so a level step is two shuffles and an even/odd bit split:
// a parent is FIRST iff both children are, FIXED iff both are (R7), "SHIFT pair" iff both
// are SHIFT, otherwise DONE (mixed). Only the set bits that need a digest (phase 2:
// FIRST pairs -> hash + insert, Alg.1 l.28-29; phase 3: SHIFT pairs -> hash + lookup,
// l.38-39) do memory work, spread evenly over the 32 lanes. Groups holding no
// non-FIXED leaf are never visited (K1b builds the stage-0 worklist and counts dirty
// children per upper group); the warp that finishes the LAST dirty child of an upper
// group climbs and processes that group too, so every stage runs in the same launch.
//
// Phase-3 emission ("save roots", R8/R10): a FIRST/SHIFT child of a DONE parent (or the
// FIRST/SHIFT root) becomes a region. Stage 0 records its regions per tile in leaf
// order (FIRST list, then SHIFT list); an upper-stage region starts at a tile boundary
// and is recorded in the tile holding its first leaf, so the per-tile lists in tile
// order are the regions sorted by first chunk (R13) — k_compact.cu relies on it.
#include "kernels.h"

namespace ckpt {

namespace {

constexpr int kWarps = kTreeThreads / 32;

// ------------------------------------------------------------------ bit helpers
__device__ __forceinline__ uint32_t even_bits64(uint64_t x) {   // bits 0,2,...,62 -> 0..31
  x &= 0x5555555555555555ull;
  x = (x | (x >> 1)) & 0x3333333333333333ull;
  x = (x | (x >> 2)) & 0x0F0F0F0F0F0F0F0Full;
  x = (x | (x >> 4)) & 0x00FF00FF00FF00FFull;
  x = (x | (x >> 8)) & 0x0000FFFF0000FFFFull;
  x = (x | (x >> 16)) & 0x00000000FFFFFFFFull;
  return (uint32_t)x;
}
__device__ __forceinline__ uint32_t spread16(uint32_t x) {      // bit i -> bits 2i and 2i+1
  x &= 0xFFFFu;
  x = (x | (x << 8)) & 0x00FF00FFu;
  x = (x | (x << 4)) & 0x0F0F0F0Fu;
  x = (x | (x << 2)) & 0x33333333u;
  x = (x | (x << 1)) & 0x55555555u;
  return x | (x << 1);
}
__device__ __forceinline__ uint32_t low_mask(uint64_t nbits) { return nbits >= 32 ? 0xFFFFFFFFu : ((1u << nbits) - 1u); }

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
  uint32_t pw[32];      // words of the current work mask
  uint32_t px[32];      // exclusive prefix of their popcounts
  uint32_t hitF[32];    // result bits written by work items (FIRST / lookup hit)
  uint32_t hitS[32];    // result bits (SHIFT leaves)
  uint32_t stF[32];     // stage-0 emission: FIRST region start slots
  uint32_t stS[32];     //                   SHIFT region start slots
  uint8_t lvl[1 << kTileLog];   // level of the region starting at each slot
};

// Balanced distribution of the set bits of per-lane words `m` (word index = lane) over
// the 32 lanes: calls f(word, bit, position) once per set bit.
template <class F>
__device__ __forceinline__ void for_each_bit_balanced(WarpSmem& ws, uint32_t m, F&& f) {
  const int lane = threadIdx.x & 31;
  const uint32_t cnt = __popc(m);
  uint32_t incl = cnt;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  if (total == 0) return;
  ws.pw[lane] = m;
  ws.px[lane] = incl - cnt;
  __syncwarp();
  for (uint32_t base = 0; base < total; base += 32) {
    const uint32_t j = base + lane;
    if (j < total) {
      int lo = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1)
        if (lo + step < 32 && ws.px[lo + step] <= j) lo += step;
      const uint32_t b = __fns(ws.pw[lo], 0, (int)(j - ws.px[lo]) + 1);
      f((uint32_t)lo, b, (uint32_t)lo * 32 + b);
    }
  }
  __syncwarp();
}

__device__ __forceinline__ uint64_t lvl_off(uint64_t P0, int lv) { return P0 - (P0 >> (lv - 1)); }  // lv >= 1

struct Ctx {
  const TreeParams* p;
  int s;             // stage
  uint64_t G;        // group index
  int Lin, gsz;
  uint64_t P0;       // positions at the input height
  bool leaf;         // stage 0
  Digest* tdig;      // this group's internal digests (P0 entries)
  unsigned long long* tsrc;   // this group's sources (2 P0 entries: level 0, then internal)
};

// digest of the child at (lv, pos) of the current group
__device__ __forceinline__ Digest child_digest(const Ctx& c, int lv, uint64_t pos) {
  const TreeParams& p = *c.p;
  if (lv == 0) {
    if (c.leaf) {
      const ulonglong2 v = __ldg(reinterpret_cast<const ulonglong2*>(p.prev) + ((c.G << c.gsz) + pos));
      return Digest{v.x, v.y};
    }
    const ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2*>(p.st[c.s].in.dig) + ((c.G << c.gsz) + pos));
    return Digest{v.x, v.y};
  }
  if (lv == 1 && c.leaf) {
    const uint64_t gq = (c.G << (c.gsz - 1)) + pos;
    if (2 * gq >= p.g.m) {
      const ulonglong2 v = __ldg(reinterpret_cast<const ulonglong2*>(p.prev) + (gq + p.g.m / 2));
      return Digest{v.x, v.y};
    }
  }
  const ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2*>(c.tdig) + (lvl_off(c.P0, lv) + pos));
  return Digest{v.x, v.y};
}

__device__ __forceinline__ unsigned long long child_src(const Ctx& c, int lv, uint64_t pos) {
  const TreeParams& p = *c.p;
  if (lv == 0) {
    if (c.leaf) return __ldcg(c.tsrc + pos);
    return __ldcg(p.st[c.s].in.src + ((c.G << c.gsz) + pos));
  }
  return __ldcg(c.tsrc + c.P0 + lvl_off(c.P0, lv) + pos);
}

// Leaf labels of a chunk range mapped onto one level's words (stage 0, phase 2): every
// candidate is resolved against the record (R6: FIRST iff the record's entry is this
// leaf; otherwise SHIFT with that entry as its source), the rest are FIXED. Sets masks
// F/S/X (lane word) for positions [0, npos); SHIFT sources go to tsrc[src_base + pos].
// The leaf classes (first / spatial / temporal) are counted here.
struct LeafCount {
  uint32_t f, s, t;
};

__device__ __forceinline__ void resolve_leaves(const Ctx& c, WarpSmem& ws, uint64_t chunk0, uint64_t npos,
                                               uint64_t src_base, uint32_t& F, uint32_t& S, uint32_t& X,
                                               LeafCount& lc) {
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
  for_each_bit_balanced(ws, cand, [&](uint32_t w, uint32_t b, uint32_t pos) {
    const uint64_t ch = chunk0 + pos;
    const uint32_t slot = __ldg(p.slot_of + ch);
    const unsigned long long val = __ldcg(&p.tab[slot].val);
    if (val == pack_entry(k, node_of_chunk(p.g, ch))) {
      atomicOr(&ws.hitF[w], 1u << b);
      ++lc.f;
    } else {
      atomicOr(&ws.hitS[w], 1u << b);
      c.tsrc[src_base + pos] = val;
      if ((uint32_t)(val >> 32) == k) ++lc.s; else ++lc.t;
    }
  });
  F = ws.hitF[lane];
  S = ws.hitS[lane];
  X = valid & ~cand;
}

// Phase-2 record insert of a FIRST-FIRST node (Alg.1 l.29): the key is new, so the CAS
// claim of an empty slot settles it; the value is then written plainly.
__device__ __forceinline__ bool insert_new(Slot* tab, uint64_t cap, const Digest& d, unsigned long long packed) {
  uint64_t s = slot_home(d.lo, cap);
  for (;;) {
    unsigned long long olo, ohi;
    cas128(tab + s, kEmpty, kEmpty, d.lo, d.hi, olo, ohi);
    if (olo == kEmpty && ohi == kEmpty) {
      tab[s].val = packed;
      return true;
    }
    if (olo == d.lo && ohi == d.hi) return false;   // already recorded: a collision (R14)
    if (++s == cap) s = 0;
  }
}

// Emit the region (lv, pos) of the current group (phase 3).
__device__ __forceinline__ void emit_region(const Ctx& c, WarpSmem& ws, int lv, uint64_t pos, bool first,
                                           unsigned long long src) {
  const TreeParams& p = *c.p;
  if (c.leaf) {
    const uint32_t slot = (uint32_t)(pos << lv);
    atomicOr(first ? &ws.stF[slot >> 5] : &ws.stS[slot >> 5], 1u << (slot & 31));
    ws.lvl[slot] = (uint8_t)lv;
    return;
  }
  const int Lc = c.Lin + lv;
  const uint64_t gpos = (c.G << (c.gsz - lv)) + pos;
  const uint32_t node = node_id(p.g, Lc, gpos);
  const uint64_t tile = (gpos << Lc) >> p.g.t0;
  uint32_t bytes = 0;
  if (first) {
    uint64_t lo, hi;
    chunk_range(p.g, Lc, gpos, lo, hi);
    bytes = (uint32_t)range_bytes(p.g, lo, hi);
  }
  p.scratch[tile << p.g.t0] = make_uint4(node, (uint32_t)(src & 0xffffffffu), (uint32_t)(src >> 32),
                                         first ? L_FIRST : L_SHIFT);
  p.tilecnt[tile] = make_uint4(first ? 1u : 0u, first ? 0u : 1u, bytes, p.g.epoch);
}

// Process one group through its gsz levels. PHASE 2 or 3.
template <int PHASE>
__device__ void process_group(const Ctx& c, WarpSmem& ws, unsigned long long& ins_cnt, unsigned long long& coll_cnt,
                              LeafCount& lc) {
  const TreeParams& p = *c.p;
  const Geo& g = p.g;
  const int lane = threadIdx.x & 31;
  const uint64_t P0 = c.P0;
  uint32_t F = 0, S = 0, X = 0;    // current level's masks (lane word)
  uint32_t* lm = c.leaf ? p.lmask + (c.G << 7) : nullptr;   // per tile: F0 S0 F1 S1 (32 words each)

  // ---- input level
  if (c.leaf) {
    const uint64_t base = c.G << c.gsz;
    const uint64_t npos0 = base < g.m ? (g.m - base < P0 ? g.m - base : P0) : 0;   // real leaves at height 0
    if (PHASE == 2) {
      resolve_leaves(c, ws, base, npos0, 0, F, S, X, lc);
      lm[lane] = F;
      lm[32 + lane] = S;
    } else {
      const uint32_t valid = ((uint64_t)lane * 32 < npos0) ? low_mask(npos0 - (uint64_t)lane * 32) : 0u;
      F = __ldcg(lm + lane);
      S = __ldcg(lm + 32 + lane);
      X = valid & ~(F | S);
      ws.stF[lane] = 0;
      ws.stS[lane] = 0;
    }
  } else {
    // 32 positions per lane: dirty marks (128 B) and labels (32 B) as vector loads
    const StageParams& sp = p.st[c.s];
    const uint64_t j0 = (c.G << c.gsz) + (uint64_t)lane * 32;
    const uint8_t* labs = PHASE == 2 ? sp.in.lab2 : sp.in.lab3;
    if (P0 >= 32) {
      uint4 dv[8], lv2[2];
#pragma unroll
      for (int i = 0; i < 8; ++i) dv[i] = __ldcg(reinterpret_cast<const uint4*>(sp.dirty_in + j0) + i);
#pragma unroll
      for (int i = 0; i < 2; ++i) lv2[i] = __ldcg(reinterpret_cast<const uint4*>(labs + j0) + i);
      const uint32_t* dw = reinterpret_cast<const uint32_t*>(dv);
      const uint8_t* lb = reinterpret_cast<const uint8_t*>(lv2);
#pragma unroll
      for (int b = 0; b < 32; ++b) {
        const uint8_t L = (dw[b] == g.epoch) ? lb[b] : (uint8_t)L_FIXED;
        F |= (uint32_t)(L == L_FIRST) << b;
        S |= (uint32_t)(L == L_SHIFT) << b;
        X |= (uint32_t)(L == L_FIXED) << b;
      }
    } else if (lane == 0) {
      for (uint32_t b = 0; b < P0; ++b) {
        const uint8_t L = (__ldcg(sp.dirty_in + j0 + b) == g.epoch) ? __ldcg(labs + j0 + b) : (uint8_t)L_FIXED;
        F |= (uint32_t)(L == L_FIRST) << b;
        S |= (uint32_t)(L == L_SHIFT) << b;
        X |= (uint32_t)(L == L_FIXED) << b;
      }
    }
  }
  __syncwarp();

  // ---- levels
  for (int lv = 1; lv <= c.gsz; ++lv) {
    const uint64_t Nc = P0 >> (lv - 1), Np = Nc >> 1;
    uint32_t eF, oF, eS, oS, eX, oX;
    if (Nc > 32) {
      const int s0 = (2 * lane) & 31, s1 = (2 * lane + 1) & 31;
      const uint32_t fl = __shfl_sync(0xffffffffu, F, s0), fh = __shfl_sync(0xffffffffu, F, s1);
      const uint32_t sl = __shfl_sync(0xffffffffu, S, s0), sh = __shfl_sync(0xffffffffu, S, s1);
      const uint32_t xl = __shfl_sync(0xffffffffu, X, s0), xh = __shfl_sync(0xffffffffu, X, s1);
      const uint64_t f64 = (uint64_t)fl | ((uint64_t)fh << 32);
      const uint64_t s64 = (uint64_t)sl | ((uint64_t)sh << 32);
      const uint64_t x64 = (uint64_t)xl | ((uint64_t)xh << 32);
      eF = even_bits64(f64); oF = even_bits64(f64 >> 1);
      eS = even_bits64(s64); oS = even_bits64(s64 >> 1);
      eX = even_bits64(x64); oX = even_bits64(x64 >> 1);
    } else {
      const uint32_t f = __shfl_sync(0xffffffffu, F, 0), s = __shfl_sync(0xffffffffu, S, 0),
                     x = __shfl_sync(0xffffffffu, X, 0);
      eF = even_bits64(f); oF = even_bits64(f >> 1);
      eS = even_bits64(s); oS = even_bits64(s >> 1);
      eX = even_bits64(x); oX = even_bits64(x >> 1);
    }
    const uint32_t valid = ((uint64_t)lane * 32 < Np) ? low_mask(Np - (uint64_t)lane * 32) : 0u;
    const uint32_t bothF = eF & oF & valid;
    const uint32_t bothX = eX & oX & valid;
    const uint32_t bothS = eS & oS & valid;
    const uint64_t pbase = c.G << (c.gsz - lv);     // global position of this level's first node

    // height-1 leaves of depth h-1 (R3): their labels come from the record, not children
    uint32_t leafm = 0, lF = 0, lS = 0, lX = 0;
    if (c.leaf && lv == 1) {
      const uint64_t first_leaf = (g.m / 2 > pbase) ? g.m / 2 - pbase : 0;   // local position
      if (first_leaf < Np) {
        const uint64_t q0 = (uint64_t)lane * 32;
        if (q0 + 32 > first_leaf && q0 < Np) {
          const uint64_t lo = first_leaf > q0 ? first_leaf - q0 : 0;
          leafm = valid & ~low_mask(lo);
        }
        if (PHASE == 2) {
          // resolve chunks gq + m/2 for local positions [first_leaf, Np); sources land at
          // tsrc[P0 + off(1) + pos]
          uint32_t tF, tS, tX;
          resolve_leaves(c, ws, pbase + first_leaf + g.m / 2, Np - first_leaf, c.P0 + lvl_off(c.P0, 1) + first_leaf,
                         tF, tS, tX, lc);
          // realign: resolve_leaves numbered positions from first_leaf
          const uint32_t sh = (uint32_t)(first_leaf & 31);
          const int wsrc = (int)(first_leaf >> 5);
          auto realign = [&](uint32_t m) {
            const int a = lane - wsrc;
            const uint32_t cur = __shfl_sync(0xffffffffu, m, a < 0 ? 0 : (a & 31));
            const uint32_t prv = __shfl_sync(0xffffffffu, m, (a - 1) < 0 ? 0 : ((a - 1) & 31));
            uint32_t r = 0;
            if (a >= 0) r = cur << sh;
            if (a >= 1 && sh) r |= prv >> (32 - sh);
            return r & leafm;
          };
          lF = realign(tF);
          lS = realign(tS);
          lm[64 + lane] = lF;
          lm[96 + lane] = lS;
        } else {
          lF = __ldcg(lm + 64 + lane);
          lS = __ldcg(lm + 96 + lane);
        }
        lX = leafm & ~(lF | lS);
      }
    }

    uint32_t nF, nS, nX, nD;
    if (PHASE == 2) {
      // Alg.1 l.24-32: FIRST pairs -> hash, label FIRST, insert (node, chkptID)
      const uint32_t work = bothF & ~leafm;
      for_each_bit_balanced(ws, work, [&](uint32_t, uint32_t, uint32_t q) {
        const Digest d = mm::node(child_digest(c, lv - 1, 2 * (uint64_t)q), child_digest(c, lv - 1, 2 * (uint64_t)q + 1));
        if (insert_new(p.tab, p.cap, d, pack_entry(g.k, node_id(g, c.Lin + lv, pbase + q)))) ++ins_cnt;
        else ++coll_cnt;   // R14: a FIRST-FIRST digest already in the record = 128-bit collision
        reinterpret_cast<ulonglong2*>(c.tdig)[lvl_off(P0, lv) + q] = make_ulonglong2(d.lo, d.hi);
      });
      nF = (work) | lF;
      nS = 0; nX = 0; nD = 0;
      (void)lS; (void)lX;
    } else {
      // Alg.1 l.33-46 on non-FIRST nodes
      const uint32_t work = bothS & ~leafm;
      ws.hitF[lane] = 0;
      __syncwarp();
      for_each_bit_balanced(ws, work, [&](uint32_t w, uint32_t b, uint32_t q) {
        const Digest d = mm::node(child_digest(c, lv - 1, 2 * (uint64_t)q), child_digest(c, lv - 1, 2 * (uint64_t)q + 1));
        const unsigned long long v = table_lookup(p.tab, p.cap, d);
        if (v != kEmpty) {
          atomicOr(&ws.hitF[w], 1u << b);
          reinterpret_cast<ulonglong2*>(c.tdig)[lvl_off(P0, lv) + q] = make_ulonglong2(d.lo, d.hi);
          c.tsrc[P0 + lvl_off(P0, lv) + q] = v;
        }
      });
      const uint32_t hit = ws.hitF[lane];
      nF = (bothF & ~leafm) | lF;
      nX = (bothX & ~leafm) | lX;
      nS = hit | lS;
      nD = valid & ~leafm & ~bothF & ~bothX & ~hit;
      // emission of the children of DONE parents: spread parent bits onto child words
      uint32_t dchild;
      if (Nc > 32) {
        const uint32_t dp = __shfl_sync(0xffffffffu, nD, lane >> 1);
        dchild = spread16((lane & 1) ? (dp >> 16) : dp);
      } else {
        const uint32_t dp = __shfl_sync(0xffffffffu, nD, 0);
        dchild = lane == 0 ? spread16(dp) : 0u;
      }
      const uint32_t emF = dchild & F, emS = dchild & S;
      for (uint32_t m = emF | emS; m; m &= m - 1) {
        const uint32_t b = __ffs(m) - 1;
        const uint64_t pos = (uint64_t)lane * 32 + b;
        const bool isF = (emF >> b) & 1u;
        emit_region(c, ws, lv - 1, pos, isF, isF ? 0ull : child_src(c, lv - 1, pos));
      }
      __syncwarp();
    }
    F = nF; S = nS; X = nX;
    (void)nD;
  }

  // ---- group root (single position at level gsz, lane 0 bit 0)
  const uint32_t rF = __shfl_sync(0xffffffffu, F, 0) & 1u;
  const uint32_t rS = __shfl_sync(0xffffffffu, S, 0) & 1u;
  const uint32_t rX = __shfl_sync(0xffffffffu, X, 0) & 1u;
  const bool last = (c.s == p.S - 1);
  if (last) {
    if (PHASE == 3 && lane == 0 && (rF | rS))
      emit_region(c, ws, c.gsz, 0, rF != 0, rS ? child_src(c, c.gsz, 0) : 0ull);   // R10
  } else if (lane == 0) {
    const StageParams& nx = p.st[c.s + 1];
    uint8_t L;
    if (PHASE == 2) {
      L = rF ? L_FIRST : L_FIXED;
      nx.in.lab2[c.G] = L;
      if (rF) {
        const Digest d = child_digest(c, c.gsz, 0);
        reinterpret_cast<ulonglong2*>(nx.in.dig)[c.G] = make_ulonglong2(d.lo, d.hi);
      }
    } else {
      L = rF ? L_FIRST : (rS ? L_SHIFT : (rX ? L_FIXED : L_DONE));
      nx.in.lab3[c.G] = L;
      if (rS) {
        const Digest d = child_digest(c, c.gsz, 0);
        reinterpret_cast<ulonglong2*>(nx.in.dig)[c.G] = make_ulonglong2(d.lo, d.hi);
        nx.in.src[c.G] = child_src(c, c.gsz, 0);
      }
    }
  }
  __syncwarp();

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
    uint32_t rf = iF - __popc(wF), rs = nFt + iS - __popc(wS);
    uint32_t bytes = 0;
    uint4* out = p.scratch + (c.G << g.t0);
    for (uint32_t m = wF; m; m &= m - 1) {
      const uint32_t b = __ffs(m) - 1;
      const uint32_t slot = lane * 32 + b;
      const int lv = ws.lvl[slot];
      const uint64_t gpos = (c.G << (c.gsz - lv)) + (slot >> lv);
      uint64_t lo, hi;
      chunk_range(g, lv, gpos, lo, hi);
      bytes += (uint32_t)range_bytes(g, lo, hi);
      out[rf++] = make_uint4(node_id(g, lv, gpos), 0u, 0u, L_FIRST);
    }
    for (uint32_t m = wS; m; m &= m - 1) {
      const uint32_t b = __ffs(m) - 1;
      const uint32_t slot = lane * 32 + b;
      const int lv = ws.lvl[slot];
      const uint64_t gpos = (c.G << (c.gsz - lv)) + (slot >> lv);
      const unsigned long long src = child_src(c, lv, slot >> lv);
      out[rs++] = make_uint4(node_id(g, lv, gpos), (uint32_t)(src & 0xffffffffu), (uint32_t)(src >> 32), L_SHIFT);
    }
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) bytes += __shfl_xor_sync(0xffffffffu, bytes, o);
    if (lane == 0) p.tilecnt[c.G] = make_uint4(nFt, nSt, bytes, g.epoch);
    __syncwarp();
  }
}

}  // namespace

// ================================================================= kernel
template <int PHASE>
__global__ void __launch_bounds__(kTreeThreads) tree_kernel(const __grid_constant__ TreeParams p) {
  __shared__ WarpSmem sm[kWarps];
  __shared__ unsigned long long s_cnt[4];
  LeafCount lc{0, 0, 0};
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  WarpSmem& ws = sm[wid];
  if (threadIdx.x < 4) s_cnt[threadIdx.x] = 0;
  __syncthreads();
  unsigned long long ins = 0, coll = 0;
  const uint32_t count = *(volatile uint32_t*)&p.tot->wl_count[0];
  unsigned* next = &p.tot->tree_next[PHASE - 2];
  for (;;) {
    uint32_t w = 0;
    if (lane == 0) w = atomicAdd(next, 1u);
    w = __shfl_sync(0xffffffffu, w, 0);
    if (w >= count) break;
    Ctx c;
    c.p = &p;
    c.s = 0;
    c.G = p.wl0[w];
    c.Lin = 0;
    c.gsz = p.st[0].gsz;
    c.P0 = 1ull << c.gsz;
    c.leaf = true;
    c.tdig = p.st[0].tdig + (c.G << c.gsz);
    c.tsrc = p.st[0].tsrc + ((c.G << c.gsz) << 1);
    process_group<PHASE>(c, ws, ins, coll, lc);
    // climb: the warp finishing the last dirty child of a group processes that group
    while (c.s < p.S - 1) {
      const StageParams& up = p.st[c.s + 1];
      const uint64_t P = c.G >> up.gsz;
      uint32_t old = 0;
      __threadfence();
      if (lane == 0) old = atomicAdd((PHASE == 2 ? up.done2 : up.done3) + P, 1u);
      old = __shfl_sync(0xffffffffu, old, 0);
      const uint32_t need = __ldcg(up.cnt + P);
      if (old + 1 != need) break;
      __threadfence();
      c.s += 1;
      c.G = P;
      c.Lin = up.Lin;
      c.gsz = up.gsz;
      c.P0 = 1ull << c.gsz;
      c.leaf = false;
      c.tdig = up.tdig + (P << c.gsz);
      c.tsrc = up.tsrc + ((P << c.gsz) << 1);
      process_group<PHASE>(c, ws, ins, coll, lc);
    }
  }
  if (ins) atomicAdd(&s_cnt[3], ins);
  if (PHASE == 2 && coll) atomicAdd(&p.tot->collisions, coll);
  if (PHASE == 2) {
    if (lc.f) atomicAdd(&s_cnt[0], (unsigned long long)lc.f);
    if (lc.s) atomicAdd(&s_cnt[1], (unsigned long long)lc.s);
    if (lc.t) atomicAdd(&s_cnt[2], (unsigned long long)lc.t);
  }
  __syncthreads();
  if (threadIdx.x == 0 && PHASE == 2) {
    if (s_cnt[3]) atomicAdd(&p.tot->p2_inserts, s_cnt[3]);
    if (s_cnt[0]) atomicAdd(&p.tot->n_first, s_cnt[0]);
    if (s_cnt[1]) atomicAdd(&p.tot->n_spatial, s_cnt[1]);
    if (s_cnt[2]) atomicAdd(&p.tot->n_temporal, s_cnt[2]);
  }
}

cudaError_t launch_tree(const TreeParams& p, int phase, int num_sms, cudaStream_t st) {
  uint64_t grid = (uint64_t)num_sms * 8;
  const uint64_t need = (p.n_tiles + kWarps - 1) / kWarps;
  if (grid > need) grid = need ? need : 1;
  if (phase == 2) tree_kernel<2><<<(unsigned)grid, kTreeThreads, 0, st>>>(p);
  else tree_kernel<3><<<(unsigned)grid, kTreeThreads, 0, st>>>(p);
  return cudaGetLastError();
}

}  // namespace ckpt
