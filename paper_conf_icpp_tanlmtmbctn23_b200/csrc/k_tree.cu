// k_tree.cu — Merkle level reduction: phase 2 (Alg.1 l.24-32) and phase 3 (l.33-46).
//
// The paper parallelises Algorithm 1 "level-by-level" in two stages: first the
// sub-trees of first-time occurrences, then those of shifted duplicates. Here
// each stage is a hierarchy of segmented reductions: stage 0 takes a 1024-slot tile of
// the virtual leaf level (R3 geometry, dev.cuh) through t0 levels in shared memory;
// stage s >= 1 takes 1024 stage-(s-1) roots through the next levels. Only tiles/groups
// holding a non-FIXED leaf are visited (worklists built by K1b / phase 2); all others
// are FIXED sub-trees (R7) and cost nothing. All of phase 2 (every stage) finishes
// before any phase-3 lookup (R11), because the phase-3 kernels are launched after the
// last phase-2 kernel on the same stream.
//
// Phase 3 emission ("save roots", R8): a FIRST/SHIFT child of a DONE parent (or a
// FIRST/SHIFT root, R10) becomes a region. Stage 0 records its regions per tile in
// leaf order; an upper-stage region starts at a tile boundary and is recorded in the
// tile holding its first leaf, so the per-tile lists concatenated in tile order are the
// regions sorted by their first chunk (R13) — the compaction (k_compact.cu) relies on it.
#include "kernels.h"

namespace ckpt {

namespace {

struct LeafInfo {
  uint8_t lab;
  Digest d;
  unsigned long long src;
};

// Leaf label after the record insert (Alg.1 l.3-19, R6): FIXED if not a candidate;
// FIRST iff the record's (ckpt, node) for this digest is this very leaf.
__device__ __forceinline__ LeafInfo resolve_leaf(const TreeParams& p, uint64_t c, bool need_digest_first,
                                                 bool need_digest_shift) {
  LeafInfo r;
  r.src = 0;
  const uint32_t w = __ldg(p.cand + (c >> 5));
  if (!((w >> (c & 31)) & 1u)) {
    r.lab = L_FIXED;
    return r;
  }
  const uint32_t slot = __ldg(p.slot_of + c);
  const unsigned long long val = __ldcg(&p.tab[slot].val);
  const unsigned long long own = pack_entry(p.g.k, node_of_chunk(p.g, c));
  r.lab = (val == own) ? L_FIRST : L_SHIFT;
  r.src = val;
  if ((r.lab == L_FIRST && need_digest_first) || (r.lab == L_SHIFT && need_digest_shift)) {
    const ulonglong2 v = __ldg(reinterpret_cast<const ulonglong2*>(p.prev) + c);
    r.d = Digest{v.x, v.y};
  }
  return r;
}

__device__ __forceinline__ void mark_parent(const TreeParams& p, uint64_t G) {
  if (p.last) return;
  const uint64_t P = G >> p.g_next;
  if (atomicExch(&p.dirty_next[P], p.g.epoch) != p.g.epoch) {
    const uint32_t i = atomicAdd(&p.tot->wl_count[p.s + 1], 1u);
    p.wl_next[i] = (uint32_t)P;
  }
}

}  // namespace

// ================================================================= phase 2
// LEAF = stage 0 (tile over the virtual leaf level) / upper stage.
template <bool LEAF>
__global__ void __launch_bounds__(kTreeThreads) phase2_kernel(TreeParams p) {
  __shared__ uint8_t lab[2][1 << kTileLog];
  __shared__ Digest dig[2][1 << kTileLog];
  __shared__ unsigned s_ins, s_coll;
  const int tid = threadIdx.x;
  const Geo& g = p.g;
  const uint32_t count = *(volatile uint32_t*)&p.tot->wl_count[p.wl_slot];
  const int gsz = p.gsz;
  const uint64_t P0 = 1ull << gsz;
  if (tid == 0) { s_ins = 0; s_coll = 0; }
  for (uint32_t w = blockIdx.x; w < count; w += gridDim.x) {
    const uint64_t G = p.wl[w];
    const uint64_t base = G << gsz;
    for (uint32_t q = tid; q < P0; q += kTreeThreads) {
      const uint64_t j = base + q;
      uint8_t L = L_FIXED;
      Digest d{0, 0};
      if (LEAF) {
        if (j < g.m) {
          const LeafInfo li = resolve_leaf(p, j, true, false);
          L = li.lab; d = li.d;
        } else {
          L = L_ABSENT;
        }
      } else if (p.dirty_in[j] == g.epoch) {
        L = p.in.lab2[j];
        if (L == L_FIRST) d = p.in.dig[j];
      }
      lab[0][q] = L;
      if (L == L_FIRST) dig[0][q] = d;
    }
    __syncthreads();
    int cur = 0;
    unsigned ins = 0, coll = 0;
    for (int lv = 1; lv <= gsz; ++lv) {
      const uint32_t cnt = (uint32_t)(P0 >> lv);
      const int Lh = p.Lin + lv;
      for (uint32_t q = tid; q < cnt; q += kTreeThreads) {
        const uint64_t gq = (G << (gsz - lv)) + q;
        uint8_t L;
        Digest d{0, 0};
        if (LEAF && lv == 1 && 2 * gq >= g.m) {          // a leaf of depth h-1 (R3)
          const LeafInfo li = resolve_leaf(p, gq + g.m / 2, true, false);
          L = li.lab; d = li.d;
        } else if (lab[cur][2 * q] == L_FIRST && lab[cur][2 * q + 1] == L_FIRST) {
          // Alg.1 l.26-29: both children first-time -> hash, label, insert (node, chkptID)
          d = mm::node(dig[cur][2 * q], dig[cur][2 * q + 1]);
          bool claimed;
          const uint64_t s = table_find_or_claim(p.tab, p.cap, d, &claimed);
          if (claimed) {
            atomicMin(&p.tab[s].val, pack_entry(g.k, node_id(g, Lh, gq)));
            ++ins;
          } else {
            ++coll;   // R14: a FIRST-FIRST digest already recorded = 128-bit collision
          }
          L = L_FIRST;
        } else {
          L = L_FIXED;   // "not first" is all phase 2 needs
        }
        lab[cur ^ 1][q] = L;
        if (L == L_FIRST) dig[cur ^ 1][q] = d;
      }
      __syncthreads();
      cur ^= 1;
    }
    if (ins) atomicAdd(&s_ins, ins);
    if (coll) atomicAdd(&s_coll, coll);
    if (tid == 0 && !p.last) {
      p.out.lab2[G] = lab[cur][0];
      if (lab[cur][0] == L_FIRST) p.out.dig[G] = dig[cur][0];
      mark_parent(p, G);
    }
    __syncthreads();
  }
  __syncthreads();
  if (tid == 0) {
    if (s_ins) atomicAdd(&p.tot->p2_inserts, (unsigned long long)s_ins);
    if (s_coll) atomicAdd(&p.tot->collisions, (unsigned long long)s_coll);
  }
}

// ================================================================= phase 3
struct P3Smem {
  uint8_t lab[2][1 << kTileLog];
  Digest dig[2][1 << kTileLog];
  unsigned long long src[2][1 << kTileLog];
  // stage-0 emission buffer, indexed by the region's first virtual leaf slot in the tile
  uint8_t emk[1 << kTileLog];
  uint32_t emn[1 << kTileLog];
  unsigned long long ems[1 << kTileLog];
  uint32_t wsum[kTreeThreads / 32];
  uint32_t wsumB[kTreeThreads / 32];
  unsigned long long cls[3];
};

__device__ __forceinline__ uint4 region_rec(uint32_t node, uint8_t kind, unsigned long long src) {
  return make_uint4(node, (uint32_t)(src & 0xffffffffu), (uint32_t)(src >> 32), kind);
}

template <bool LEAF>
__global__ void __launch_bounds__(kTreeThreads) phase3_kernel(TreeParams p) {
  extern __shared__ __align__(16) uint8_t smem_raw[];
  P3Smem& S = *reinterpret_cast<P3Smem*>(smem_raw);
  const int tid = threadIdx.x;
  const Geo& g = p.g;
  const uint32_t count = *(volatile uint32_t*)&p.tot->wl_count[p.wl_slot];
  const int gsz = p.gsz;
  const uint64_t P0 = 1ull << gsz;
  if (tid < 3) S.cls[tid] = 0;
  unsigned long long my_first = 0, my_spat = 0, my_temp = 0;

  for (uint32_t w = blockIdx.x; w < count; w += gridDim.x) {
    const uint64_t G = p.wl[w];
    const uint64_t base = G << gsz;
    for (uint32_t q = tid; q < P0; q += kTreeThreads) {
      const uint64_t j = base + q;
      uint8_t L = L_FIXED;
      Digest d{0, 0};
      unsigned long long src = 0;
      if (LEAF) {
        S.emk[q] = 0;
        if (j < g.m) {
          const LeafInfo li = resolve_leaf(p, j, false, true);
          L = li.lab; d = li.d; src = li.src;
          if (L == L_FIRST) ++my_first;
          else if (L == L_SHIFT) { if ((uint32_t)(src >> 32) == g.k) ++my_spat; else ++my_temp; }
        } else {
          L = L_ABSENT;
        }
      } else if (p.dirty_in[j] == g.epoch) {
        L = p.in.lab3[j];
        if (L == L_SHIFT) { d = p.in.dig[j]; src = p.in.src[j]; }
      }
      S.lab[0][q] = L;
      if (L == L_SHIFT) { S.dig[0][q] = d; S.src[0][q] = src; }
    }
    __syncthreads();

    // emit(v) for v = (height Lc, local position qc) of this group
    auto emit = [&](int lvc, uint32_t qc, uint8_t L, unsigned long long src) {
      if (L != L_FIRST && L != L_SHIFT) return;
      const int Lc = p.Lin + lvc;
      const uint64_t gpos = (G << (gsz - lvc)) + qc;
      const uint32_t node = node_id(g, Lc, gpos);
      if (LEAF) {
        const uint32_t slot = qc << lvc;
        S.emk[slot] = L;
        S.emn[slot] = node;
        S.ems[slot] = src;
      } else {
        const uint64_t tile = (gpos << Lc) >> g.t0;
        uint32_t bytes = 0;
        if (L == L_FIRST) {
          uint64_t lo, hi;
          chunk_range(g, Lc, gpos, lo, hi);
          bytes = (uint32_t)range_bytes(g, lo, hi);
        }
        p.scratch[tile << g.t0] = region_rec(node, L, src);
        p.tilecnt[tile] = make_uint4(L == L_FIRST ? 1u : 0u, L == L_SHIFT ? 1u : 0u, bytes, g.epoch);
      }
    };

    int cur = 0;
    for (int lv = 1; lv <= gsz; ++lv) {
      const uint32_t cnt = (uint32_t)(P0 >> lv);
      const int Lh = p.Lin + lv;
      for (uint32_t q = tid; q < cnt; q += kTreeThreads) {
        const uint64_t gq = (G << (gsz - lv)) + q;
        uint8_t L;
        Digest d{0, 0};
        unsigned long long src = 0;
        if (LEAF && lv == 1 && 2 * gq >= g.m) {          // a leaf of depth h-1 (R3)
          const uint64_t c = gq + g.m / 2;
          const LeafInfo li = resolve_leaf(p, c, false, true);
          L = li.lab; d = li.d; src = li.src;
          if (L == L_FIRST) ++my_first;
          else if (L == L_SHIFT) { if ((uint32_t)(src >> 32) == g.k) ++my_spat; else ++my_temp; }
        } else {
          const uint8_t a = S.lab[cur][2 * q], b = S.lab[cur][2 * q + 1];
          if (a == L_FIRST && b == L_FIRST) {
            L = L_FIRST;                                  // phase-2 sub-tree, skipped (l.33-46 only see the rest)
          } else if (a == L_FIXED && b == L_FIXED) {
            L = L_FIXED;                                  // R7
          } else if (a == L_SHIFT && b == L_SHIFT) {      // Alg.1 l.37-43
            d = mm::node(S.dig[cur][2 * q], S.dig[cur][2 * q + 1]);
            const unsigned long long v = table_lookup(p.tab, p.cap, d);
            if (v != kEmpty) {
              L = L_SHIFT;
              src = v;
            } else {                                      // l.41-42 (R9: not inserted)
              emit(lv - 1, 2 * q, a, S.src[cur][2 * q]);
              emit(lv - 1, 2 * q + 1, b, S.src[cur][2 * q + 1]);
              L = L_DONE;
            }
          } else {                                        // l.35-36, R8
            emit(lv - 1, 2 * q, a, S.src[cur][2 * q]);
            emit(lv - 1, 2 * q + 1, b, S.src[cur][2 * q + 1]);
            L = L_DONE;
          }
          (void)Lh;
        }
        S.lab[cur ^ 1][q] = L;
        if (L == L_SHIFT) { S.dig[cur ^ 1][q] = d; S.src[cur ^ 1][q] = src; }
      }
      __syncthreads();
      cur ^= 1;
    }
    // root of this group
    if (tid == 0) {
      const uint8_t L = S.lab[cur][0];
      if (p.last) {
        emit(gsz, 0, L, S.src[cur][0]);                   // R10
      } else {
        p.out.lab3[G] = L;
        if (L == L_SHIFT) { p.out.dig[G] = S.dig[cur][0]; p.out.src[G] = S.src[cur][0]; }
      }
    }
    __syncthreads();

    if (LEAF) {
      // compact this tile's regions in leaf order -> scratch, counts -> tilecnt
      constexpr int PER = (1 << kTileLog) / kTreeThreads;  // 4 slots per thread
      uint32_t fl[PER];
      uint32_t mine = 0, myb = 0;
      for (int i = 0; i < PER; ++i) {
        const uint32_t slot = tid * PER + i;
        uint32_t f = 0;
        if (slot < P0) {
          const uint8_t k = S.emk[slot];
          if (k == L_FIRST) {
            f = 1u;
            const uint32_t node = S.emn[slot];
            const int depth = 31 - __clz(node + 1);
            const int Lc = g.h - depth;
            uint64_t lo, hi;
            chunk_range(g, Lc, (uint64_t)node + 1 - (1ull << depth), lo, hi);
            myb += (uint32_t)range_bytes(g, lo, hi);
          } else if (k == L_SHIFT) {
            f = 1u << 16;
          }
        }
        fl[i] = f;
        mine += f;
      }
      // block exclusive scan of packed (F count | S count << 16)
      const int lane = tid & 31, wid = tid >> 5;
      uint32_t incl = mine, bsum = myb;
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
      }
      for (int o = 16; o > 0; o >>= 1) bsum += __shfl_xor_sync(0xffffffffu, bsum, o);
      if (lane == 31) S.wsum[wid] = incl;
      if (lane == 0) S.wsumB[wid] = bsum;
      __syncthreads();
      uint32_t woff = 0, tot = 0, totB = 0;
      for (int i = 0; i < kTreeThreads / 32; ++i) {
        if (i < wid) woff += S.wsum[i];
        tot += S.wsum[i];
        totB += S.wsumB[i];
      }
      const uint32_t nF = tot & 0xffffu, nS = tot >> 16;
      uint32_t run = woff + incl - mine;
      for (int i = 0; i < PER; ++i) {
        const uint32_t slot = tid * PER + i;
        if (fl[i]) {
          const uint32_t fidx = run & 0xffffu, sidx = run >> 16;
          // FIRST records first, then SHIFT records, each in leaf order
          const uint32_t idx = (fl[i] == 1u) ? fidx : nF + sidx;
          p.scratch[(G << gsz) + idx] = region_rec(S.emn[slot], S.emk[slot], S.ems[slot]);
        }
        run += fl[i];
      }
      if (tid == 0) p.tilecnt[G] = make_uint4(nF, nS, totB, g.epoch);
      __syncthreads();
    }
  }
  if (LEAF) {
    for (int o = 16; o > 0; o >>= 1) {
      my_first += __shfl_xor_sync(0xffffffffu, my_first, o);
      my_spat += __shfl_xor_sync(0xffffffffu, my_spat, o);
      my_temp += __shfl_xor_sync(0xffffffffu, my_temp, o);
    }
    if ((tid & 31) == 0) {
      if (my_first) atomicAdd(&S.cls[0], my_first);
      if (my_spat) atomicAdd(&S.cls[1], my_spat);
      if (my_temp) atomicAdd(&S.cls[2], my_temp);
    }
    __syncthreads();
    if (tid == 0) {
      if (S.cls[0]) atomicAdd(&p.tot->n_first, S.cls[0]);
      if (S.cls[1]) atomicAdd(&p.tot->n_spatial, S.cls[1]);
      if (S.cls[2]) atomicAdd(&p.tot->n_temporal, S.cls[2]);
    }
  }
}

// ================================================================= launchers
static unsigned tree_grid(uint64_t n_groups, int num_sms) {
  uint64_t gmax = (uint64_t)num_sms * 4;
  return (unsigned)(n_groups < gmax ? (n_groups ? n_groups : 1) : gmax);
}

cudaError_t launch_phase2(const TreeParams& p, uint64_t n_groups, int num_sms, cudaStream_t st) {
  const unsigned grid = tree_grid(n_groups, num_sms);
  if (p.s == 0) phase2_kernel<true><<<grid, kTreeThreads, 0, st>>>(p);
  else phase2_kernel<false><<<grid, kTreeThreads, 0, st>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_phase3(const TreeParams& p, uint64_t n_groups, int num_sms, cudaStream_t st) {
  const unsigned grid = tree_grid(n_groups, num_sms);
  const size_t smem = sizeof(P3Smem);
  if (p.s == 0) {
    cudaFuncSetAttribute(phase3_kernel<true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    phase3_kernel<true><<<grid, kTreeThreads, smem, st>>>(p);
  } else {
    cudaFuncSetAttribute(phase3_kernel<false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    phase3_kernel<false><<<grid, kTreeThreads, smem, st>>>(p);
  }
  return cudaGetLastError();
}

}  // namespace ckpt
