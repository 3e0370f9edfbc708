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
//     32 candidate-mask words, warp-level de-duplication of equal digests (__match_any)
//     so a hot key (e.g. all-zero chunks) costs one atomic per warp; marks stage-0
//     tiles dirty and appends them to the phase-2/3 worklist.
#include "kernels.h"
#include "tma.cuh"

namespace ckpt {

// ------------------------------------------------------------------ shared epilogue
// Fixed test (Alg.1 l.3-4) and digest update (l.21) for chunk c with digest d.
__device__ __forceinline__ bool leaf_is_candidate(const Geo& g, const Digest& d, const Digest& prevd) {
  return !(g.k > 0 && d == prevd);
}

// ------------------------------------------------------------------ K1
template <int MODE3D>
__global__ void __launch_bounds__(kLeafThreads, 2) leaf_hash_kernel(const __grid_constant__ CUtensorMap tmap, LeafParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-B alignment for the 128B swizzle atom, kept as a shared-space pointer (LDS, not LD)
  const uint32_t pad = (1024u - (smem_u32(smem_raw) & 1023u)) & 1023u;
  uint8_t* const data = smem_raw + pad;                                    // nst * stage_bytes
  const int nst = p.nst;
  const uint32_t stage_bytes = p.stage_bytes;
  Digest* const prevbuf = reinterpret_cast<Digest*>(data + nst * stage_bytes);   // nst * 256 digests
  uint64_t* const bars = reinterpret_cast<uint64_t*>(prevbuf + nst * kLeafThreads);

  const int tid = threadIdx.x;
  const uint32_t n_tiles = (uint32_t)(p.n_main / kLeafThreads);
  const int segs = p.segs;
  const uint32_t my_tiles = (blockIdx.x < n_tiles) ? (n_tiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  const uint32_t total = my_tiles * (uint32_t)segs;
  const bool use_prev = p.g.k > 0;

  pdl_launch_dependents();
  if (tid == 0) {
    prefetch_tmap(&tmap);
    for (int s = 0; s < nst; ++s) mbar_init(&bars[s], 1);
    fence_mbar_init();
  }
  __syncthreads();

  // producer state (thread 0): next step to issue, as (stage, tile, seg) counters
  int is_st = 0, is_seg = 0;
  uint32_t is_tile = blockIdx.x, issued = 0;
  const uint64_t pol_stream = policy_evict_first();
  const uint64_t pol_keep = policy_evict_last();
  auto issue_next = [&]() {
    const bool with_prev = use_prev && is_seg == segs - 1;
    mbar_arrive_expect_tx(&bars[is_st], stage_bytes + (with_prev ? kLeafThreads * 16u : 0u));
    if (MODE3D)
      tma_load_3d(data + (size_t)is_st * stage_bytes, &tmap, &bars[is_st], 0, is_seg, (int)(is_tile * kLeafThreads),
                  pol_stream);
    else
      tma_load_2d(data + (size_t)is_st * stage_bytes, &tmap, &bars[is_st], 0, (int)(is_tile * (stage_bytes / 128)),
                  pol_stream);
    if (with_prev)
      bulk_load(prevbuf + is_st * kLeafThreads, p.prev + (uint64_t)is_tile * kLeafThreads, kLeafThreads * 16u, &bars[is_st],
                pol_stream);
    ++issued;
    if (++is_st == nst) is_st = 0;
    if (++is_seg == segs) { is_seg = 0; is_tile += gridDim.x; }
  };
  if (tid == 0)
    while (issued < (uint32_t)nst && issued < total) issue_next();

  const int units = MODE3D ? 8 : (int)(p.g.C / 16);   // 16-byte blocks of this thread per stage
  const uint32_t ubase = (uint32_t)tid * (uint32_t)units;
  uint64_t h1 = 0, h2 = 0;
  int st = 0, seg = 0;
  uint32_t phase = 0, tile = blockIdx.x;
  for (uint32_t step = 0; step < total; ++step) {
    mbar_wait(&bars[st], phase);
    if (seg == 0) { h1 = 0; h2 = 0; }   // seed 0 (R1)
    const uint8_t* sd = data + (size_t)st * stage_bytes;
#pragma unroll 8
    for (int j = 0; j < units; ++j) {
      const uint32_t u = ubase + j;
      const uint32_t row = u >> 3;
      const uint32_t off = (row << 7) | ((((u & 7) ^ (row & 7))) << 4);   // SWIZZLE_128B
      const ulonglong2 v = *reinterpret_cast<const ulonglong2*>(sd + off);
      mm::block(h1, h2, v.x, v.y);
    }
    if (seg == segs - 1) {
      const Digest d = mm::finish(h1, h2, p.g.C);
      const uint64_t c = (uint64_t)tile * kLeafThreads + tid;
      Digest pd{0, 0};
      if (use_prev) pd = prevbuf[st * kLeafThreads + tid];
      const bool cand = leaf_is_candidate(p.g, d, pd);
      const unsigned mask = __ballot_sync(0xffffffffu, cand);
      if ((tid & 31) == 0) st_evict_last_u32(p.cand + (c >> 5), mask, pol_keep);
      if (cand) st_evict_last_v2(p.prev + c, d.lo, d.hi, pol_keep);
    }
    __syncthreads();   // every thread is done with stage st
    if (tid == 0 && issued < total) issue_next();
    if (++st == nst) { st = 0; phase ^= 1u; }
    if (++seg == segs) { seg = 0; tile += gridDim.x; }
  }
}

// ------------------------------------------------------------------ K1t
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
  const unsigned mask = __ballot_sync(0xffffffffu, cand);
  if ((threadIdx.x & 31) == 0 && c < p.g.n) p.cand[c >> 5] = mask;
  if (cand) reinterpret_cast<ulonglong2*>(p.prev)[c] = make_ulonglong2(d.lo, d.hi);
}

// ------------------------------------------------------------------ K1b
// One warp per 32 candidate-mask words (1024 chunks). The warp's candidates are spread
// evenly over its lanes (warp prefix over popcounts; lane j takes candidate j, j+32, ...)
// so a clustered run of changed chunks costs ceil(count/32) dependent insert chains, not
// one chain per candidate of the densest word.
__global__ void __launch_bounds__(256) insert_kernel(InsertParams p) {
  pdl_launch_dependents();
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  const uint64_t warp = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
  const uint64_t wbase = warp * 32;                 // first mask word of this warp
  __shared__ uint32_t s_cnt, s_base;
  __shared__ uint32_t s_tiles[256];
  __shared__ uint32_t s_word[8][32], s_excl[8][32];
  if (threadIdx.x == 0) s_cnt = 0;
  __syncthreads();
  pdl_wait();

  const uint32_t word = (wbase + lane < p.nwords) ? p.cand[wbase + lane] : 0u;
  const uint32_t cnt = __popc(word);
  uint32_t incl = cnt;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t v = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += v;
  }
  const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
  s_word[wid][lane] = word;
  s_excl[wid][lane] = incl - cnt;
  __syncwarp();

  for (uint32_t base = 0; base < total; base += 32) {
    const uint32_t j = base + lane;
    const bool has = j < total;
    const unsigned active = __ballot_sync(0xffffffffu, has);
    if (has) {
      // source lane: last l with excl[l] <= j
      int lo = 0;
#pragma unroll
      for (int step = 16; step > 0; step >>= 1)
        if (lo + step < 32 && s_excl[wid][lo + step] <= j) lo += step;
      const uint32_t b = __fns(s_word[wid][lo], 0, (int)(j - s_excl[wid][lo]) + 1);
      const uint64_t c = (wbase + lo) * 32 + b;
      const ulonglong2 v = reinterpret_cast<const ulonglong2*>(p.prev)[c];
      const Digest d{v.x, v.y};
      const uint32_t node = node_of_chunk(p.g, c);
      // warp-level de-duplication of identical digests
      const unsigned m1 = __match_any_sync(active, d.lo);
      const unsigned m2 = __match_any_sync(active, d.hi);
      const unsigned grp = m1 & m2;
      const int leader = __ffs(grp) - 1;
      uint32_t minnode = node;   // minimum node id of the group (every active lane shuffles)
      for (unsigned a = active; a; a &= a - 1) {
        const int sl = __ffs(a) - 1;
        const uint32_t vv = __shfl_sync(active, node, sl);
        if ((grp >> sl) & 1u) minnode = vv < minnode ? vv : minnode;
      }
      uint32_t slot = 0;
      if (lane == leader) {
        bool claimed;
        slot = (uint32_t)table_insert_min(p.tab, p.cap, d, pack_entry(p.g.k, minnode), &claimed);
      }
      slot = __shfl_sync(active, slot, leader);
      st_evict_last_u32(p.slot_of + c, slot, policy_evict_last());
      // dirty stage-0 tile of this chunk (R3 virtual positions)
      const uint32_t T = (uint32_t)(vpos_of_chunk(p.g, c) >> p.g.t0);
      const unsigned tg = __match_any_sync(active, T);
      if (lane == __ffs(tg) - 1) {
        if (atomicExch(&p.dirty[0][T], p.g.epoch) != p.g.epoch) {
          const uint32_t i = atomicAdd(&s_cnt, 1u);
          if (i < 256) s_tiles[i] = T;
          else p.wl0[atomicAdd(&p.tot->wl_count[0], 1u)] = T;   // overflow: direct append
          // count dirty children up the stage hierarchy (the tree kernels' climb target)
          uint64_t x = T;
          for (int s = 1; s < p.S; ++s) {
            const uint64_t P = x >> p.gsz[s];
            if (atomicAdd(&p.cnt[s][P], 1u) != 0) break;
            p.dirty[s][P] = p.g.epoch;
            x = P;
          }
        }
      }
    }
  }
  if (lane == 0 && total) atomicAdd(&p.tot->n_cand, (unsigned long long)total);
  __syncthreads();
  const uint32_t nt = s_cnt < 256 ? s_cnt : 256;
  if (threadIdx.x == 0 && nt) s_base = atomicAdd(&p.tot->wl_count[0], nt);
  __syncthreads();
  if (threadIdx.x < nt) p.wl0[s_base + threadIdx.x] = s_tiles[threadIdx.x];
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
cudaError_t leaf_smem_config(const LeafParams& p, size_t* smem_bytes) {
  *smem_bytes = 1024 + (size_t)p.nst * p.stage_bytes + (size_t)p.nst * kLeafThreads * 16 + (size_t)p.nst * 8;
  return cudaSuccess;
}

cudaError_t launch_leaf(const CUtensorMap* tmap, const LeafParams& p, int num_sms, cudaStream_t st) {
  if (p.n_main == 0) return cudaSuccess;
  size_t smem;
  leaf_smem_config(p, &smem);
  const uint64_t n_tiles = p.n_main / kLeafThreads;
  uint64_t grid = (uint64_t)num_sms * 2;
  if (grid > n_tiles) grid = n_tiles;
  if (p.mode3d) leaf_hash_kernel<1><<<(unsigned)grid, kLeafThreads, smem, st>>>(*tmap, p);
  else leaf_hash_kernel<0><<<(unsigned)grid, kLeafThreads, smem, st>>>(*tmap, p);
  return cudaGetLastError();
}

cudaError_t launch_leaf_tail(const LeafParams& p, cudaStream_t st) {
  if (p.tail_begin >= p.g.n) return cudaSuccess;
  const uint64_t cnt = p.g.n - p.tail_begin;
  leaf_tail_kernel<<<(unsigned)((cnt + 255) / 256), 256, 0, st>>>(p);
  return cudaGetLastError();
}

cudaError_t launch_insert(const InsertParams& p, cudaStream_t st) {
  const uint64_t warps = (p.nwords + 31) / 32;
  const uint64_t blocks = (warps + 7) / 8;
  if (blocks) return launch_pdl(insert_kernel, (unsigned)blocks, 256, 0, st, p);
  return cudaSuccess;
}

cudaError_t leaf_setup_attributes() {
  // the largest dynamic smem any leaf configuration asks for (C >= 128: 3 x 36 KB; C < 128: <= 96 KB)
  const int smem = 1024 + 110 * 1024;
  cudaError_t e = cudaFuncSetAttribute(leaf_hash_kernel<1>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess) e = cudaFuncSetAttribute(leaf_hash_kernel<0>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  return e;
}

cudaError_t launch_rehash(const Slot* old_tab, uint64_t old_cap, Slot* new_tab, uint64_t new_cap, cudaStream_t st) {
  uint64_t blocks = (old_cap + 255) / 256;
  if (blocks > 148 * 16) blocks = 148 * 16;
  if (blocks) rehash_kernel<<<(unsigned)blocks, 256, 0, st>>>(old_tab, old_cap, new_tab, new_cap);
  return cudaGetLastError();
}

}  // namespace ckpt
