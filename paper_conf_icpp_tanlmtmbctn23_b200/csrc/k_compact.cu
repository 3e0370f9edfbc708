// k_compact.cu — consolidated-difference serialisation.
//
// "we propose serializing the metadata and the unique chunks into a consolidated
// difference directly on the GPU memory ... pre-calculates offsets in the consolidated
// difference and assigns GPU threads to parallelize the data transfers", with "a
// team of threads to copy each chunk" so accesses coalesce.
//   (the phase-3 kernel writes every dirty tile's counts {#FIRST regions, #SHIFT regions,
//    FIRST bytes} and adds them to per-32-tile and per-1024-tile sums)
//   KG gather_kernel : one warp per dirty tile. Its offsets in the three sections are the
//                      exclusive prefix of the counts, summed directly from <= 2048 block
//                      sums, <= 31 group sums and <= 31 tile counts (one round of loads);
//                      it writes its FIRST entries (u32 node) and SHIFT entries (u32 node,
//                      src node, src ckpt) (R13) and copies its FIRST bytes.
//                      Block 0 writes the 64-B header, the zero pad and the totals.
#include "kernels.h"
#include "tma.cuh"

namespace ckpt {

__device__ __forceinline__ void warp_sum3(unsigned long long& a, unsigned long long& b, unsigned long long& c) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, o);
    b += __shfl_xor_sync(0xffffffffu, b, o);
    c += __shfl_xor_sync(0xffffffffu, c, o);
  }
}


#ifndef CKPT_GATHER_THREADS
#define CKPT_GATHER_THREADS 256
#endif
constexpr int kCT = CKPT_GATHER_THREADS;

// Every counter the host reports is final once the gather kernel runs (tree kernels done,
// pdl_wait): block 0 copies them to mapped host memory early, in 16-byte stores, and
// orders them at system scope right away (one fence, one thread), so they are visible to
// the host before the epoch the last block publishes (which is ordered after block 0's
// arrival on the completion counter).
__device__ __forceinline__ void host_totals(const CompactParams& p) {
  static_assert(offsetof(Totals, done) % 4 == 0, "Totals layout");
  const uint4* src = reinterpret_cast<const uint4*>(p.tot);
  uint4* dst = reinterpret_cast<uint4*>(p.tot_host);
  constexpr uint32_t nv = (uint32_t)(offsetof(Totals, done) / 16);
  for (uint32_t i = 0; i < nv; ++i) dst[i] = __ldcg(src + i);
  const uint32_t* s32 = reinterpret_cast<const uint32_t*>(p.tot);
  uint32_t* d32 = reinterpret_cast<uint32_t*>(p.tot_host);
  for (uint32_t w = nv * 4; w < (uint32_t)(offsetof(Totals, done) / 4); ++w) d32[w] = __ldcg(s32 + w);
  __threadfence_system();
}

// The call's statistics are final here (phases 2-3 are complete, the totals are summed): the
// host may return (one host wait per call, include/ckpt.h). The rest of this kernel (entries,
// data) completes in stream order; the library's diff consumers wait for it on an event.
__device__ __forceinline__ void publish_done(const CompactParams& p) {
  *reinterpret_cast<volatile uint32_t*>(&p.tot_host->done) = p.g.epoch;   // after host_totals' fence
}

// KG: one WARP per dirty tile (worklist of the phase-2 kernel). Writes the tile's metadata
// entries (its region records from phase 3) and copies its FIRST bytes. The data section
// is the FIRST chunks in chunk order (every FIRST leaf lies in exactly one FIRST region,
// and FIRST regions hold only FIRST leaves), so the tile's part of it is its FIRST-chunk
// mask (phase 2) compacted: the k-th FIRST chunk of the tile goes to tile offset + k C.
// A lane-strided stream of 16-byte units covers the tile's FIRST bytes (coalesced); unit
// -> chunk is a 5-step search over the 32 per-word ranks plus a find-n-th-set-bit.
// Everything read here was written by earlier kernels, so the loads take the L1-cached
// read-only path: the block sums are read by every warp, and through L2 alone one slice
// would serialise those requests.
constexpr int kGW = kCT / 32;

constexpr int kStageUnits = 640;   // 10 KB of 16-byte units staged per warp and round

struct GatherWarp {
  uint32_t pre[32];   // FIRST chunks in the mask words before word i
  uint32_t fw[32];    // the tile's FIRST-chunk mask words
  uint16_t idx[1 << kTileLog];   // the k-th FIRST chunk of the tile (offset from its first chunk)
  uint4 stage[kStageUnits];
};

__device__ __forceinline__ void cp_async16(void* smem, const void* gmem, uint32_t src_bytes) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(smem)), "l"(gmem), "r"(src_bytes)
               : "memory");
}
__device__ __forceinline__ void cp_async_wait_all() {
  asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}

__global__ void __launch_bounds__(kCT, 512 / kCT) gather_kernel(CompactParams p) {
  extern __shared__ __align__(16) uint8_t gather_smem[];
  GatherWarp* gsm = reinterpret_cast<GatherWarp*>(gather_smem);
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  GatherWarp& gw = gsm[wid];
  const Geo& g = p.g;
  const unsigned long long bt0 = p.trace ? gtime_ns() : 0;
  // the next call's counters (not touched by this call's kernels)
  for (uint64_t i = (uint64_t)blockIdx.x * kCT + threadIdx.x; i < p.ctr_next_words; i += (uint64_t)gridDim.x * kCT)
    p.ctr_next[i] = make_uint4(0, 0, 0, 0);
  pdl_launch_dependents();
  pdl_wait();
  const unsigned long long bt1 = p.trace ? gtime_ns() : 0;
  const uint64_t nblk = (p.n_tiles + kTilesPerBlock - 1) / kTilesPerBlock;
  const uint64_t nwarps = (uint64_t)gridDim.x * kGW;
  // R22 / R23: the difference is stored in full (one FIRST region, the root, and the whole
  // buffer); the dirty-tile work below is skipped
  const bool sw = switched_full(p.tot, p.sw_permille, g);
  const bool full = sw || p.full_first;
  const uint32_t count = full ? 0u : *(volatile uint32_t*)&p.tot->wl_count[0];
  if (full) {
    if (blockIdx.x == 0 && threadIdx.x == 0) {
      Totals* t = p.tot;
      t->nF = 1; t->nS = 0; t->data_bytes = g.B; t->meta_bytes = 80;
      if (sw) {   // every changed chunk is stored; no record operation ran
        t->n_first = t->n_nonfixed; t->n_spatial = 0; t->n_temporal = 0; t->p2_inserts = 0;
      }
      t->full_kind = sw ? 2 : 1;
      uint8_t* o = p.out;
      *reinterpret_cast<uint32_t*>(o + 0) = 0x44504B43u;   // 'CKPD'
      *reinterpret_cast<uint16_t*>(o + 4) = 1;
      *reinterpret_cast<uint16_t*>(o + 6) = 3;             // flags: stored in full
      *reinterpret_cast<uint32_t*>(o + 8) = g.k;
      *reinterpret_cast<uint32_t*>(o + 12) = g.C;
      *reinterpret_cast<unsigned long long*>(o + 16) = g.B;
      *reinterpret_cast<unsigned long long*>(o + 24) = g.n;
      *reinterpret_cast<unsigned long long*>(o + 32) = 1;
      *reinterpret_cast<unsigned long long*>(o + 40) = 0;
      *reinterpret_cast<unsigned long long*>(o + 48) = g.B;
      *reinterpret_cast<unsigned long long*>(o + 56) = 0;  // hash seed, reserved
      *reinterpret_cast<uint4*>(o + 64) = make_uint4(0, 0, 0, 0);   // root entry (node 0) + pad
      host_totals(p);
      publish_done(p);
    }
    // the whole buffer, 16-byte units, kFullUnroll loads in flight per thread before the
    // stores (2 CTAs x 256 threads per SM: 64 KB in flight per SM covers HBM latency)
    constexpr int kFullUnroll = 8;
    const uint4* src = reinterpret_cast<const uint4*>(p.buf);
    uint4* dst = reinterpret_cast<uint4*>(p.out + 80);
    const uint64_t nu = g.B / 16, nth = (uint64_t)gridDim.x * kCT;
    for (uint64_t i = (uint64_t)blockIdx.x * kCT + threadIdx.x; i < nu; i += kFullUnroll * nth) {
      uint4 v[kFullUnroll];
#pragma unroll
      for (int u = 0; u < kFullUnroll; ++u)
        if (i + u * nth < nu) v[u] = __ldcs(src + i + u * nth);
#pragma unroll
      for (int u = 0; u < kFullUnroll; ++u)
        if (i + u * nth < nu) __stcs(dst + i + u * nth, v[u]);
    }
    if (blockIdx.x == 0 && threadIdx.x == 0)
      for (uint64_t b = nu * 16; b < g.B; ++b) p.out[80 + b] = p.buf[b];
  }
  // worklist entry w -> block w mod grid, warp w / grid: with few dirty tiles (large chunks)
  // every SM still gets work
  uint64_t w = (uint64_t)wid * gridDim.x + blockIdx.x;
  // A tile's data may be split over `parts` warps (large chunks, few tiles): work item w is
  // part w mod parts of the (w / parts)-th dirty tile; part j copies staging rounds
  // j, j + parts, ... and part 0 also writes the tile's entries.
  const uint32_t parts = p.parts;
  // the worklist entry is loaded before the count check (the array has n_tiles entries)
  uint64_t T = w / parts < p.n_tiles ? __ldg(p.wl0 + w / parts) : 0;

  // totals = sum of the per-1024-tile block sums (every warp; 8 values at 1 GiB, C = 128)
  unsigned long long nF_tot = 0, nS_tot = 0, data_tot = 0;
  for (uint64_t i = lane; i < nblk; i += 32) {
    nF_tot += __ldg(p.blocksum + 3 * i);
    nS_tot += __ldg(p.blocksum + 3 * i + 1);
    data_tot += __ldg(p.blocksum + 3 * i + 2);
  }
  warp_sum3(nF_tot, nS_tot, data_tot);
  const bool basic = p.mode == kModeBasic;
  // Basic: the changed-chunk bitmap replaces the entry lists (nF_tot = changed chunks)
  const unsigned long long raw = basic ? 64 + 4ull * p.nwords : 64 + 4 * nF_tot + 12 * nS_tot;
  const unsigned long long meta = (raw + 15) & ~15ull;
  // the header is written by a warp without a tile when there is one (the last warp):
  // the mapped-memory totals and their system-scope fence would otherwise delay a tile
  const uint64_t hdr_warp = (uint64_t)count * parts < nwarps ? nwarps - 1 : 0;
  if ((uint64_t)wid * gridDim.x + blockIdx.x == hdr_warp && lane == 0 && !full) {
    // totals and the 64-byte header (R13)
    p.tot->nF = nF_tot; p.tot->nS = nS_tot; p.tot->data_bytes = data_tot; p.tot->meta_bytes = meta;
    if (basic) p.tot->n_first = nF_tot;   // every changed chunk is stored (no record)
    uint8_t* o = p.out;
    *reinterpret_cast<uint32_t*>(o + 0) = 0x44504B43u;   // 'CKPD'
    *reinterpret_cast<uint16_t*>(o + 4) = 1;             // version
    *reinterpret_cast<uint16_t*>(o + 6) = (uint16_t)p.flags;  // flags: the method, 4 under R24
    *reinterpret_cast<uint32_t*>(o + 8) = g.k;
    *reinterpret_cast<uint32_t*>(o + 12) = g.C;
    *reinterpret_cast<unsigned long long*>(o + 16) = g.B;
    *reinterpret_cast<unsigned long long*>(o + 24) = g.n;
    *reinterpret_cast<unsigned long long*>(o + 32) = nF_tot;
    *reinterpret_cast<unsigned long long*>(o + 40) = nS_tot;
    *reinterpret_cast<unsigned long long*>(o + 48) = data_tot;
    *reinterpret_cast<uint32_t*>(o + 56) = 0;            // hash seed
    *reinterpret_cast<uint32_t*>(o + 60) = 0;            // reserved
    for (unsigned long long x = raw; x < meta; ++x) o[x] = 0;
    host_totals(p);
    publish_done(p);
  }
  if (basic) {   // the bitmap: K1's candidate words, all n bits
    uint32_t* bm = reinterpret_cast<uint32_t*>(p.out + 64);
    for (uint64_t i = (uint64_t)blockIdx.x * kCT + threadIdx.x; i < p.nwords; i += (uint64_t)gridDim.x * kCT)
      bm[i] = (i + 1 == p.nwords && (p.g.n & 31)) ? (__ldg(p.cand + i) & ((1u << (p.g.n & 31)) - 1u)) : __ldg(p.cand + i);
  }
  uint8_t* const ent_f = p.out + 64;
  uint8_t* const ent_s = p.out + 64 + 4 * nF_tot;
  uint8_t* const dat = p.out + meta;
  const uint32_t U = g.C / 16;   // 16-byte units per chunk
  const int ulog = (U & (U - 1)) ? -1 : __ffs(U) - 1;   // shift instead of a division when C = 2^j

  for (; w < (uint64_t)count * parts; w += nwarps) {
    const uint32_t part = (uint32_t)(w % parts);
    unsigned long long tg0 = 0, tg1 = 0, tg2 = 0;
    if (p.trace) tg0 = gtime_ns();
    // one round of loads: counts, FIRST-chunk mask, the first 64 region records, prefix sums
    uint64_t lo, hi;
    chunk_range(g, g.t0, T, lo, hi);
    uint4 cnt;
    uint32_t fw;
    if (basic) {   // the tile's changed chunks, chunk order, straight from K1's bitmap
      cnt = make_uint4(0, 0, 0, g.epoch);
      const uint64_t c0 = lo + 32ull * lane;
      fw = 0;
      if (c0 < hi) {
        const uint32_t sh = (uint32_t)(c0 & 31);
        const uint32_t a = __ldg(p.cand + (c0 >> 5));
        const uint32_t b = (c0 >> 5) + 1 < p.nwords ? __ldg(p.cand + (c0 >> 5) + 1) : 0u;
        fw = sh ? ((a >> sh) | (b << (32 - sh))) : a;
        if (hi - c0 < 32) fw &= (1u << (hi - c0)) - 1u;
      }
    } else {
      cnt = __ldg(p.tilecnt + T);
      fw = __ldg(p.lmask + T * kLmWords + kLmFirstChunks + lane);
    }
    const uint4* recs = p.scratch + (T << g.t0);
    const uint32_t tcap = 1u << g.t0;   // records per tile
    uint4 rec0 = make_uint4(0, 0, 0, 0), rec1 = make_uint4(0, 0, 0, 0);
    if ((uint32_t)lane < tcap) rec0 = __ldg(recs + lane);
    if ((uint32_t)lane + 32 < tcap) rec1 = __ldg(recs + 32 + lane);
    // exclusive prefix of tile T: earlier 1024-tile blocks, earlier 32-tile groups of its
    // block, earlier tiles of its group (stale tile counts carry an older epoch)
    unsigned long long pF = 0, pS = 0, pD = 0;
    {
      const uint64_t B0 = T / kTilesPerBlock, G0 = T / 32;
      for (uint64_t i = lane; i < B0; i += 32) {
        pF += __ldg(p.blocksum + 3 * i);
        pS += __ldg(p.blocksum + 3 * i + 1);
        pD += __ldg(p.blocksum + 3 * i + 2);
      }
      const uint64_t gq = B0 * (kTilesPerBlock / 32) + lane;
      if (gq < G0) {
        pF += __ldg(p.gsum + 3 * gq);
        pS += __ldg(p.gsum + 3 * gq + 1);
        pD += __ldg(p.gsum + 3 * gq + 2);
      }
      const uint64_t tq = G0 * 32 + lane;
      if (tq < T) {
        if (basic) {   // an earlier tile never holds the short last chunk
          const unsigned long long x = __ldg(p.tcc + tq);
          pF += x;
          pD += x * g.C;
        } else {
          const uint4 x = __ldg(p.tilecnt + tq);
          if (x.w == g.epoch) { pF += x.x; pS += x.y; pD += x.z; }
        }
      }
    }
    const uint64_t Tcur = T;
    if (w + nwarps < (uint64_t)count * parts) T = __ldg(p.wl0 + (w + nwarps) / parts);   // next tile, early
    if (cnt.w != g.epoch) {
      warp_sum3(pF, pS, pD);
      continue;
    }
    const uint32_t nF = basic ? 0u : cnt.x, nS = basic ? 0u : cnt.y;   // Basic: no entries
    if (p.trace) tg1 = gtime_ns();
    // ranks of the FIRST chunks (chunk order)
    const uint32_t pc = __popc(fw);
    uint32_t incl = pc;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t u = __shfl_up_sync(0xffffffffu, incl, o);
      if (lane >= o) incl += u;
    }
    gw.pre[lane] = incl - pc;
    gw.fw[lane] = fw;
    {   // the tile's FIRST chunks as a list (k-th FIRST chunk -> offset in the tile)
      uint32_t r = incl - pc;
      for (uint32_t m = fw; m; m &= m - 1) gw.idx[r++] = (uint16_t)(32u * lane + (__ffs(m) - 1));
    }
    const uint32_t nch = __shfl_sync(0xffffffffu, incl, 31);
    __syncwarp();
    // the FIRST bytes: unit x of the tile's stream = unit (x mod U) of its (x / U)-th chunk,
    // source found from the mask alone; up to kStageUnits units go global -> shared with
    // cp.async in one round trip, then shared -> the data section at tile offset + 16 x.
    // The buffer's last chunk may be short: its last unit is zero-filled past B (the store
    // may then write up to 15 bytes past the data section, inside the arena's slack) and
    // units entirely past B are skipped.
    const uint32_t nunits = nch * U;
    auto unit_src = [&](uint32_t x) -> unsigned long long {
      const uint32_t k = ulog >= 0 ? x >> ulog : x / U, sub = x - k * U;
      return (lo + gw.idx[k]) * (unsigned long long)g.C + 16u * sub;
    };
    bool entries_done = part != 0;
    if (entries_done) warp_sum3(pF, pS, pD);   // part 0 sums them while its first round is in flight
    for (uint32_t x0 = part * kStageUnits; x0 < nunits || !entries_done; x0 += parts * kStageUnits) {
      const uint32_t x1 = x0 + kStageUnits < nunits ? x0 + kStageUnits : nunits;
      for (uint32_t x = x0 + lane; x < x1; x += 32) {
        const unsigned long long so = unit_src(x);
        if (so + 16 <= g.B) {
          cp_async16(&gw.stage[x - x0], p.buf + so, 16u);
        } else if (so < g.B) {
          // the buffer's last, partial unit: only its bytes are read (the caller's allocation
          // may end at B), the rest of the staged unit is zero
          uint32_t w4[4] = {0, 0, 0, 0};
          for (uint32_t q = 0; q < (uint32_t)(g.B - so); ++q) w4[q >> 2] |= (uint32_t)p.buf[so + q] << (8 * (q & 3));
          gw.stage[x - x0] = make_uint4(w4[0], w4[1], w4[2], w4[3]);
        }
      }
      if (!entries_done) {
        // while the first round is in flight: the tile's offsets and its region entries
        // (R13): FIRST u32 node; SHIFT u32 node, u32 src node, u32 src ckpt
        warp_sum3(pF, pS, pD);
        for (uint32_t i = lane; i < nF + nS; i += 32) {
          const uint4 r = i < 32 ? rec0 : (i < 64 ? rec1 : __ldg(recs + i));
          if (i < nF) {
            *reinterpret_cast<uint32_t*>(ent_f + 4ull * (pF + i)) = r.x;
          } else {
            uint32_t* e = reinterpret_cast<uint32_t*>(ent_s + 12ull * (pS + i - nF));
            e[0] = r.x; e[1] = r.y; e[2] = r.z;
          }
        }
        entries_done = true;
      }
      cp_async_wait_all();
      __syncwarp();
      for (uint32_t x = x0 + lane; x < x1; x += 32) {
        // only the tile's last FIRST chunk, in the tile holding the buffer's end, can be short
        if (hi == g.n && (ulog >= 0 ? x >> ulog : x / U) + 1 == nch && unit_src(x) >= g.B) continue;
        *reinterpret_cast<uint4*>(dat + pD + 16ull * x) = gw.stage[x - x0];
      }
      __syncwarp();
    }
    __syncwarp();
    if (p.trace && lane == 0) {
      tg2 = gtime_ns();
      if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 2)) {
        r[0] = make_ulonglong4(tg0, tg1, tg2, 77);
        r[1] = make_ulonglong4(Tcur, ((unsigned long long)nS << 32) | nF, cnt.z, 78);
      }
    }
  }
  __syncthreads();
  trace_block(p.trace, p.trace_n, bt0, bt1, 5);
}

static int g_gather_blocks_per_sm = 0;

uint32_t gather_parts(uint64_t n_tiles, uint32_t C, int num_sms) {
  // split tiles over warps only when there are fewer tiles than resident warps and the
  // tiles carry many bytes (C >= 512: a 1024-chunk tile spans >= 512 KB)
  const int bps = g_gather_blocks_per_sm > 0 ? g_gather_blocks_per_sm : 2;
  const uint64_t warps = (uint64_t)num_sms * bps * kGW;
  if (C < 512 || n_tiles == 0 || n_tiles >= warps) return 1;
  const uint64_t r = warps / n_tiles;
  return (uint32_t)(r > 8 ? 8 : r);
}

cudaError_t launch_compact(const CompactParams& p, int num_sms, cudaStream_t st) {
  // one resident wave of gather blocks (the dirty-tile count is only known on the device,
  // and blocks beyond one wave would only arrive late to find no work)
  const int bps = g_gather_blocks_per_sm > 0 ? g_gather_blocks_per_sm : 2;
  uint64_t grid = p.n_tiles * p.parts;   // worklist entries are spread over the blocks first
  // a difference that may be stored in full (R22 / R23) copies the whole buffer: full wave
  if (grid > (uint64_t)num_sms * bps || p.full_first || p.sw_permille >= 0) grid = (uint64_t)num_sms * bps;
  return launch_pdl(gather_kernel, (unsigned)grid, kCT, kGW * sizeof(GatherWarp), st, p);
}


// Load this file's kernels now (CUDA lazy module loading would otherwise stall the first
// launch of each kernel inside the first checkpoint).
cudaError_t preload_compact() {
  cudaFuncAttributes a;
  const int smem = (int)(kGW * sizeof(GatherWarp));
  cudaError_t e = cudaFuncSetAttribute(gather_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
  if (e == cudaSuccess)
    e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_gather_blocks_per_sm, gather_kernel, kCT, smem);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, gather_kernel);
  return e;
}

}  // namespace ckpt
