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
//   KD data_kernel   : copies the FIRST chunks into the data section, warp per 8-KiB
//                      segment, coalesced 16-byte loads/stores (balanced even when one
//                      region is the whole buffer).
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


constexpr int kCT = 256;

// KG: one WARP per dirty tile (worklist of the phase-2 kernel). Writes the tile's metadata entries
// and copies its FIRST bytes: the tile's FIRST regions are taken 32 at a time (lane i ->
// region i), a warp scan gives their data offsets, and the batch's bytes are copied as
// one lane-strided stream of 16-byte units (coalesced; the region of a unit is found by
// a 5-step search in the warp's shared table). Regions above kBig bytes are deferred to
// KD, which spreads each over the whole grid.
constexpr unsigned long long kBig = 1ull << 20;
constexpr int kGW = kCT / 32;

struct GatherWarp {
  unsigned long long off[33];    // batch-relative offsets of the inline stream
  unsigned long long dst[32];    // data-section offset of each region
  unsigned long long src[32];    // source byte offset in the checkpoint buffer
};

__global__ void __launch_bounds__(kCT) gather_kernel(CompactParams p) {
  __shared__ GatherWarp gsm[kGW];
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  GatherWarp& gw = gsm[wid];
  const Geo& g = p.g;
  const unsigned long long bt0 = p.trace ? gtime_ns() : 0;
  pdl_launch_dependents();
  pdl_wait();
  const unsigned long long bt1 = p.trace ? gtime_ns() : 0;
  // totals = sum of the per-1024-tile block sums (every warp; 8 values at 1 GiB, C = 128)
  const uint64_t nblk = (p.n_tiles + kTilesPerBlock - 1) / kTilesPerBlock;
  unsigned long long nF_tot = 0, nS_tot = 0, data_tot = 0;
  for (uint64_t i = lane; i < nblk; i += 32) {
    nF_tot += __ldcg(p.blocksum + 3 * i);
    nS_tot += __ldcg(p.blocksum + 3 * i + 1);
    data_tot += __ldcg(p.blocksum + 3 * i + 2);
  }
  warp_sum3(nF_tot, nS_tot, data_tot);
  const unsigned long long raw = 64 + 4 * nF_tot + 12 * nS_tot;
  const unsigned long long meta = (raw + 15) & ~15ull;
  if (blockIdx.x == 0 && wid == 0 && lane == 0) {
    // totals and the 64-byte header (R13)
    p.tot->nF = nF_tot; p.tot->nS = nS_tot; p.tot->data_bytes = data_tot; p.tot->meta_bytes = meta;
    uint8_t* o = p.out;
    *reinterpret_cast<uint32_t*>(o + 0) = 0x44504B43u;   // 'CKPD'
    *reinterpret_cast<uint16_t*>(o + 4) = 1;             // version
    *reinterpret_cast<uint16_t*>(o + 6) = 0;             // flags
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
    // every counter the host reports is final here (tree kernels done, pdl_wait above)
    *p.tot_host = *p.tot;
  }
  uint8_t* const ent_f = p.out + 64;
  uint8_t* const ent_s = p.out + 64 + 4 * nF_tot;
  uint8_t* const dat = p.out + meta;

  const uint64_t nwarps = (uint64_t)gridDim.x * kGW;
  const uint32_t count = *(volatile uint32_t*)&p.tot->wl_count[0];
  for (uint64_t w = (uint64_t)blockIdx.x * kGW + wid; w < count; w += nwarps) {
    unsigned long long tg0 = 0, tg1 = 0, tg2 = 0;
    if (p.trace) asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tg0));
    const uint64_t T = __ldcg(p.wl0 + w);
    const uint4 cnt = __ldcg(p.tilecnt + T);
    // exclusive prefix of tile T: earlier 1024-tile blocks, earlier 32-tile groups of its
    // block, earlier tiles of its group (stale tile counts carry an older epoch)
    unsigned long long pF = 0, pS = 0, pD = 0;
    {
      const uint64_t B0 = T / kTilesPerBlock, G0 = T / 32;
      for (uint64_t i = lane; i < B0; i += 32) {
        pF += __ldcg(p.blocksum + 3 * i);
        pS += __ldcg(p.blocksum + 3 * i + 1);
        pD += __ldcg(p.blocksum + 3 * i + 2);
      }
      const uint64_t gq = B0 * (kTilesPerBlock / 32) + lane;
      if (gq < G0) {
        pF += __ldcg(p.gsum + 3 * gq);
        pS += __ldcg(p.gsum + 3 * gq + 1);
        pD += __ldcg(p.gsum + 3 * gq + 2);
      }
      const uint64_t tq = G0 * 32 + lane;
      if (tq < T) {
        const uint4 x = __ldcg(p.tilecnt + tq);
        if (x.w == g.epoch) { pF += x.x; pS += x.y; pD += x.z; }
      }
      warp_sum3(pF, pS, pD);
    }
    if (cnt.w != g.epoch) continue;
    const uint32_t nF = cnt.x, nS = cnt.y;
    if (nF + nS == 0) continue;
    const uint4 off = make_uint4((uint32_t)pF, (uint32_t)pS, 0u, 0u);
    const unsigned long long doff = pD;
    const uint4* recs = p.scratch + ((uint64_t)T << g.t0);
    if (p.trace) asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tg1));
    // SHIFT entries (R13): u32 node, u32 src node, u32 src ckpt
    for (uint32_t i = lane; i < nS; i += 32) {
      const uint4 r = recs[nF + i];
      uint32_t* e = reinterpret_cast<uint32_t*>(ent_s + 12ull * (off.y + i));
      e[0] = r.x; e[1] = r.y; e[2] = r.z;
    }
    // FIRST entries + data, 32 regions per batch
    unsigned long long carry = doff;
    for (uint32_t b0 = 0; b0 < nF; b0 += 32) {
      const uint32_t i = b0 + lane;
      unsigned long long len = 0, s0 = 0;
      if (i < nF) {
        const uint32_t node = recs[i].x;
        *reinterpret_cast<uint32_t*>(ent_f + 4ull * (off.x + i)) = node;
        const int depth = 31 - __clz(node + 1);
        uint64_t lo, hi;
        chunk_range(g, g.h - depth, (uint64_t)node + 1 - (1ull << depth), lo, hi);
        len = range_bytes(g, lo, hi);
        s0 = lo * (unsigned long long)g.C;
      }
      const bool big = len > kBig;
      const unsigned long long leff = big ? 0 : len;
      unsigned long long incl = len, ieff = leff;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long u = __shfl_up_sync(0xffffffffu, incl, o);
        const unsigned long long v = __shfl_up_sync(0xffffffffu, ieff, o);
        if (lane >= o) { incl += u; ieff += v; }
      }
      const unsigned long long my_dst = carry + incl - len;
      if (big) {
        const uint32_t slot = atomicAdd(&p.tot->big_count, 1u);
        p.big[slot] = make_ulonglong2(my_dst, s0);
        p.big_len[slot] = len;
      }
      gw.off[lane] = ieff - leff;
      gw.dst[lane] = my_dst;
      gw.src[lane] = s0;
      const unsigned long long btot = __shfl_sync(0xffffffffu, ieff, 31);
      if (lane == 31) gw.off[32] = btot;
      carry += __shfl_sync(0xffffffffu, incl, 31);
      __syncwarp();
      const uint32_t nreg = (nF - b0) < 32 ? (nF - b0) : 32;
      // stream copy of the inline bytes: unit x covers [16x, 16x+16); 8 independent units
      // per lane per iteration (4 KB per warp) so a typical tile needs one round trip
      const unsigned long long nunits = (btot + 15) / 16;
      constexpr int kU = 8;
      for (unsigned long long x0 = 0; x0 < nunits; x0 += 32 * kU) {
        uint4 v[kU];
        uint8_t* d[kU];
        unsigned long long rem[kU];
        const uint8_t* sp[kU];
#pragma unroll
        for (int u = 0; u < kU; ++u) {
          const unsigned long long x = x0 + u * 32 + lane;
          rem[u] = 0;
          if (x < nunits) {
            const unsigned long long o = 16 * x;
            int r = 0;
#pragma unroll
            for (int step = 16; step > 0; step >>= 1)
              if (r + step < (int)nreg && gw.off[r + step] <= o) r += step;
            while (r + 1 < (int)nreg && gw.off[r + 1] <= o) ++r;   // skip deferred (zero-length) regions
            const unsigned long long rel = o - gw.off[r];
            sp[u] = p.buf + gw.src[r] + rel;
            d[u] = dat + gw.dst[r] + rel;
            rem[u] = (r + 1 < (int)nreg ? gw.off[r + 1] : btot) - o;
            if (rem[u] >= 16) v[u] = __ldg(reinterpret_cast<const uint4*>(sp[u]));
          }
        }
#pragma unroll
        for (int u = 0; u < kU; ++u) {
          if (rem[u] >= 16) *reinterpret_cast<uint4*>(d[u]) = v[u];
          else
            for (unsigned long long b = 0; b < rem[u]; ++b) d[u][b] = sp[u][b];
        }
      }
      __syncwarp();
    }
    if (p.trace && lane == 0) {
      asm volatile("mov.u64 %0, %globaltimer;" : "=l"(tg2));
      if (ulonglong4* r = trace_alloc(p.trace, p.trace_n, 1)) *r = make_ulonglong4(tg0, tg1, tg2, 77);
    }
  }
  __syncthreads();
  trace_block(p.trace, p.trace_n, bt0, bt1, 5);
}

// KD: first-occurrence regions above kBig bytes (e.g. a fully new checkpoint is one
// region), each spread over the whole grid with coalesced 16-byte units.
__global__ void __launch_bounds__(kCT) data_kernel(CompactParams p) {
  const unsigned long long bt0 = p.trace ? gtime_ns() : 0;
  // the next call's counters (not touched by this call's kernels)
  for (uint64_t i = (uint64_t)blockIdx.x * kCT + threadIdx.x; i < p.ctr_next_words; i += (uint64_t)gridDim.x * kCT)
    p.ctr_next[i] = make_uint4(0, 0, 0, 0);
  pdl_wait();
  const unsigned long long bt1 = p.trace ? gtime_ns() : 0;
  const uint32_t nbig = *(volatile uint32_t*)&p.tot->big_count;
  if (nbig == 0) {
    trace_block(p.trace, p.trace_n, bt0, bt1, 6);
    return;
  }
  uint8_t* const dat = p.out + p.tot->meta_bytes;
  const unsigned long long stride = (unsigned long long)gridDim.x * kCT * 16;
  for (uint32_t b = 0; b < nbig; ++b) {
    const ulonglong2 e = p.big[b];
    const unsigned long long len = p.big_len[b];
    const uint8_t* s = p.buf + e.y;
    uint8_t* d = dat + e.x;
    const unsigned long long full = len & ~15ull;
    for (unsigned long long o = ((unsigned long long)blockIdx.x * kCT + threadIdx.x) * 16; o < full; o += stride)
      *reinterpret_cast<uint4*>(d + o) = __ldg(reinterpret_cast<const uint4*>(s + o));
    if (blockIdx.x == 0 && threadIdx.x == 0)
      for (unsigned long long o = full; o < len; ++o) d[o] = s[o];
  }
  trace_block(p.trace, p.trace_n, bt0, bt1, 6);
}

cudaError_t launch_compact(const CompactParams& p, int num_sms, cudaStream_t st) {
  // the tile offsets are prefix sums the gather warps compute themselves (see above)
  uint64_t grid = (p.n_tiles + kGW - 1) / kGW;
  if (grid > (uint64_t)num_sms * 8) grid = (uint64_t)num_sms * 8;
  cudaError_t e = launch_pdl(gather_kernel, (unsigned)grid, kCT, 0, st, p);
  if (e == cudaSuccess) e = launch_pdl(data_kernel, (unsigned)(num_sms * 4), kCT, 0, st, p);
  return e;
}


// Load this file's kernels now (CUDA lazy module loading would otherwise stall the first
// launch of each kernel inside the first checkpoint).
cudaError_t preload_compact() {
  cudaFuncAttributes a;
  cudaError_t e = cudaSuccess;
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, gather_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, data_kernel);
  return e;
}

}  // namespace ckpt
