// k_compact.cu — consolidated-difference serialisation.
//
// "we propose serializing the metadata and the unique chunks into a consolidated
// difference directly on the GPU memory ... pre-calculates offsets in the consolidated
// difference and assigns GPU threads to parallelize the data transfers", with "a
// team of threads to copy each chunk" so accesses coalesce.
//   KR reduce_kernel : per 1024 stage-0 tiles, sums of (#FIRST regions, #SHIFT regions,
//                      FIRST bytes) over tiles dirty in this checkpoint.
//   KO offsets_kernel: prefix over earlier blocks + block scan -> per-tile offsets;
//                      the last block writes the 64-B header, the zero pad and totals.
//   KG gather_kernel : one CTA per dirty tile writes its FIRST entries (u32 node) and
//                      SHIFT entries (u32 node, src node, src ckpt) (R13)
//                      and the global data offset of each FIRST region.
//   KD data_kernel   : copies the FIRST chunks into the data section, warp per 8-KiB
//                      segment, coalesced 16-byte loads/stores (balanced even when one
//                      region is the whole buffer).
#include "kernels.h"

namespace ckpt {

__device__ __forceinline__ void block_sum3(unsigned long long& a, unsigned long long& b, unsigned long long& c,
                                           unsigned long long* sh /* 3 * nwarps */) {
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5, nw = blockDim.x >> 5;
  for (int o = 16; o > 0; o >>= 1) {
    a += __shfl_xor_sync(0xffffffffu, a, o);
    b += __shfl_xor_sync(0xffffffffu, b, o);
    c += __shfl_xor_sync(0xffffffffu, c, o);
  }
  if (lane == 0) { sh[wid] = a; sh[nw + wid] = b; sh[2 * nw + wid] = c; }
  __syncthreads();
  a = b = c = 0;
  for (int i = 0; i < nw; ++i) { a += sh[i]; b += sh[nw + i]; c += sh[2 * nw + i]; }
  __syncthreads();
}

constexpr int kCT = 256;
constexpr int kPer = kTilesPerBlock / kCT;

__global__ void __launch_bounds__(kCT) reduce_kernel(CompactParams p) {
  __shared__ unsigned long long sh[3 * (kCT / 32)];
  unsigned long long a = 0, b = 0, c = 0;
  const uint64_t t0 = (uint64_t)blockIdx.x * kTilesPerBlock + threadIdx.x * kPer;
  for (int i = 0; i < kPer; ++i) {
    const uint64_t T = t0 + i;
    if (T < p.n_tiles) {
      const uint4 v = p.tilecnt[T];
      if (v.w == p.g.epoch) { a += v.x; b += v.y; c += v.z; }
    }
  }
  block_sum3(a, b, c, sh);
  if (threadIdx.x == 0) {
    p.blocksum[3 * blockIdx.x] = a;
    p.blocksum[3 * blockIdx.x + 1] = b;
    p.blocksum[3 * blockIdx.x + 2] = c;
  }
}

__global__ void __launch_bounds__(kCT) offsets_kernel(CompactParams p) {
  __shared__ unsigned long long sh[3 * (kCT / 32)];
  __shared__ unsigned long long wx[kCT / 32], wy[kCT / 32], wz[kCT / 32];
  // prefix of earlier blocks
  unsigned long long a = 0, b = 0, c = 0;
  for (uint32_t i = threadIdx.x; i < blockIdx.x; i += kCT) {
    a += p.blocksum[3 * i];
    b += p.blocksum[3 * i + 1];
    c += p.blocksum[3 * i + 2];
  }
  block_sum3(a, b, c, sh);
  const unsigned long long pa = a, pb = b, pc = c;
  // per-thread values
  const uint64_t t0 = (uint64_t)blockIdx.x * kTilesPerBlock + threadIdx.x * kPer;
  uint4 v[kPer];
  unsigned long long ma = 0, mb = 0, mc = 0;
  for (int i = 0; i < kPer; ++i) {
    const uint64_t T = t0 + i;
    v[i] = make_uint4(0, 0, 0, 0);
    if (T < p.n_tiles) {
      const uint4 x = p.tilecnt[T];
      if (x.w == p.g.epoch) v[i] = x;
    }
    ma += v[i].x; mb += v[i].y; mc += v[i].z;
  }
  // block exclusive scan (warp shuffles + warp totals)
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  unsigned long long ia = ma, ib = mb, ic = mc;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long ua = __shfl_up_sync(0xffffffffu, ia, o);
    const unsigned long long ub = __shfl_up_sync(0xffffffffu, ib, o);
    const unsigned long long uc = __shfl_up_sync(0xffffffffu, ic, o);
    if (lane >= o) { ia += ua; ib += ub; ic += uc; }
  }
  if (lane == 31) { wx[wid] = ia; wy[wid] = ib; wz[wid] = ic; }
  __syncthreads();
  unsigned long long oa = pa, ob = pb, oc = pc, ta = pa, tb = pb, tc = pc;
  for (int i = 0; i < kCT / 32; ++i) {
    if (i < wid) { oa += wx[i]; ob += wy[i]; oc += wz[i]; }
    ta += wx[i]; tb += wy[i]; tc += wz[i];
  }
  oa += ia - ma; ob += ib - mb; oc += ic - mc;
  for (int i = 0; i < kPer; ++i) {
    const uint64_t T = t0 + i;
    if (T < p.n_tiles && (v[i].x | v[i].y))
      p.toff[T] = make_uint4((uint32_t)oa, (uint32_t)ob, (uint32_t)(oc & 0xffffffffu), (uint32_t)(oc >> 32));
    oa += v[i].x; ob += v[i].y; oc += v[i].z;
  }
  if (blockIdx.x == gridDim.x - 1 && threadIdx.x == 0) {
    // totals and the 64-byte header (R13)
    const unsigned long long nF = ta, nS = tb, data = tc;
    const unsigned long long raw = 64 + 4 * nF + 12 * nS;
    const unsigned long long meta = (raw + 15) & ~15ull;
    p.tot->nF = nF; p.tot->nS = nS; p.tot->data_bytes = data; p.tot->meta_bytes = meta;
    uint8_t* o = p.out;
    *reinterpret_cast<uint32_t*>(o + 0) = 0x44504B43u;   // 'CKPD'
    *reinterpret_cast<uint16_t*>(o + 4) = 1;             // version
    *reinterpret_cast<uint16_t*>(o + 6) = 0;             // flags
    *reinterpret_cast<uint32_t*>(o + 8) = p.g.k;
    *reinterpret_cast<uint32_t*>(o + 12) = p.g.C;
    *reinterpret_cast<unsigned long long*>(o + 16) = p.g.B;
    *reinterpret_cast<unsigned long long*>(o + 24) = p.g.n;
    *reinterpret_cast<unsigned long long*>(o + 32) = nF;
    *reinterpret_cast<unsigned long long*>(o + 40) = nS;
    *reinterpret_cast<unsigned long long*>(o + 48) = data;
    *reinterpret_cast<uint32_t*>(o + 56) = 0;            // hash seed
    *reinterpret_cast<uint32_t*>(o + 60) = 0;            // reserved
    for (unsigned long long x = raw; x < meta; ++x) o[x] = 0;
  }
}

__global__ void __launch_bounds__(kCT) gather_kernel(CompactParams p) {
  __shared__ uint4 recs[1 << kTileLog];
  __shared__ unsigned long long wtot[kCT / 32];
  const Geo& g = p.g;
  const uint32_t count = *(volatile uint32_t*)&p.tot->wl_count[0];
  const unsigned long long nF_tot = p.tot->nF;
  uint8_t* const ent_f = p.out + 64;
  uint8_t* const ent_s = p.out + 64 + 4 * nF_tot;
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;

  for (uint32_t w = blockIdx.x; w < count; w += gridDim.x) {
    const uint32_t T = p.wl0[w];
    const uint4 cnt = p.tilecnt[T];
    const uint32_t nF = cnt.x, nS = cnt.y;
    if (nF + nS == 0) continue;   // uniform across the CTA
    const uint4 off = p.toff[T];
    const unsigned long long doff = (unsigned long long)off.z | ((unsigned long long)off.w << 32);
    const uint4* src = p.scratch + ((uint64_t)T << g.t0);
    for (uint32_t i = threadIdx.x; i < nF + nS; i += kCT) recs[i] = src[i];
    __syncthreads();
    // metadata entries (R13): FIRST = u32 node; SHIFT = u32 node, u32 src node, u32 src ckpt
    for (uint32_t i = threadIdx.x; i < nF; i += kCT)
      *reinterpret_cast<uint32_t*>(ent_f + 4ull * (off.x + i)) = recs[i].x;
    for (uint32_t i = threadIdx.x; i < nS; i += kCT) {
      uint32_t* e = reinterpret_cast<uint32_t*>(ent_s + 12ull * (off.y + i));
      const uint4 r = recs[nF + i];
      e[0] = r.x; e[1] = r.y; e[2] = r.z;
    }
    // FIRST regions: global data offset and source offset, for the data pass (KD)
    unsigned long long carry = doff;
    for (uint32_t b0 = 0; b0 < nF; b0 += kCT) {
      const uint32_t i = b0 + threadIdx.x;
      unsigned long long len = 0, s0 = 0;
      if (i < nF) {
        const uint32_t node = recs[i].x;
        const int depth = 31 - __clz(node + 1);
        const int L = g.h - depth;
        uint64_t lo, hi;
        chunk_range(g, L, (uint64_t)node + 1 - (1ull << depth), lo, hi);
        len = range_bytes(g, lo, hi);
        s0 = lo * (unsigned long long)g.C;
      }
      unsigned long long incl = len;
      for (int o = 1; o < 32; o <<= 1) {
        const unsigned long long u = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += u;
      }
      if (lane == 31) wtot[wid] = incl;
      __syncthreads();
      unsigned long long wo = 0, bt = 0;
      for (int k = 0; k < kCT / 32; ++k) {
        if (k < wid) wo += wtot[k];
        bt += wtot[k];
      }
      if (i < nF) {
        p.freg_off[off.x + i] = carry + wo + incl - len;
        p.freg_src[off.x + i] = s0;
      }
      carry += bt;
      __syncthreads();
    }
    __syncthreads();   // recs[] is reused by the next tile
  }
}

// KD: copy all first-occurrence bytes into the data section. Each warp owns an 8-KiB
// segment of the data stream, finds the FIRST region holding the segment start by
// binary search once, then walks forward with coalesced 16-byte loads/stores.
constexpr unsigned long long kSeg = 8192;

__global__ void __launch_bounds__(kCT) data_kernel(CompactParams p) {
  const unsigned long long D = p.tot->data_bytes;
  const unsigned long long nF = p.tot->nF;
  if (D == 0) return;
  uint8_t* const dat = p.out + p.tot->meta_bytes;
  const int lane = threadIdx.x & 31;
  const unsigned long long nseg = (D + kSeg - 1) / kSeg;
  const unsigned long long wglobal = ((unsigned long long)blockIdx.x * kCT + threadIdx.x) >> 5;
  const unsigned long long nwarps = ((unsigned long long)gridDim.x * kCT) >> 5;
  for (unsigned long long sg = wglobal; sg < nseg; sg += nwarps) {
    const unsigned long long s0 = sg * kSeg;
    unsigned long long lo = 0, hi = nF;            // last region with off <= s0
    while (hi - lo > 1) {
      const unsigned long long mid = (lo + hi) >> 1;
      if (__ldg(p.freg_off + mid) <= s0) lo = mid; else hi = mid;
    }
    unsigned long long r = lo;
    unsigned long long next = (r + 1 < nF) ? __ldg(p.freg_off + r + 1) : ~0ull;
    const unsigned long long send = (s0 + kSeg < D) ? s0 + kSeg : D;
    for (unsigned long long o = s0 + 16ull * lane; o < send; o += 512) {
      while (o >= next) {
        ++r;
        next = (r + 1 < nF) ? __ldg(p.freg_off + r + 1) : ~0ull;
      }
      const unsigned long long s = __ldg(p.freg_src + r) + (o - __ldg(p.freg_off + r));
      uint8_t* d = dat + o;
      if (o + 16 <= D) {
        *reinterpret_cast<uint4*>(d) = __ldg(reinterpret_cast<const uint4*>(p.buf + s));
      } else {
        for (unsigned long long b = 0; b < D - o; ++b) d[b] = p.buf[s + b];
      }
    }
  }
}

cudaError_t launch_compact(const CompactParams& p, int num_sms, cudaStream_t st) {
  const unsigned nblk = (unsigned)((p.n_tiles + kTilesPerBlock - 1) / kTilesPerBlock);
  reduce_kernel<<<nblk, kCT, 0, st>>>(p);
  offsets_kernel<<<nblk, kCT, 0, st>>>(p);
  uint64_t grid = (uint64_t)num_sms * 4;
  if (grid > p.n_tiles) grid = p.n_tiles;
  gather_kernel<<<(unsigned)grid, kCT, 0, st>>>(p);
  data_kernel<<<(unsigned)(num_sms * 8), kCT, 0, st>>>(p);
  return cudaGetLastError();
}

}  // namespace ckpt
