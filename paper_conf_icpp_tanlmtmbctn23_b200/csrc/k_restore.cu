// k_restore.cu — restore scatter (reading R16), direct form.
//
// "To restore a checkpoint from the differences, it is enough to start from the
// first-time occurrences, then fill the fixed duplicates and finally assemble the
// shifted duplicates from the corresponding checkpoint ID (which can be a previous
// checkpoint or the current checkpoint to be restored)".
//
// Replaying diffs 0..id writes every chunk once per diff that touches it, and the LAST
// such diff wins: a FIXED chunk of diff c keeps what an earlier diff wrote. So the result
// is, per chunk, the bytes of the latest diff c <= id whose regions cover it, and every
// chunk is covered by diff 0 (no FIXED leaf at checkpoint 0, R5). The restore is therefore
// CHUNK-MAJOR: per diff, newest first, claim_kernel records in owner[chunk] the device
// address of the chunk's bytes unless a newer diff already claimed it (8 B per covered
// chunk); then ONE copy_kernel writes every output chunk once from its owner, coalesced on
// the output side — B bytes written, at most B read, instead of one copy per diff.
//
// Per diff, a restore plan is built once and cached (diffs are immutable):
//   FIRST: Flo[r] (first chunk of region r), Foff[r] (its offset in the data section)
//   SHIFT: Slo[r] (first chunk), Soff[r] (exclusive scan of byte lengths, Soff[nS] = total),
//          Ssrc[r] (device address of the source bytes: v's bytes inside the FIRST region of
//          diff c' holding v's first chunk, binary search over c''s sorted region starts)
//   segment maps Fseg / Sseg (region holding the first byte of every 2-KB stream segment)
//   claim list Cch / Csrc: the chunk and source address of every C-byte step of the FIRST
//          then SHIFT stream (claimlist_kernel), so a warm claim is two coalesced loads.
#include "kernels.h"
#include "tma.cuh"

namespace ckpt {

namespace {
constexpr int kRT = 256;
constexpr int kScanPer = 4;
constexpr uint64_t kScanBlock = kRT * kScanPer;   // 1024 elements per scan block

__device__ __forceinline__ void node_range(const Geo& g, uint32_t node, uint64_t& lo, uint64_t& hi) {
  const int depth = 31 - __clz(node + 1);
  chunk_range(g, g.h - depth, (uint64_t)node + 1 - (1ull << depth), lo, hi);
}

__device__ __forceinline__ uint32_t rd32(const uint8_t* p) { return *reinterpret_cast<const uint32_t*>(p); }

// ------------------------------------------------------------------ scan
__global__ void __launch_bounds__(kRT) scan_block_kernel(const unsigned long long* in, unsigned long long* out,
                                                        uint64_t count, unsigned long long* bsum) {
  __shared__ unsigned long long wt[kRT / 32];
  const uint64_t base = (uint64_t)blockIdx.x * kScanBlock + threadIdx.x * kScanPer;
  unsigned long long v[kScanPer], mine = 0;
  for (int i = 0; i < kScanPer; ++i) {
    v[i] = (base + i < count) ? in[base + i] : 0ull;
    mine += v[i];
  }
  const int lane = threadIdx.x & 31, wid = threadIdx.x >> 5;
  unsigned long long incl = mine;
  for (int o = 1; o < 32; o <<= 1) {
    const unsigned long long u = __shfl_up_sync(0xffffffffu, incl, o);
    if (lane >= o) incl += u;
  }
  if (lane == 31) wt[wid] = incl;
  __syncthreads();
  unsigned long long off = 0, tot = 0;
  for (int i = 0; i < kRT / 32; ++i) {
    if (i < wid) off += wt[i];
    tot += wt[i];
  }
  off += incl - mine;
  for (int i = 0; i < kScanPer; ++i) {
    if (base + i < count) out[base + i] = off;
    off += v[i];
  }
  if (threadIdx.x == 0 && bsum) bsum[blockIdx.x] = tot;
}

__global__ void scan_add_kernel(unsigned long long* out, uint64_t count, const unsigned long long* boff) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < count) out[i] += boff[i / kScanBlock];
}

// ------------------------------------------------------------------ restore kernels
__global__ void prepare_first_kernel(Geo g, RestoreDiff d, unsigned long long* len) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= d.nF) return;
  const uint32_t node = rd32(d.base + 64 + 4 * i);
  uint64_t lo, hi;
  node_range(g, node, lo, hi);
  d.Flo[i] = lo;
  len[i] = range_bytes(g, lo, hi);
}

constexpr uint32_t kSegBytes = 2048;   // segment map granularity of a diff's byte streams

// first index r in [0, nr) with off[r] > x, minus one (off[0] == 0 <= x)
__device__ __forceinline__ uint64_t region_at(const unsigned long long* off, uint64_t nr, unsigned long long x) {
  uint64_t lo = 0, hi = nr;
  while (hi - lo > 1) {
    const uint64_t mid = (lo + hi) >> 1;
    if (__ldg(off + mid) <= x) lo = mid; else hi = mid;
  }
  return lo;
}

// ---- chunk-major restore: claim, then one copy pass
// claimlist_kernel (plan building, once per diff): one thread per chunk of the diff's FIRST
// stream then SHIFT stream writes the chunk's id and the device address of its bytes.
__global__ void __launch_bounds__(kRT) claimlist_kernel(Geo g, RestoreDiff d) {
  const unsigned long long C = g.C;
  const uint64_t nxF = (d.data_bytes + C - 1) / C, nxS = (d.shift_bytes + C - 1) / C;
  const uint8_t* data = d.base + d.meta_bytes;
  for (uint64_t t = (uint64_t)blockIdx.x * kRT + threadIdx.x; t < nxF + nxS; t += (uint64_t)gridDim.x * kRT) {
    const bool first = t < nxF;
    const unsigned long long o = (first ? t : t - nxF) * C;   // stream offset (every region but the
                                                              // stream's last is whole chunks)
    const unsigned long long* off = first ? d.Foff : d.Soff;
    const unsigned long long* seg = first ? d.Fseg : d.Sseg;
    const uint64_t nr = first ? d.nF : d.nS;
    const uint64_t sg = o / kSegBytes;
    // last region r with off[r] <= o, between the regions holding this segment's first byte
    // and the next segment's
    uint64_t lo = __ldg(seg + sg), hi = __ldg(seg + sg + 1) + 1;
    if (hi > nr) hi = nr;
    while (hi - lo > 1) {
      const uint64_t mid = (lo + hi) >> 1;
      if (__ldg(off + mid) <= o) lo = mid; else hi = mid;
    }
    const unsigned long long rel = o - __ldg(off + lo);
    d.Cch[t] = (uint32_t)((first ? __ldg(d.Flo + lo) : __ldg(d.Slo + lo)) + rel / C);
    // Ssrc == 0: a source node whose bytes are no first-occurrence data (R25), resolved
    // chunk by chunk by resolve_kernel
    const unsigned long long ss = first ? 0ull : __ldg(d.Ssrc + lo);
    d.Csrc[t] = first ? (unsigned long long)(data + o) : (ss ? ss + rel : 0ull);
  }
}

// resolve_kernel (R25, plan building of a SHIFT-insert lineage): a SHIFT claim step whose
// source node v of checkpoint c' holds no first-occurrence data takes the address of the
// corresponding chunk x of checkpoint c': inside a FIRST region of diff c', its data; inside
// a SHIFT region of diff c', that step's own resolved address in c''s claim list. v's range
// is non-FIXED in c' (every leaf below v was a shifted duplicate), so one of the two holds.
// For c' = this diff the source's steps belong to smaller regions: one pass resolves one
// more level; steps still unresolved after the last pass flag the chain as malformed.
__device__ __forceinline__ uint64_t last_le(const unsigned long long* a, uint64_t n, unsigned long long x) {
  uint64_t lo = 0, hi = n;   // last index with a[i] <= x (a[0] <= x assumed by the caller)
  while (hi - lo > 1) {
    const uint64_t mid = (lo + hi) >> 1;
    if (a[mid] <= x) lo = mid; else hi = mid;
  }
  return lo;
}

__global__ void __launch_bounds__(kRT) resolve_kernel(Geo g, RestoreDiff d, const RestoreDiff* chain, int last, int* err) {
  const unsigned long long C = g.C;
  const uint64_t nxF = (d.data_bytes + C - 1) / C, nxS = (d.shift_bytes + C - 1) / C;
  for (uint64_t t = nxF + (uint64_t)blockIdx.x * kRT + threadIdx.x; t < nxF + nxS; t += (uint64_t)gridDim.x * kRT) {
    if (d.Csrc[t]) continue;
    const unsigned long long o = (t - nxF) * C;
    const uint64_t r = region_at(d.Soff, d.nS, o);
    const uint8_t* e = d.base + 64 + 4 * d.nF + 12 * r;
    const uint32_t u = rd32(e), v = rd32(e + 4), c2 = rd32(e + 8);
    uint64_t ulo, uhi, vlo, vhi;
    node_range(g, u, ulo, uhi);
    node_range(g, v, vlo, vhi);
    const uint64_t x = vlo + (d.Cch[t] - ulo);
    const RestoreDiff& s = chain[c2 <= d.id ? c2 : d.id];
    unsigned long long addr = 0;
    bool found = false;
    if (s.nF && s.Flo[0] <= x) {
      const uint64_t f = last_le(s.Flo, s.nF, x);
      const unsigned long long fend = f + 1 < s.nF ? s.Foff[f + 1] : s.data_bytes;
      if ((x - s.Flo[f]) * C < fend - s.Foff[f]) {
        addr = (unsigned long long)(s.base + s.meta_bytes + s.Foff[f]) + (x - s.Flo[f]) * C;
        found = true;
      }
    }
    if (!found && s.nS && s.Slo[0] <= x) {
      const uint64_t q = last_le(s.Slo, s.nS, x);
      if ((x - s.Slo[q]) * C < s.Soff[q + 1] - s.Soff[q]) {
        const uint64_t sxF = (s.data_bytes + C - 1) / C;
        addr = s.Csrc[sxF + s.Soff[q] / C + (x - s.Slo[q])];   // 0 while not yet resolved
        found = true;
      }
    }
    if (addr) d.Csrc[t] = addr;
    else if (last || !found || c2 > d.id) atomicExch(err, 1);
  }
}

// claim_kernel (one launch per diff, newest first): the chunk's first claimer (the newest
// diff covering it) records the address of its bytes in owner[chunk]. Regions of one diff
// are disjoint, so a diff never races with itself; diffs run in stream order.
__global__ void __launch_bounds__(kRT) claim_kernel(RestoreDiff d, uint64_t ncl, uint64_t n, unsigned long long* owner) {
  pdl_launch_dependents();
  pdl_wait();   // the newer diffs' claims are complete
  for (uint64_t t = (uint64_t)blockIdx.x * kRT + threadIdx.x; t < ncl; t += (uint64_t)gridDim.x * kRT) {
    const uint32_t ch = __ldg(d.Cch + t);
    const unsigned long long src = __ldg(d.Csrc + t);
    if (ch < n && __ldcg(owner + ch) == 0) owner[ch] = src;   // ch < n: guard against malformed plans
  }
}

// claim_bitmap_kernel: the same for lineages whose newer diffs rewrote many chunks. Whether a
// newer diff owns the chunk is read from a bitmap of claimed chunks (n / 8 bytes, in L2)
// instead of the 8-B owner entry, and the source address is loaded only for a chunk still
// unclaimed: an older diff of a long lineage, most of whose chunks newer diffs rewrote,
// costs 4 B of claim list per covered chunk instead of 20 (restore).
#ifndef CKPT_CLAIM_UNROLL
#define CKPT_CLAIM_UNROLL 8   // claim entries per thread in flight (bitmap claims; 1 / 4 / 8: config 4 at 30 diffs 1.10 / 1.04 / 0.99 ms)
#endif
__global__ void __launch_bounds__(kRT) claim_bitmap_kernel(RestoreDiff d, uint64_t ncl, uint64_t n,
                                                           unsigned long long* owner, int last) {
  constexpr int U = CKPT_CLAIM_UNROLL;
  pdl_launch_dependents();
  pdl_wait();   // the newer diffs' claims are complete
  uint32_t* const claimed = reinterpret_cast<uint32_t*>(owner + n);
  const int lane = threadIdx.x & 31;
  const uint64_t wstride = (uint64_t)gridDim.x * kRT * U;
  // warp-uniform trip count (the bitmap updates are combined across the warp); a warp takes
  // 32 U consecutive entries per round, U per lane in flight (the bitmap reads are L2 round
  // trips that depend on the entry's chunk)
  for (uint64_t base = ((uint64_t)blockIdx.x * kRT + (threadIdx.x & ~31u)) * U; base < ncl; base += wstride) {
    uint32_t ch[U], wd[U];
    unsigned long long src[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const uint64_t t = base + 32 * u + lane;
      ch[u] = t < ncl ? __ldg(d.Cch + t) : 0xFFFFFFFFu;
      if (last && ch[u] < n) src[u] = __ldg(d.Csrc + t);   // the oldest diff: mostly unclaimed
    }
#pragma unroll
    for (int u = 0; u < U; ++u) wd[u] = ch[u] < n ? __ldcg(claimed + (ch[u] >> 5)) : ~0u;   // ch < n: malformed-plan guard
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const bool take = ch[u] < n && !((wd[u] >> (ch[u] & 31)) & 1u);
      if (take) owner[ch[u]] = last ? src[u] : __ldg(d.Csrc + base + 32 * u + lane);
      if (last) continue;   // no later claim pass reads the bitmap
      const uint32_t key = take ? (ch[u] >> 5) : 0xFFFFFFFFu;
      const unsigned grp = __match_any_sync(0xffffffffu, key);
      const uint32_t bits = __reduce_or_sync(grp, take ? 1u << (ch[u] & 31) : 0u);
      if (take && lane == __ffs(grp) - 1) atomicOr(claimed + key, bits);
    }
  }
}

// copy_kernel: the output as a stream of 16-byte units (C is a multiple of 16, so a unit
// never straddles chunks); each unit reads its chunk's owner address, then its 16 bytes.
// kCopyUnroll units per thread are in flight before any store. A chunk no diff claimed
// (impossible for a well-formed lineage: diff 0 covers every chunk) reads as zeros, the
// replay's starting buffer.
#ifndef CKPT_COPY_UNROLL
#define CKPT_COPY_UNROLL 2
#endif
constexpr int kCopyUnroll = CKPT_COPY_UNROLL;   // measured: 2 ~ 1 < 4 < 8 (0.56 / 0.60 / 0.69 ms, config 2)
#ifndef CKPT_COPY_LDG
#define CKPT_COPY_LDG 1
#endif
__global__ void __launch_bounds__(kRT) copy_kernel(Geo g, const unsigned long long* owner, uint8_t* out) {
  pdl_launch_dependents();
  pdl_wait();
  const uint64_t U = g.C / 16;
  const uint64_t nu = (g.B + 15) / 16;
  const uint64_t nth = (uint64_t)gridDim.x * kRT;
  for (uint64_t u0 = (uint64_t)blockIdx.x * kRT + threadIdx.x; u0 < nu; u0 += kCopyUnroll * nth) {
    unsigned long long src[kCopyUnroll];
#pragma unroll
    for (int j = 0; j < kCopyUnroll; ++j) {
      const uint64_t u = u0 + j * nth;
      src[j] = u < nu ? __ldg(owner + u / U) : 0ull;
      if (src[j]) src[j] += (u % U) * 16;
    }
    uint4 v[kCopyUnroll];
#pragma unroll
    for (int j = 0; j < kCopyUnroll; ++j) {
      const uint64_t u = u0 + j * nth;
      v[j] = make_uint4(0, 0, 0, 0);
      if (u >= nu || !src[j]) continue;
      if (16 * u + 16 <= g.B) {
#if CKPT_COPY_LDG
        v[j] = __ldg(reinterpret_cast<const uint4*>(src[j]));
#else
        v[j] = __ldcs(reinterpret_cast<const uint4*>(src[j]));
#endif
      } else {   // the buffer's last, partial unit: only its bytes (the source may end there)
        const uint8_t* sp = reinterpret_cast<const uint8_t*>(src[j]);
        uint32_t w[4] = {0, 0, 0, 0};
        for (uint32_t q = 0; q < (uint32_t)(g.B - 16 * u); ++q) w[q >> 2] |= (uint32_t)sp[q] << (8 * (q & 3));
        v[j] = make_uint4(w[0], w[1], w[2], w[3]);
      }
    }
#pragma unroll
    for (int j = 0; j < kCopyUnroll; ++j) {
      const uint64_t u = u0 + j * nth;
      if (u >= nu) continue;
      if (16 * u + 16 <= g.B) {
        __stcs(reinterpret_cast<uint4*>(out + 16 * u), v[j]);
      } else {
        const uint32_t w[4] = {v[j].x, v[j].y, v[j].z, v[j].w};
        for (uint32_t q = 0; q < (uint32_t)(g.B - 16 * u); ++q) out[16 * u + q] = (uint8_t)(w[q >> 2] >> (8 * (q & 3)));
      }
    }
  }
}

__global__ void prepare_shift_kernel(Geo g, RestoreDiff d, const RestoreDiff* chain, unsigned long long* len, int* err) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i >= d.nS) return;
  const uint8_t* e = d.base + 64 + 4 * d.nF + 12 * i;
  const uint32_t u = rd32(e), v = rd32(e + 4), c2 = rd32(e + 8);
  uint64_t ulo, uhi, vlo, vhi;
  node_range(g, u, ulo, uhi);
  node_range(g, v, vlo, vhi);
  len[i] = range_bytes(g, ulo, uhi);
  d.Slo[i] = ulo;
  // guards (malformed diffs, e.g. a corrupted import): the source checkpoint is in the chain
  // and the source bytes lie inside one FIRST region of its data section; otherwise the
  // plan is flagged and no restore kernel runs
  if (c2 > d.id) { atomicExch(err, 1); d.Ssrc[i] = (unsigned long long)d.base; return; }
  const RestoreDiff& s = chain[c2];
  // FIRST region r of diff c2 with Flo[r] <= vlo (the last such): it contains v. Under the
  // SHIFT-insert variant (R25) v may instead be a node of c2 whose bytes are c2's own
  // regions below it: Ssrc = 0, resolved per chunk after the claim list is built.
  if (s.nF == 0 || !s.Flo) {
    if (!d.composite) atomicExch(err, 1);
    d.Ssrc[i] = d.composite ? 0ull : (unsigned long long)s.base;
    return;
  }
  uint64_t lo = 0, hi = s.nF;
  while (hi - lo > 1) {
    const uint64_t mid = (lo + hi) >> 1;
    if (s.Flo[mid] <= vlo) lo = mid; else hi = mid;
  }
  const unsigned long long rel = (vlo - s.Flo[lo]) * (unsigned long long)g.C;
  const unsigned long long rend = lo + 1 < s.nF ? s.Foff[lo + 1] : s.data_bytes;
  if (s.Flo[lo] > vlo || s.Foff[lo] + rel + range_bytes(g, vlo, vhi) > rend) {
    if (!d.composite) atomicExch(err, 1);
    d.Ssrc[i] = d.composite ? 0ull : (unsigned long long)s.base;
    return;
  }
  d.Ssrc[i] = (unsigned long long)(s.base + s.meta_bytes + s.Foff[lo] + rel);
}

// Basic diffs: every changed chunk is a one-chunk "FIRST region" of the plan.
// popcount per bitmap word, then (after an exclusive scan) the chunk ids of the set bits.
__global__ void basic_count_kernel(const uint8_t* base, uint64_t nwords, unsigned long long* cnt) {
  const uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (w < nwords) cnt[w] = __popc(rd32(base + 64 + 4 * w));
}
__global__ void basic_expand_kernel(Geo g, RestoreDiff d, uint64_t nwords, const unsigned long long* off) {
  const uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (w >= nwords) return;
  uint32_t m = rd32(d.base + 64 + 4 * w);
  unsigned long long r = off[w];
  for (; m && r < d.nF; m &= m - 1, ++r) {   // r < nF: a malformed bitmap cannot overrun
    d.Flo[r] = 32ull * w + (__ffs(m) - 1);
    d.Foff[r] = r * (unsigned long long)g.C;   // only the buffer's last chunk can be short
  }
}

// segment map: region holding the first byte of each 2-KB segment; map[nseg] = nr - 1
__global__ void segmap_kernel(const unsigned long long* off, uint64_t nr, uint64_t nseg, unsigned long long* map) {
  const uint64_t sg = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (sg > nseg) return;
  map[sg] = sg == nseg ? nr - 1 : region_at(off, nr, sg * (unsigned long long)kSegBytes);
}

__global__ void write_total_kernel(unsigned long long* off, const unsigned long long* len, uint64_t n) {
  off[n] = off[n - 1] + len[n - 1];
}
}  // namespace

size_t scan_tmp_bytes_for(uint64_t count) {
  size_t b = 0;
  uint64_t c = count;
  while (c > kScanBlock) {
    const uint64_t nb = (c + kScanBlock - 1) / kScanBlock;
    b += 2 * nb * sizeof(unsigned long long);
    c = nb;
  }
  return b + 256;
}

cudaError_t scan_u64_exclusive(const unsigned long long* in, unsigned long long* out, uint64_t count, void* tmp,
                               size_t tmp_bytes, cudaStream_t st) {
  if (count == 0) return cudaSuccess;
  const uint64_t nb = (count + kScanBlock - 1) / kScanBlock;
  if (nb == 1) {
    scan_block_kernel<<<1, kRT, 0, st>>>(in, out, count, nullptr);
    note_launch();
    return cudaGetLastError();
  }
  unsigned long long* bsum = reinterpret_cast<unsigned long long*>(tmp);
  unsigned long long* boff = bsum + nb;
  const size_t used = 2 * nb * sizeof(unsigned long long);
  if (used > tmp_bytes) return cudaErrorInvalidValue;
  scan_block_kernel<<<(unsigned)nb, kRT, 0, st>>>(in, out, count, bsum);
  note_launch();
  cudaError_t e = scan_u64_exclusive(bsum, boff, nb, boff + nb, tmp_bytes - used, st);
  if (e != cudaSuccess) return e;
  scan_add_kernel<<<(unsigned)((count + 255) / 256), 256, 0, st>>>(out, count, boff);
  note_launch();
  return cudaGetLastError();
}

cudaError_t restore_prepare_first(const Geo& g, RestoreDiff& d, unsigned long long* tmp_len, void* scan_tmp,
                                  size_t scan_tmp_bytes, cudaStream_t st) {
  if (d.nF == 0) return cudaSuccess;
  prepare_first_kernel<<<(unsigned)((d.nF + 255) / 256), 256, 0, st>>>(g, d, tmp_len);
  note_launch();
  return scan_u64_exclusive(tmp_len, d.Foff, d.nF, scan_tmp, scan_tmp_bytes, st);
}

cudaError_t restore_prepare_shift(const Geo& g, RestoreDiff& d, const RestoreDiff* chain_dev, unsigned long long* tmp_len,
                                  int* err, void* scan_tmp, size_t scan_tmp_bytes, cudaStream_t st) {
  if (d.nS == 0) return cudaSuccess;
  prepare_shift_kernel<<<(unsigned)((d.nS + 255) / 256), 256, 0, st>>>(g, d, chain_dev, tmp_len, err);
  note_launch();
  cudaError_t e = scan_u64_exclusive(tmp_len, d.Soff, d.nS, scan_tmp, scan_tmp_bytes, st);
  if (e != cudaSuccess) return e;
  write_total_kernel<<<1, 1, 0, st>>>(d.Soff, tmp_len, d.nS);
  note_launch();
  return cudaGetLastError();
}

cudaError_t restore_prepare_basic(const Geo& g, RestoreDiff& d, uint64_t nwords, unsigned long long* tmp_cnt,
                                  void* scan_tmp, size_t scan_tmp_bytes, cudaStream_t st) {
  if (d.nF == 0) return cudaSuccess;
  const unsigned blocks = (unsigned)((nwords + 255) / 256);
  basic_count_kernel<<<blocks, 256, 0, st>>>(d.base, nwords, tmp_cnt);
  note_launch();
  cudaError_t e = scan_u64_exclusive(tmp_cnt, tmp_cnt + nwords, nwords, scan_tmp, scan_tmp_bytes, st);
  if (e != cudaSuccess) return e;
  basic_expand_kernel<<<blocks, 256, 0, st>>>(g, d, nwords, tmp_cnt + nwords);
  note_launch();
  return cudaGetLastError();
}

__global__ void compare_kernel(const uint4* a, const uint4* b, uint64_t n16, const uint8_t* ta, const uint8_t* tb,
                               uint32_t ntail, int* diff) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint4 x = a[i], y = b[i];
    if (x.x != y.x || x.y != y.y || x.z != y.z || x.w != y.w) *diff = 1;
  }
  if (blockIdx.x == 0 && threadIdx.x < ntail && ta[threadIdx.x] != tb[threadIdx.x]) *diff = 1;
}

cudaError_t device_compare(const void* a, const void* b, uint64_t bytes, int* diff, int num_sms, cudaStream_t st) {
  const uint64_t n16 = bytes / 16;
  compare_kernel<<<num_sms * 4, 256, 0, st>>>(reinterpret_cast<const uint4*>(a), reinterpret_cast<const uint4*>(b), n16,
                                              static_cast<const uint8_t*>(a) + 16 * n16,
                                              static_cast<const uint8_t*>(b) + 16 * n16, (uint32_t)(bytes % 16), diff);
  note_launch();
  return cudaGetLastError();
}

cudaError_t restore_segmaps(RestoreDiff& d, cudaStream_t st) {
  if (d.nF) {
    const uint64_t ns = (d.data_bytes + kSegBytes - 1) / kSegBytes;
    segmap_kernel<<<(unsigned)((ns + 256) / 256), 256, 0, st>>>(d.Foff, d.nF, ns, d.Fseg);
    note_launch();
  }
  if (d.nS) {
    const uint64_t ns = (d.shift_bytes + kSegBytes - 1) / kSegBytes;
    segmap_kernel<<<(unsigned)((ns + 256) / 256), 256, 0, st>>>(d.Soff, d.nS, ns, d.Sseg);
    note_launch();
  }
  return cudaGetLastError();
}

uint64_t restore_segments(uint64_t bytes) { return (bytes + kSegBytes - 1) / kSegBytes; }

static int g_copy_bps = 0, g_claim_bps = 0;   // resident blocks per SM (occupancy, preload_restore)

static uint64_t claim_count(const Geo& g, const RestoreDiff& d) {
  return (d.data_bytes + g.C - 1) / g.C + (d.shift_bytes + g.C - 1) / g.C;
}

cudaError_t restore_claimlist(const Geo& g, const RestoreDiff& d, int num_sms, cudaStream_t st) {
  const uint64_t nx = claim_count(g, d);
  if (nx == 0) return cudaSuccess;
  uint64_t grid = (nx + kRT - 1) / kRT;
  const uint64_t cap = (uint64_t)num_sms * 8;
  if (grid > cap) grid = cap;
  claimlist_kernel<<<(unsigned)grid, kRT, 0, st>>>(g, d);
  note_launch();
  return cudaGetLastError();
}

cudaError_t restore_resolve(const Geo& g, const RestoreDiff& d, const RestoreDiff* chain_dev, int passes, int* err,
                            int num_sms, cudaStream_t st) {
  const uint64_t nx = (d.shift_bytes + g.C - 1) / g.C;
  if (nx == 0) return cudaSuccess;
  uint64_t grid = (nx + kRT - 1) / kRT;
  if (grid > (uint64_t)num_sms * 8) grid = (uint64_t)num_sms * 8;
  for (int i = 0; i < passes; ++i) {
    resolve_kernel<<<(unsigned)grid, kRT, 0, st>>>(g, d, chain_dev, i + 1 == passes ? 1 : 0, err);
    note_launch();
  }
  return cudaGetLastError();
}

cudaError_t restore_claim(const Geo& g, const RestoreDiff& d, unsigned long long* owner, bool bitmap, int num_sms,
                          cudaStream_t st) {
  const uint64_t nx = claim_count(g, d);
  if (nx == 0) return cudaSuccess;
  uint64_t grid = (nx + kRT - 1) / kRT;
  const uint64_t cap = (uint64_t)num_sms * (g_claim_bps > 0 ? g_claim_bps : 4);
  if (grid > cap) grid = cap;
  if (bitmap) {
    grid = std::min<uint64_t>(cap, (nx + kRT * CKPT_CLAIM_UNROLL - 1) / (kRT * CKPT_CLAIM_UNROLL));
    return launch_pdl(claim_bitmap_kernel, (unsigned)grid, kRT, 0, st, d, nx, (uint64_t)g.n, owner, d.id == 0 ? 1 : 0);
  }
  return launch_pdl(claim_kernel, (unsigned)grid, kRT, 0, st, d, nx, (uint64_t)g.n, owner);
}

cudaError_t restore_copy(const Geo& g, const unsigned long long* owner, uint8_t* out, int num_sms, cudaStream_t st) {
  const uint64_t nu = (g.B + 15) / 16;
  uint64_t grid = (nu + kRT * kCopyUnroll - 1) / (kRT * kCopyUnroll);
  // one resident wave: the grid-stride loop gives every block the same share, so blocks
  // beyond what fits would run as a second, mostly idle wave
  const uint64_t cap = (uint64_t)num_sms * (g_copy_bps > 0 ? g_copy_bps : 4);
  if (grid > cap) grid = cap;
  return launch_pdl(copy_kernel, (unsigned)grid, kRT, 0, st, g, owner, out);
}



// Load this file's kernels now (CUDA lazy module loading would otherwise stall the first
// launch of each kernel inside the first checkpoint).
cudaError_t preload_restore() {
  cudaFuncAttributes a;
  cudaError_t e = cudaSuccess;
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, scan_block_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, scan_add_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, prepare_first_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, claim_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, claim_bitmap_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, claimlist_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, copy_kernel);
  if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_copy_bps, copy_kernel, kRT, 0);
  if (e == cudaSuccess) e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&g_claim_bps, claim_kernel, kRT, 0);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, prepare_shift_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, write_total_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, segmap_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, basic_count_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, basic_expand_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, compare_kernel);
  if (e == cudaSuccess) e = cudaFuncGetAttributes(&a, resolve_kernel);
  return e;
}

}  // namespace ckpt
