// dev.cuh — device building blocks of the sm_100a de-duplication path.
//
// "P:n" = /root/reference/PAPER.md line n; "Rk" = reading k in DESIGN.md §3.
// Nothing here is shared with oracle/ (the CPU checker); this is the GPU's own
// implementation of MurmurHash3_x64_128, the tree geometry (R3) and the
// open-addressing digest table that holds the historical record.
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

namespace ckpt {

// ------------------------------------------------------------------ labels
// Alg.1 labels + DONE (R8: mixed node whose roots were already saved)
// + ABSENT (a virtual tree slot that holds no node, see geometry below).
enum : uint8_t { L_ABSENT = 0, L_FIRST = 1, L_FIXED = 2, L_SHIFT = 3, L_DONE = 4 };

struct __align__(16) Digest {
  uint64_t lo, hi;  // h1, h2 of MurmurHash3_x64_128; bytes h1 LE || h2 LE (R1)
};

__device__ __forceinline__ bool operator==(const Digest& a, const Digest& b) { return a.lo == b.lo && a.hi == b.hi; }

// ------------------------------------------------------------------ MurmurHash3_x64_128
namespace mm {
constexpr uint64_t c1 = 0x87c37b91114253d5ull;
constexpr uint64_t c2 = 0x4cf5ad432745937full;

// 64-bit rotate as two 32-bit funnel shifts (SHF.L.W), r in 1..63 (compile-time).
template <int R>
__device__ __forceinline__ uint64_t rotl(uint64_t x) {
  const uint32_t lo = (uint32_t)x, hi = (uint32_t)(x >> 32);
  constexpr unsigned sh = R < 32 ? (unsigned)R : (unsigned)(R - 32);
  uint32_t nlo, nhi;
  if (R < 32) {
    nhi = __funnelshift_l(lo, hi, sh);
    nlo = __funnelshift_l(hi, lo, sh);
  } else {
    nhi = __funnelshift_l(hi, lo, sh);
    nlo = __funnelshift_l(lo, hi, sh);
  }
  return ((uint64_t)nhi << 32) | nlo;
}
__device__ __forceinline__ uint64_t rotl(uint64_t x, int r) { return (x << r) | (x >> (64 - r)); }

// x * C mod 2^64 (C a compile-time constant)
template <uint64_t C>
__device__ __forceinline__ uint64_t mulc(uint64_t x) {
  const uint32_t lo = (uint32_t)x, hi = (uint32_t)(x >> 32);
#ifndef CKPT_MULC_WIDE
  // lo*lo as mul.lo / mul.hi and the high word accumulated through two mad.lo (no 64-bit
  // IMAD.WIDE, no separate add): measured 4-7 % faster K1 at C = 32 / 64, where hashing is
  // the bound, and neutral at C >= 128 (memory-bound)
  uint32_t wlo, whi, h;
  asm("mul.lo.u32 %0, %3, %4;\n\t"
      "mul.hi.u32 %1, %3, %4;\n\t"
      "mad.lo.u32 %2, %5, %4, %1;\n\t"
      "mad.lo.u32 %2, %3, %6, %2;"
      : "=r"(wlo), "=r"(whi), "=r"(h)
      : "r"(lo), "n"((uint32_t)C), "r"(hi), "n"((uint32_t)(C >> 32)));
  return ((uint64_t)h << 32) | wlo;
#else
  const uint64_t w = (uint64_t)lo * (uint32_t)C;
  const uint32_t h = (uint32_t)(w >> 32) + hi * (uint32_t)C + lo * (uint32_t)(C >> 32);
  return ((uint64_t)h << 32) | (uint32_t)w;
#endif
}

__device__ __forceinline__ uint64_t fmix(uint64_t k) {
  k ^= k >> 33;
  k = mulc<0xff51afd7ed558ccdull>(k);
  k ^= k >> 33;
  k = mulc<0xc4ceb9fe1a85ec53ull>(k);
  k ^= k >> 33;
  return k;
}

// One 16-byte body block (k1 = bytes 0..7 LE, k2 = bytes 8..15 LE).
__device__ __forceinline__ void block(uint64_t& h1, uint64_t& h2, uint64_t k1, uint64_t k2) {
  k1 = mulc<c1>(k1); k1 = rotl<31>(k1); k1 = mulc<c2>(k1); h1 ^= k1;
  h1 = rotl<27>(h1); h1 += h2; h1 = h1 * 5 + 0x52dce729ull;
  k2 = mulc<c2>(k2); k2 = rotl<33>(k2); k2 = mulc<c1>(k2); h2 ^= k2;
  h2 = rotl<31>(h2); h2 += h1; h2 = h2 * 5 + 0x38495ab5ull;
}

// Tail of 1..15 bytes already packed little-endian into t1 (bytes 0..7) / t2 (8..14).
__device__ __forceinline__ void tail(uint64_t& h1, uint64_t& h2, uint64_t t1, uint64_t t2, unsigned rem) {
  if (rem > 8) { t2 = mulc<c2>(t2); t2 = rotl<33>(t2); t2 = mulc<c1>(t2); h2 ^= t2; }
  if (rem > 0) { t1 = mulc<c1>(t1); t1 = rotl<31>(t1); t1 = mulc<c2>(t1); h1 ^= t1; }
}

__device__ __forceinline__ Digest finish(uint64_t h1, uint64_t h2, uint64_t len) {
  h1 ^= len; h2 ^= len;
  h1 += h2; h2 += h1;
  h1 = fmix(h1); h2 = fmix(h2);
  h1 += h2; h2 += h1;
  return Digest{h1, h2};
}

// Internal Merkle node: MMH3(T[l] || T[r]) over 32 bytes, seed 0 (R2).
__device__ __forceinline__ Digest node(const Digest& l, const Digest& r) {
  uint64_t h1 = 0, h2 = 0;
  block(h1, h2, l.lo, l.hi);
  block(h1, h2, r.lo, r.hi);
  return finish(h1, h2, 32);
}
}  // namespace mm

// ------------------------------------------------------------------ geometry (R3)
// The heap tree of N = 2n-1 nodes with the in-order leaf rotation is handled as a
// "virtual perfect tree" of height h = ceil(log2 n): virtual position j at height L
// is heap node (2^(h-L) - 1) + j and covers virtual leaf slots [j 2^L, (j+1) 2^L).
// The m = 2n - 2^h leaves of depth h are chunks 0..m-1 at height 0; the remaining
// n - m/2 ... leaves sit at height 1, positions j >= m/2, chunk j + m/2. Virtual
// slots j >= m at height 0 hold no node (ABSENT). For n = 2^h, m = n.
struct Geo {
  uint64_t B;     // buffer bytes
  uint64_t n;     // leaves (chunks)
  uint64_t m;     // leaves at depth h
  uint32_t C;     // chunk bytes
  int h;          // tree height
  int t0;         // log2 of stage-0 tile (virtual leaf slots per tile)
  uint32_t k;     // checkpoint id (R19)
  uint32_t epoch; // k + 1, tags per-checkpoint dirty marks
};

__device__ __forceinline__ uint64_t vpos_of_chunk(const Geo& g, uint64_t c) { return c < g.m ? c : g.m + 2 * (c - g.m); }

__device__ __forceinline__ uint32_t node_id(const Geo& g, int L, uint64_t j) {
  return (uint32_t)(((1ull << (g.h - L)) - 1) + j);
}

__device__ __forceinline__ uint32_t node_of_chunk(const Geo& g, uint64_t c) {
  return c < g.m ? node_id(g, 0, c) : node_id(g, 1, c - g.m / 2);
}

__device__ __forceinline__ uint64_t chunk_of_vslot(const Geo& g, uint64_t v) { return v <= g.m ? v : g.m + (v - g.m) / 2; }

// chunk range [lo, hi) of virtual position (L, j)
__device__ __forceinline__ void chunk_range(const Geo& g, int L, uint64_t j, uint64_t& lo, uint64_t& hi) {
  lo = chunk_of_vslot(g, j << L);
  hi = chunk_of_vslot(g, (j + 1) << L);
}

// A stage-0 tree tile is FULL when every one of its leaves is a candidate (non-FIXED):
// only then can its root be FIRST or SHIFT (Alg.1: a parent is FIRST / SHIFT only if
// both children are). tcc = candidate leaves counted by K1/K1t.
__device__ __forceinline__ bool tile_full(const Geo& g, const uint32_t* tcc, uint64_t T) {
  uint64_t lo, hi;
  chunk_range(g, g.t0, T, lo, hi);
  return (uint64_t)__ldcg(tcc + T) == hi - lo;
}

__device__ __forceinline__ uint64_t range_bytes(const Geo& g, uint64_t lo, uint64_t hi) {
  uint64_t e = hi * (uint64_t)g.C;
  if (e > g.B) e = g.B;
  return e - lo * (uint64_t)g.C;
}

// ------------------------------------------------------------------ record table
// Open addressing, linear probing, 32-byte slots (one DRAM sector): 128-bit key +
// packed value (ckpt << 32 | node) — Alg.1's (node, chkptID) entry. The value
// only ever decreases (atomicMin), which realises R6: among same-checkpoint duplicates
// the minimum node id wins; entries of earlier checkpoints (smaller ckpt) never change.
struct __align__(32) Slot {
  unsigned long long klo, khi, val, pad;
};
constexpr unsigned long long kEmpty = ~0ull;

__device__ __forceinline__ uint64_t slot_home(uint64_t klo, uint64_t cap) { return __umul64hi(klo, cap); }

// The whole 32-B slot (key and value) in ONE 256-bit load (LDG.E.ENL2.256, sm_100). Two
// loads of the same sector (key, then value) cost two random DRAM accesses when the slot
// is not in L2: tools/rand_probe.cu measured 19.6 G slot reads/s with two loads against
// 38.8 G/s with one, over a 2-GiB table (profiles/rand_probe_r2.txt). Key and value were
// never read as one atomic unit (a concurrent claim can be seen torn), and the callers
// handle that: a half equal to EMPTY sends the insert to the CAS, and a value still EMPTY
// after its key was claimed reads as "not final" (phase 2 re-reads it).
__device__ __forceinline__ void ld_slot_relaxed(const Slot* s, unsigned long long& lo, unsigned long long& hi,
                                                unsigned long long& val) {
  [[maybe_unused]] unsigned long long pad;
  asm volatile("ld.relaxed.gpu.global.v4.u64 {%0, %1, %2, %3}, [%4];"
               : "=l"(lo), "=l"(hi), "=l"(val), "=l"(pad)
               : "l"(s)
               : "memory");
}

// Same, through the L2-only path, for tables with no concurrent writer (phase 3 lookups).
__device__ __forceinline__ void ld_slot_cg(const Slot* s, unsigned long long& lo, unsigned long long& hi,
                                           unsigned long long& val) {
  [[maybe_unused]] unsigned long long pad;
  asm volatile("ld.global.cg.v4.u64 {%0, %1, %2, %3}, [%4];" : "=l"(lo), "=l"(hi), "=l"(val), "=l"(pad) : "l"(s));
}

__device__ __forceinline__ unsigned long long ld_val_relaxed(const Slot* s) {
  unsigned long long v;
  asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(&s->val) : "memory");
  return v;
}

// 128-bit compare-and-swap (sm_90+: ATOMG.E.CAS.128). Returns the previous key.
__device__ __forceinline__ void cas128(Slot* s, unsigned long long cmp_lo, unsigned long long cmp_hi,
                                       unsigned long long new_lo, unsigned long long new_hi,
                                       unsigned long long& old_lo, unsigned long long& old_hi) {
  asm volatile(
      "{\n\t.reg .b128 d, c, v;\n\t"
      "mov.b128 c, {%2, %3};\n\t"
      "mov.b128 v, {%4, %5};\n\t"
      "atom.relaxed.gpu.global.cas.b128 d, [%6], c, v;\n\t"
      "mov.b128 {%0, %1}, d;\n\t}"
      : "=l"(old_lo), "=l"(old_hi)
      : "l"(cmp_lo), "l"(cmp_hi), "l"(new_lo), "l"(new_hi), "l"(s)
      : "memory");
}

// Find-or-claim the slot of key d. Safe against concurrent inserters: a plain read is
// trusted only when it shows a complete key with no all-ones half (a torn read of a
// slot being claimed always shows one EMPTY half); otherwise the CAS decides. The value
// is read in the same round trip (both loads in flight): *val_seen is the slot's value
// as read when the key was found by the plain read, else kEmpty.
// Returns the slot index; *claimed = true if this call created the key.
__device__ __forceinline__ uint64_t table_find_or_claim(Slot* tab, uint64_t cap, const Digest& d, bool* claimed,
                                                        unsigned long long* val_seen = nullptr) {
  uint64_t s = slot_home(d.lo, cap);
  *claimed = false;
  if (val_seen) *val_seen = kEmpty;
  for (;;) {
    Slot* p = tab + s;
    unsigned long long lo, hi, v;
    ld_slot_relaxed(p, lo, hi, v);
    if (lo == d.lo && hi == d.hi && lo != kEmpty && hi != kEmpty) {
      if (val_seen) *val_seen = v;
      return s;
    }
    if (lo == kEmpty || hi == kEmpty) {
      unsigned long long olo, ohi;
      cas128(p, kEmpty, kEmpty, d.lo, d.hi, olo, ohi);
      if (olo == kEmpty && ohi == kEmpty) { *claimed = true; return s; }
      if (olo == d.lo && ohi == d.hi) return s;
    }
    if (++s == cap) s = 0;
  }
}

// Find-or-claim by CAS first (no plain read): one round trip when the key is new, which
// is the common case after checkpoint 0; hot repeated keys should use the read-first form.
__device__ __forceinline__ uint64_t table_claim_cas(Slot* tab, uint64_t cap, const Digest& d, bool* claimed) {
  uint64_t s = slot_home(d.lo, cap);
  for (;;) {
    unsigned long long olo, ohi;
    cas128(tab + s, kEmpty, kEmpty, d.lo, d.hi, olo, ohi);
    if (olo == kEmpty && ohi == kEmpty) { *claimed = true; return s; }
    if (olo == d.lo && ohi == d.hi) { *claimed = false; return s; }
    if (++s == cap) s = 0;
  }
}

// Insert-or-min: Map.insert(digest, entry) of Alg.1 l.7 with the R6 tie-break. The value
// only decreases, so a value already <= packed (an entry of an earlier checkpoint, the
// common case for temporal duplicates) needs no atomic at all.
// *seen_out: the value observed when the key already existed (kEmpty when this call claimed
// it); a value below (ckpt k) << 32 is an entry of an earlier checkpoint and final.
__device__ __forceinline__ uint64_t table_insert_min(Slot* tab, uint64_t cap, const Digest& d, unsigned long long packed,
                                                    bool* claimed, bool cas_first, unsigned long long* seen_out) {
  if (cas_first) {
    const uint64_t s = table_claim_cas(tab, cap, d, claimed);
    Slot* p = tab + s;
    const unsigned long long v = *claimed ? kEmpty : ld_val_relaxed(p);
    if (*claimed || v > packed) atomicMin(&p->val, packed);
    *seen_out = v;
    return s;
  }
  unsigned long long seen;
  const uint64_t s = table_find_or_claim(tab, cap, d, claimed, &seen);
  Slot* p = tab + s;
  if (*claimed || seen > packed) atomicMin(&p->val, packed);
  *seen_out = *claimed ? kEmpty : seen;
  return s;
}

// Lookup in a table with no concurrent writers (phase 3, Alg.1 l.39). Returns the
// packed value or kEmpty when absent.
__device__ __forceinline__ unsigned long long table_lookup(const Slot* tab, uint64_t cap, const Digest& d) {
  uint64_t s = slot_home(d.lo, cap);
  for (;;) {
    unsigned long long klo, khi, val;
    ld_slot_cg(tab + s, klo, khi, val);   // key and value: one sector, one load
    if (klo == d.lo && khi == d.hi) return val;
    if (klo == kEmpty && khi == kEmpty) return kEmpty;
    if (++s == cap) s = 0;
  }
}

// Lookup continuing at slot s (the caller already checked the home slot).
__device__ __forceinline__ unsigned long long table_lookup_from(const Slot* tab, uint64_t cap, const Digest& d, uint64_t s) {
  for (;;) {
    unsigned long long klo, khi, val;
    ld_slot_cg(tab + s, klo, khi, val);   // key and value: one sector, one load
    if (klo == d.lo && khi == d.hi) return val;
    if (klo == kEmpty && khi == kEmpty) return kEmpty;
    if (++s == cap) s = 0;
  }
}

__device__ __forceinline__ unsigned long long pack_entry(uint32_t ckpt, uint32_t node) {
  return ((unsigned long long)ckpt << 32) | node;
}

}  // namespace ckpt
