// oracle/murmur3_ref.cpp — TEST INFRASTRUCTURE ONLY (see oracle/README.md).
//
// Reference MurmurHash3_x64_128, the "128-bit Murmur3 [1]" of PAPER.md P:174
// (ref. [1] = Appleby, SMHasher & MurmurHash). Written out plainly from
// the public-domain algorithm: 16-byte body blocks, a 0..15-byte tail, then the
// length mix and fmix64 finalisation. Byte order: the digest is h1 (little-endian
// u64) followed by h2 (little-endian u64) — DESIGN.md reading R1.
//
// Pinned by tests/test_oracle_murmur.py against the SMHasher VerificationTest
// value 0x6384BA69 and published vectors (tests/golden/murmur3_vectors.txt).
//
// Shares no code with the CUDA path (paper_conf_icpp_tanlmtmbctn23_b200/csrc).

#include <cstdint>
#include <cstring>

namespace oracle {

static inline uint64_t rotl64(uint64_t x, int r) { return (x << r) | (x >> (64 - r)); }

static inline uint64_t fmix64(uint64_t k) {
  k ^= k >> 33;
  k *= 0xff51afd7ed558ccdULL;
  k ^= k >> 33;
  k *= 0xc4ceb9fe1a85ec53ULL;
  k ^= k >> 33;
  return k;
}

static inline uint64_t load_le64(const uint8_t* p) {
  uint64_t v = 0;
  for (int i = 7; i >= 0; --i) v = (v << 8) | p[i];
  return v;
}

static inline void store_le64(uint8_t* p, uint64_t v) {
  for (int i = 0; i < 8; ++i) { p[i] = (uint8_t)(v & 0xff); v >>= 8; }
}

// MurmurHash3_x64_128(key, len, seed) -> out[16] = h1 LE || h2 LE.
void mmh3_x64_128(const void* key, uint64_t len, uint32_t seed, uint8_t out[16]) {
  const uint8_t* data = static_cast<const uint8_t*>(key);
  const uint64_t nblocks = len / 16;
  uint64_t h1 = seed, h2 = seed;
  const uint64_t c1 = 0x87c37b91114253d5ULL;
  const uint64_t c2 = 0x4cf5ad432745937fULL;

  // body
  for (uint64_t i = 0; i < nblocks; ++i) {
    uint64_t k1 = load_le64(data + 16 * i);
    uint64_t k2 = load_le64(data + 16 * i + 8);
    k1 *= c1; k1 = rotl64(k1, 31); k1 *= c2; h1 ^= k1;
    h1 = rotl64(h1, 27); h1 += h2; h1 = h1 * 5 + 0x52dce729;
    k2 *= c2; k2 = rotl64(k2, 33); k2 *= c1; h2 ^= k2;
    h2 = rotl64(h2, 31); h2 += h1; h2 = h2 * 5 + 0x38495ab5;
  }

  // tail: bytes 8..14 go to k2, bytes 0..7 to k1 (little-endian within each)
  const uint8_t* tail = data + 16 * nblocks;
  const unsigned rem = (unsigned)(len & 15);
  uint64_t k1 = 0, k2 = 0;
  for (unsigned b = rem; b > 8; --b) k2 ^= (uint64_t)tail[b - 1] << (8 * (b - 9));
  if (rem > 8) { k2 *= c2; k2 = rotl64(k2, 33); k2 *= c1; h2 ^= k2; }
  for (unsigned b = (rem < 8 ? rem : 8); b > 0; --b) k1 ^= (uint64_t)tail[b - 1] << (8 * (b - 1));
  if (rem > 0) { k1 *= c1; k1 = rotl64(k1, 31); k1 *= c2; h1 ^= k1; }

  // finalisation (the reference xors in the length as a signed int; identical
  // for every length this project uses, < 2^31)
  h1 ^= len; h2 ^= len;
  h1 += h2; h2 += h1;
  h1 = fmix64(h1); h2 = fmix64(h2);
  h1 += h2; h2 += h1;
  store_le64(out, h1);
  store_le64(out + 8, h2);
}

}  // namespace oracle
