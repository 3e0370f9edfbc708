// gen.cu — device twins of the seeded workload generators in workloads/__init__.py
// (harness code: no de-duplication arithmetic). Same counter-based hash H, same recipes
// (DESIGN.md §6), so device and host produce identical bytes; libckptgen.so is loaded by
// bench.py / tests to create large checkpoint lineages directly in HBM.
#include <cstdint>
#include <cuda_runtime.h>

#define GEN_API extern "C" __attribute__((visibility("default")))

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t z) {
  z ^= z >> 30;
  z *= 0xBF58476D1CE4E5B9ull;
  z ^= z >> 27;
  z *= 0x94D049BB133111EBull;
  z ^= z >> 31;
  return z;
}
__device__ __forceinline__ uint64_t H1(uint64_t s, uint64_t a) { return splitmix64(s + (a + 1) * 0x9E3779B97F4A7C15ull); }
__device__ __forceinline__ uint64_t H2(uint64_t s, uint64_t a, uint64_t b) { return H1(H1(s, a), b); }
__device__ __forceinline__ uint64_t H3(uint64_t s, uint64_t a, uint64_t b, uint64_t c) { return H1(H2(s, a, b), c); }
__device__ __forceinline__ uint64_t H4(uint64_t s, uint64_t a, uint64_t b, uint64_t c, uint64_t d) {
  return H1(H3(s, a, b, c), d);
}

__device__ __forceinline__ uint32_t geo(uint64_t x) {
  uint32_t c = 0;
  for (int j = 0; j < 32; ++j) {
    if (((x >> (62 - 2 * j)) & 3ull) == 0) break;
    ++c;
  }
  return c;
}

constexpr int kRowOrbits = 73;
constexpr int kRowBytes = 4 * kRowOrbits;
constexpr int kNFreq = 24;
__constant__ int kFreq[kNFreq] = {0, 1, 2, 3, 4, 5, 6, 7, 9, 10, 11, 12, 13, 15, 16, 17, 18, 19, 20, 21, 22, 23, 24, 25};

__global__ void cfg1_init_kernel(uint8_t* buf, uint64_t nbytes, uint64_t seed) {
  const uint64_t nw = (nbytes + 7) / 8;
  for (uint64_t w = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; w < nw; w += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t v = H1(seed, w);
    if (8 * w + 8 <= nbytes) {
      reinterpret_cast<uint64_t*>(buf)[w] = v;
    } else {
      for (uint64_t b = 0; 8 * w + b < nbytes; ++b) buf[8 * w + b] = (uint8_t)(v >> (8 * b));
    }
  }
}

__global__ void cfg1_mutate_kernel(uint8_t* buf, uint64_t nbytes, uint32_t C, uint32_t k, uint64_t seed, uint64_t thr) {
  const uint64_t n = (nbytes + C - 1) / C;
  const uint64_t sk = H1(seed, k);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t u = H1(sk, i);
    if (u >= thr) continue;
    const uint64_t x = u | 1ull;
    const uint64_t off = i * C;
    for (uint64_t b = 0; b < 8 && b < C && off + b < nbytes; ++b) buf[off + b] ^= (uint8_t)(x >> (8 * b));
  }
}

__global__ void cfg2_init_kernel(uint8_t* buf, uint64_t rows, uint64_t seed, uint64_t thr_proto) {
  for (uint64_t r = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; r < rows; r += (uint64_t)gridDim.x * blockDim.x) {
    uint32_t* row = reinterpret_cast<uint32_t*>(buf + r * kRowBytes);   // 292 = 4 * 73: u32-aligned
    for (int j = 0; j < kRowOrbits; ++j) row[j] = 0;
    const bool live = H2(seed, 0, r / 64) >= (1ull << 63);
    if (!live) continue;
    const bool proto = H2(seed, 1, r) < thr_proto;
    const uint64_t P = H2(seed, 2, r) % 256;
    for (int q = 0; q < kNFreq; ++q) row[kFreq[q]] = proto ? geo(H3(seed, 3, P, q)) : geo(H3(seed, 4, r, q));
  }
}

__global__ void zero_kernel(uint8_t* p, uint64_t nbytes) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < nbytes; i += (uint64_t)gridDim.x * blockDim.x)
    p[i] = 0;
}

__global__ void cfg2_mutate_kernel(uint8_t* buf, uint64_t rows, uint32_t k, uint64_t seed, uint64_t thr) {
  const uint64_t total = rows * kNFreq;
  for (uint64_t t = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; t < total; t += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t r = t / kNFreq, q = t % kNFreq;
    if (H3(seed, 5, k, r / 16) >= thr) continue;
    const uint64_t v = H4(seed, 6, k, r, q);
    if (v < (1ull << 62)) {
      uint32_t* row = reinterpret_cast<uint32_t*>(buf + r * kRowBytes);
      row[kFreq[q]] += 1u + (uint32_t)(v & 3ull);
    }
  }
}

unsigned grid_for(uint64_t n) {
  uint64_t b = (n + 255) / 256;
  if (b > 148 * 32) b = 148 * 32;
  return (unsigned)(b ? b : 1);
}

}  // namespace

GEN_API int gen_freq_orbits(int* out) {
  const int f[kNFreq] = {0, 1, 2, 3, 4, 5, 6, 7, 9, 10, 11, 12, 13, 15, 16, 17, 18, 19, 20, 21, 22, 23, 24, 25};
  for (int i = 0; i < kNFreq; ++i) out[i] = f[i];
  return kNFreq;
}

GEN_API int gen_cfg1_initial(void* dev, uint64_t nbytes, uint64_t seed, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cfg1_init_kernel<<<grid_for((nbytes + 7) / 8), 256, 0, st>>>(static_cast<uint8_t*>(dev), nbytes, seed);
  return (int)cudaGetLastError();
}

GEN_API int gen_cfg1_mutate(void* dev, uint64_t nbytes, uint32_t C, uint32_t k, uint64_t seed, uint64_t thr,
                            void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  cfg1_mutate_kernel<<<grid_for((nbytes + C - 1) / C), 256, 0, st>>>(static_cast<uint8_t*>(dev), nbytes, C, k, seed,
                                                                      thr);
  return (int)cudaGetLastError();
}

GEN_API int gen_cfg2_initial(void* dev, uint64_t nbytes, uint64_t seed, uint64_t thr_proto, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const uint64_t rows = nbytes / kRowBytes;
  uint8_t* b = static_cast<uint8_t*>(dev);
  if (nbytes > rows * kRowBytes) zero_kernel<<<1, 256, 0, st>>>(b + rows * kRowBytes, nbytes - rows * kRowBytes);
  if (rows) cfg2_init_kernel<<<grid_for(rows), 256, 0, st>>>(b, rows, seed, thr_proto);
  return (int)cudaGetLastError();
}

GEN_API int gen_cfg2_mutate(void* dev, uint64_t nbytes, uint32_t k, uint64_t seed, uint64_t thr, void* stream) {
  cudaStream_t st = static_cast<cudaStream_t>(stream);
  const uint64_t rows = nbytes / kRowBytes;
  if (rows) cfg2_mutate_kernel<<<grid_for(rows * kNFreq), 256, 0, st>>>(static_cast<uint8_t*>(dev), rows, k, seed, thr);
  return (int)cudaGetLastError();
}
