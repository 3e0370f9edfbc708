// bw_probe.cu — HBM read-only vs copy bandwidth on this B200 (diagnostic, not product code).
// Answers: is K1 (a read-dominated stream: 1 GiB input + 128 MiB digests, ~1 MiB writes)
// bounded by the copy figure of MEASURED_PEAKS.json or by a higher read-only ceiling?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gpurun_out/bw_probe tools/bw_probe.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <vector>
#include <algorithm>

__global__ void read_ldg(const uint4* __restrict__ p, size_t n16, unsigned long long* out) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 7 * stride < n16; i += 8 * stride) {
    uint4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldcs(p + i + u * stride);
#pragma unroll
    for (int u = 0; u < 8; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
  }
  for (; i < n16; i += stride) { uint4 v = __ldcs(p + i); acc ^= v.x ^ v.y ^ v.z ^ v.w; }
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// persistent bulk-copy (TMA 1-D) reader: NST stages of SB bytes per CTA, no compute
template <int NST, int SB>
__global__ void read_bulk(const uint8_t* __restrict__ p, size_t nbytes, unsigned long long* out) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[NST];
  const size_t ntile = nbytes / SB;
  if (threadIdx.x == 0) {
    for (int s = 0; s < NST; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  size_t t = blockIdx.x, issued = 0;
  auto issue = [&](size_t tile, int s) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(SB));
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     su32(sm + (size_t)s * SB)),
                 "l"(p + tile * SB), "r"(SB), "r"(su32(&bar[s])) : "memory");
  };
  size_t it = 0;
  for (int s = 0; s < NST && t + (size_t)s * gridDim.x < ntile; ++s) { issue(t + (size_t)s * gridDim.x, s); ++issued; }
  uint32_t acc = 0;
  for (size_t tile = t; tile < ntile; tile += gridDim.x, ++it) {
    const int s = (int)(it % NST);
    const uint32_t ph = (uint32_t)((it / NST) & 1);
    asm volatile("{\n\t.reg .pred q;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 q, [%0], %1;\n\t@!q bra W_%=;\n\t}" ::"r"(
                     su32(&bar[s])), "r"(ph) : "memory");
    acc ^= sm[(size_t)s * SB];
    const size_t nx = tile + (size_t)NST * gridDim.x;
    if (nx < ntile) issue(nx, s);
  }
  if (acc == 0x5a) atomicAdd(out, 1ull);
}

__global__ void copy_k(const uint4* __restrict__ a, uint4* __restrict__ b, size_t n16) {
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += stride) b[i] = __ldcs(a + i);
}

int main() {
  const size_t B = 1ull << 30;
  const int NB = 4;
  std::vector<uint8_t*> bufs(NB);
  for (auto& b : bufs) { cudaMalloc(&b, B); cudaMemset(b, 1, B); }
  unsigned long long* out; cudaMalloc(&out, 8);
  cudaEvent_t e0, e1; cudaEventCreate(&e0); cudaEventCreate(&e1);
  int sms = 148; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  auto timeit = [&](const char* name, double bytes, auto fn) {
    std::vector<float> ts;
    for (int r = 0; r < 24; ++r) {
      cudaEventRecord(e0); fn(r % NB); cudaEventRecord(e1); cudaEventSynchronize(e1);
      float ms; cudaEventElapsedTime(&ms, e0, e1); if (r >= 4) ts.push_back(ms);
    }
    std::sort(ts.begin(), ts.end());
    printf("%-34s best %7.1f GB/s  median %7.1f GB/s\n", name, bytes / ts[0] / 1e6, bytes / ts[ts.size() / 2] / 1e6);
  };
  for (int bps : {4, 8, 16}) {
    char nm[64]; snprintf(nm, 64, "read LDG.128 x8, %d blk/SM x256", bps);
    timeit(nm, (double)B, [&](int i) { read_ldg<<<sms * bps, 256>>>((const uint4*)bufs[i], B / 16, out); });
  }
  {
    const int smem = 6 * 32768;
    cudaFuncSetAttribute(read_bulk<6, 32768>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem);
    timeit("read bulk 6x32KB, 1 CTA/SM", (double)B, [&](int i) { read_bulk<6, 32768><<<sms, 32, smem>>>(bufs[i], B, out); });
    const int smem2 = 3 * 32768;
    cudaFuncSetAttribute(read_bulk<3, 32768>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem2);
    timeit("read bulk 3x32KB, 2 CTA/SM", (double)B, [&](int i) { read_bulk<3, 32768><<<2 * sms, 32, smem2>>>(bufs[i], B, out); });
    const int smem3 = 12 * 16384;
    cudaFuncSetAttribute(read_bulk<12, 16384>, cudaFuncAttributeMaxDynamicSharedMemorySize, smem3);
    timeit("read bulk 12x16KB, 1 CTA/SM", (double)B, [&](int i) { read_bulk<12, 16384><<<sms, 32, smem3>>>(bufs[i], B, out); });
  }
  timeit("copy (read+write bytes)", 2.0 * B / 2, [&](int i) {
    copy_k<<<sms * 8, 256>>>((const uint4*)bufs[i], (uint4*)bufs[(i + 1) % NB], B / 32);
  });
  cudaError_t e = cudaDeviceSynchronize();
  printf("status: %s\n", cudaGetErrorString(e));
  return 0;
}
