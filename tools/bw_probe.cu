// bw_probe.cu — HBM read-only vs copy bandwidth on this B200 (diagnostic, not product code).
// Answers: is K1 (a read-dominated stream: 1 GiB input + 128 MiB digests, ~1 MiB writes)
// bounded by the copy figure of MEASURED_PEAKS.json or by a higher read-only ceiling?
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gpurun_out/bw_probe tools/bw_probe.cu
#include <cuda.h>
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

// persistent TMA tensor reader (like K1's data path): box 128 x 256 rows per stage,
// optional extra 1-D bulk side load of SIDE bytes per stage, optional evict_first hint
template <int NST, int SIDE, bool HINT>
__global__ void read_tensor(const __grid_constant__ CUtensorMap map, const uint8_t* __restrict__ side, size_t ntile,
                            unsigned long long* out) {
  extern __shared__ __align__(1024) uint8_t smraw[];
  uint8_t* sm = smraw + ((1024u - (su32(smraw) & 1023u)) & 1023u);
  __shared__ __align__(8) uint64_t bar[NST];
  if (threadIdx.x == 0) {
    for (int s = 0; s < NST; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  uint64_t pol;
  asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  const uint32_t SB = 32768 + SIDE;
  auto issue = [&](size_t tile, int s) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[s])), "r"(SB));
    if (HINT)
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes.L2::cache_hint [%0], [%1, {%2, %3}], [%4], %5;" ::"r"(
                       su32(sm + (size_t)s * SB)), "l"(&map), "r"(0), "r"((int)(tile * 256)), "r"(su32(&bar[s])), "l"(pol) : "memory");
    else
      asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(
                       su32(sm + (size_t)s * SB)), "l"(&map), "r"(0), "r"((int)(tile * 256)), "r"(su32(&bar[s])) : "memory");
    if (SIDE)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       su32(sm + (size_t)s * SB + 32768)), "l"(side + tile * SIDE), "r"(SIDE), "r"(su32(&bar[s])) : "memory");
  };
  for (int s = 0; s < NST && blockIdx.x + (size_t)s * gridDim.x < ntile; ++s) issue(blockIdx.x + (size_t)s * gridDim.x, s);
  uint32_t acc = 0;
  size_t it = 0;
  for (size_t tile = blockIdx.x; tile < ntile; tile += gridDim.x, ++it) {
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
  {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q);
    auto encode = reinterpret_cast<CUresult (*)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                                const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                                CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill)>(fn);
    std::vector<CUtensorMap> maps(NB), maps_ns(NB);
    for (int i = 0; i < NB; ++i) {
      cuuint64_t dims[2] = {128, B / 128};
      cuuint64_t strides[1] = {128};
      cuuint32_t box[2] = {128, 256};
      cuuint32_t es[2] = {1, 1};
      encode(&maps[i], CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, bufs[i], dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      encode(&maps_ns[i], CU_TENSOR_MAP_DATA_TYPE_UINT8, 2, bufs[i], dims, strides, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
             CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_NONE, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    }
    const size_t ntile = B / 32768;
    uint8_t* side; cudaMalloc(&side, ntile * 4096); cudaMemset(side, 2, ntile * 4096);
    const int sm3 = 3 * 32768 + 1024, sm3s = 3 * (32768 + 4096) + 1024;
    cudaFuncSetAttribute(read_tensor<3, 0, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm3);
    cudaFuncSetAttribute(read_tensor<3, 0, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm3);
    cudaFuncSetAttribute(read_tensor<3, 4096, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm3s);
    cudaFuncSetAttribute(read_tensor<3, 4096, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, sm3s);
    timeit("tensor 2D swz128 3x32KB x2 CTA", (double)B, [&](int i) { read_tensor<3, 0, false><<<2 * sms, 32, sm3>>>(maps[i], side, ntile, out); });
    timeit("tensor 2D noswz 3x32KB x2 CTA", (double)B, [&](int i) { read_tensor<3, 0, false><<<2 * sms, 32, sm3>>>(maps_ns[i], side, ntile, out); });
    timeit("tensor swz + evict_first", (double)B, [&](int i) { read_tensor<3, 0, true><<<2 * sms, 32, sm3>>>(maps[i], side, ntile, out); });
    timeit("tensor swz + 4KB side (K1 bytes)", (double)B * 1.125, [&](int i) { read_tensor<3, 4096, false><<<2 * sms, 32, sm3s>>>(maps[i], side, ntile, out); });
    timeit("tensor swz + side + evict_first", (double)B * 1.125, [&](int i) { read_tensor<3, 4096, true><<<2 * sms, 32, sm3s>>>(maps[i], side, ntile, out); });
  }
  timeit("copy (read+write bytes)", 2.0 * B / 2, [&](int i) {
    copy_k<<<sms * 8, 256>>>((const uint4*)bufs[i], (uint4*)bufs[(i + 1) % NB], B / 32);
  });
  cudaError_t e = cudaDeviceSynchronize();
  printf("status: %s\n", cudaGetErrorString(e));
  return 0;
}
