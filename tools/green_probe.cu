// green_probe.cu — can an HBM stream and a latency-bound kernel share the GPU by SM partition?
// (diagnostic, not product code). Green contexts split the SMs: a persistent streaming read
// kernel (K1's stand-in) on 148 - m SMs, a dependent-load chase (the tree phases' stand-in)
// on m SMs. Reports each alone and both at once: the stream's GB/s and the chase's time.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gpurun_out/green_probe tools/green_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

#define CKD(x) do { CUresult r_ = (x); if (r_ != CUDA_SUCCESS) { const char* s; cuGetErrorString(r_, &s); \
  printf("%s failed: %s\n", #x, s); return 1; } } while (0)
#define CKR(x) do { cudaError_t r_ = (x); if (r_ != cudaSuccess) { printf("%s failed: %s\n", #x, cudaGetErrorString(r_)); return 1; } } while (0)

__global__ void stream_read(const uint4* __restrict__ p, size_t n16, int reps, unsigned long long* out) {
  uint32_t acc = 0;
  const size_t stride = (size_t)gridDim.x * blockDim.x;
  for (int r = 0; r < reps; ++r) {
    size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
    for (; i + 7 * stride < n16; i += 8 * stride) {
      uint4 v[8];
#pragma unroll
      for (int u = 0; u < 8; ++u) v[u] = __ldcs(p + i + u * stride);
#pragma unroll
      for (int u = 0; u < 8; ++u) acc ^= v[u].x ^ v[u].y ^ v[u].z ^ v[u].w;
    }
  }
  if (acc == 0x12345678u) atomicAdd(out, 1ull);
}

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}
// per thread: `per` dependent random 16-B loads over a 1-GiB table
__global__ void chase(const uint4* __restrict__ tab, uint64_t n16, int per, unsigned long long* out) {
  uint64_t x = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (int r = 0; r < per; ++r) {
    const uint4 v = __ldcg(tab + __umul64hi(mix(x + r), n16));
    x += v.x & 1;
  }
  if (x == 0x123456789ull) atomicAdd(out, 1ull);
}

int main(int argc, char** argv) {
  CKR(cudaSetDevice(0));
  CKR(cudaFree(0));
  CUdevice dev;
  CKD(cuDeviceGet(&dev, 0));
  const size_t B = 1ull << 30;
  uint4 *buf, *tab;
  unsigned long long* out;
  CKR(cudaMalloc(&buf, B));
  CKR(cudaMalloc(&tab, B));
  CKR(cudaMalloc(&out, 8));
  CKR(cudaMemset(buf, 1, B));
  CKR(cudaMemset(tab, 2, B));
  CUdevResource all;
  CKD(cuDeviceGetDevResource(dev, &all, CU_DEV_RESOURCE_TYPE_SM));
  printf("SMs: %u\n", all.sm.smCount);
  for (int m : {8, 16, 24, 32}) {
    CUdevResource grp, rest;
    unsigned int ng = 1;
    CKD(cuDevSmResourceSplitByCount(&grp, &ng, &all, &rest, 0, (unsigned)m));
    CUdevResourceDesc dA, dB;
    CKD(cuDevResourceGenerateDesc(&dA, &rest, 1));
    CKD(cuDevResourceGenerateDesc(&dB, &grp, 1));
    CUgreenCtx gA, gB;
    CKD(cuGreenCtxCreate(&gA, dA, dev, CU_GREEN_CTX_DEFAULT_STREAM));
    CKD(cuGreenCtxCreate(&gB, dB, dev, CU_GREEN_CTX_DEFAULT_STREAM));
    CUstream sA, sB;
    CKD(cuGreenCtxStreamCreate(&sA, gA, CU_STREAM_NON_BLOCKING, 0));
    CKD(cuGreenCtxStreamCreate(&sB, gB, CU_STREAM_NON_BLOCKING, 0));
    const int smA = all.sm.smCount - grp.sm.smCount, smB = grp.sm.smCount;
    cudaEvent_t a0, a1, b0, b1;
    CKR(cudaEventCreate(&a0)); CKR(cudaEventCreate(&a1)); CKR(cudaEventCreate(&b0)); CKR(cudaEventCreate(&b1));
    const int reps = 4, per = 64;
    auto runA = [&] { stream_read<<<smA * 4, 512, 0, (cudaStream_t)sA>>>(buf, B / 16, reps, out); };
    auto runB = [&] { chase<<<smB * 2, 256, 0, (cudaStream_t)sB>>>(tab, B / 16, per, out); };
    for (int w = 0; w < 2; ++w) { runA(); runB(); }
    CKR(cudaDeviceSynchronize());
    float ta = 0, tb = 0, tac = 0, tbc = 0;
    cudaEventRecord(a0, (cudaStream_t)sA); runA(); cudaEventRecord(a1, (cudaStream_t)sA);
    CKR(cudaDeviceSynchronize()); cudaEventElapsedTime(&ta, a0, a1);
    cudaEventRecord(b0, (cudaStream_t)sB); runB(); cudaEventRecord(b1, (cudaStream_t)sB);
    CKR(cudaDeviceSynchronize()); cudaEventElapsedTime(&tb, b0, b1);
    // both at once: B starts after A has ramped (A is several ms long)
    cudaEventRecord(a0, (cudaStream_t)sA); runA(); cudaEventRecord(a1, (cudaStream_t)sA);
    cudaEventRecord(b0, (cudaStream_t)sB); runB(); cudaEventRecord(b1, (cudaStream_t)sB);
    CKR(cudaDeviceSynchronize()); cudaEventElapsedTime(&tac, a0, a1); cudaEventElapsedTime(&tbc, b0, b1);
    printf("m=%2d: stream on %3d SMs alone %.0f GB/s, with chase %.0f GB/s | chase on %2d SMs alone %.1f us, "
           "under stream %.1f us (x%.2f)\n",
           m, smA, reps * B / (ta * 1e6), reps * B / (tac * 1e6), smB, tb * 1e3, tbc * 1e3, tbc / tb);
    // reference: stream on all SMs (primary context)
    if (m == 8) {
      cudaEventRecord(a0); stream_read<<<all.sm.smCount * 4, 512>>>(buf, B / 16, reps, out); cudaEventRecord(a1);
      CKR(cudaDeviceSynchronize()); cudaEventElapsedTime(&ta, a0, a1);
      printf("      stream on all %u SMs: %.0f GB/s\n", all.sm.smCount, reps * B / (ta * 1e6));
    }
  }
  printf("status: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
