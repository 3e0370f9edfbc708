// Host-side cost of the allocations a growing lineage makes (record-table growth, diff arena):
// cudaMalloc vs stream-ordered cudaMallocAsync (default pool / a private pool with a high
// release threshold), and VMM cuMemCreate + cuMemMap of 1 GiB.   nvcc -o /tmp/ap tools/alloc_probe.cu -lcuda
#include <cuda.h>
#include <cuda_runtime.h>
#include <chrono>
#include <cstdio>
using clk = std::chrono::steady_clock;
static double ms(clk::time_point a) { return std::chrono::duration<double, std::milli>(clk::now() - a).count(); }
int main() {
  cudaFree(0);
  cudaStream_t st;
  cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
  size_t sizes[] = {256ull << 20, 1ull << 30, 2ull << 30, 4ull << 30};
  for (size_t sz : sizes) {
    void* p;
    auto t = clk::now(); cudaMalloc(&p, sz); double a = ms(t);
    t = clk::now(); cudaMemsetAsync(p, 0xFF, sz, st); cudaStreamSynchronize(st); double b = ms(t);
    t = clk::now(); cudaFree(p); double c = ms(t);
    t = clk::now(); cudaMallocAsync(&p, sz, st); double d = ms(t);
    t = clk::now(); cudaMemsetAsync(p, 0xFF, sz, st); cudaStreamSynchronize(st); double e = ms(t);
    t = clk::now(); cudaFreeAsync(p, st); cudaStreamSynchronize(st); double f = ms(t);
    t = clk::now(); cudaMallocAsync(&p, sz, st); double g = ms(t);
    cudaFreeAsync(p, st); cudaStreamSynchronize(st);
    printf("%5zu MiB: cudaMalloc %.3f memset %.3f free %.3f | mallocAsync %.3f memset %.3f freeAsync+sync %.3f | again %.3f ms\n",
           sz >> 20, a, b, c, d, e, f, g);
  }
  // private pool, release threshold = max
  cudaMemPool_t pool;
  cudaMemPoolProps pp = {};
  pp.allocType = cudaMemAllocationTypePinned;
  pp.location.type = cudaMemLocationTypeDevice;
  pp.location.id = 0;
  cudaMemPoolCreate(&pool, &pp);
  unsigned long long thr = ~0ull;
  cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
  for (size_t sz : sizes) {
    void* p;
    auto t = clk::now(); cudaMallocFromPoolAsync(&p, sz, pool, st); double a = ms(t);
    cudaStreamSynchronize(st);
    t = clk::now(); cudaFreeAsync(p, st); cudaStreamSynchronize(st); double b = ms(t);
    printf("%5zu MiB: private pool malloc %.3f free+sync %.3f ms\n", sz >> 20, a, b);
  }
  CUmemAllocationProp prop = {};
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = 0;
  size_t gran = 0;
  cuMemGetAllocationGranularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
  CUdeviceptr va;
  cuMemAddressReserve(&va, 64ull << 30, 0, 0, 0);
  for (int i = 0; i < 4; ++i) {
    CUmemGenericAllocationHandle h;
    auto t = clk::now();
    cuMemCreate(&h, 1ull << 30, &prop, 0); double a = ms(t);
    t = clk::now(); cuMemMap(va + ((size_t)i << 30), 1ull << 30, 0, h, 0); double b = ms(t);
    CUmemAccessDesc acc = {};
    acc.location = prop.location;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    t = clk::now(); cuMemSetAccess(va + ((size_t)i << 30), 1ull << 30, &acc, 1); double c = ms(t);
    printf("VMM 1 GiB #%d: create %.3f map %.3f access %.3f ms (gran %zu)\n", i, a, b, c, gran);
  }
  return 0;
}
