// rand_probe.cu — random 32-B sector throughput on this B200 (diagnostic, not product code).
// Answers: what is the ceiling for the record-table traffic of config 4 (K1b and phase 3 each
// issue one random 32-B slot access per candidate leaf / potential SHIFT node)? Reports
// sectors/s for plain 32-B reads (ld.global.cg.v2.u64 x2, one sector), by working-set size
// and by independent reads in flight per thread, and for 128-bit CAS that fail (key present).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gpurun_out/rand_probe tools/rand_probe.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>
#include <vector>
#include <algorithm>

__device__ __forceinline__ uint64_t mix(uint64_t x) {
  x ^= x >> 33; x *= 0xff51afd7ed558ccdull; x ^= x >> 33; x *= 0xc4ceb9fe1a85ec53ull; x ^= x >> 33;
  return x;
}

// each thread: `per` rounds of ILP independent random slot reads (32 B = one sector)
template <int ILP>
__global__ void rand_read(const ulonglong4* __restrict__ tab, uint64_t cap, uint32_t per, unsigned long long* out) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (uint32_t r = 0; r < per; ++r) {
    ulonglong2 v[ILP];
#pragma unroll
    for (int u = 0; u < ILP; ++u) {
      const uint64_t s = __umul64hi(mix(tid * 1315423911ull + (uint64_t)r * ILP + u), cap);
      v[u] = __ldcg(reinterpret_cast<const ulonglong2*>(tab + s));
    }
#pragma unroll
    for (int u = 0; u < ILP; ++u) acc += v[u].x ^ v[u].y;
  }
  if (acc == 0x123456789ull) atomicAdd(out, 1ull);
}

// K1b / phase-3 style slot read: key (16 B) and value (8 B) as two loads of one sector (MODE 0),
// or the whole 32-B slot as one 256-bit load (MODE 1, LDG.E.ENL2.256 on sm_100)
template <int MODE, int ILP>
__global__ void rand_slot(const ulonglong4* __restrict__ tab, uint64_t cap, uint32_t per, unsigned long long* out) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (uint32_t r = 0; r < per; ++r) {
    unsigned long long a[ILP], b[ILP], c[ILP];
#pragma unroll
    for (int u = 0; u < ILP; ++u) {
      const uint64_t s = __umul64hi(mix(tid * 1315423911ull + (uint64_t)r * ILP + u), cap);
      const ulonglong4* p = tab + s;
      if (MODE == 0) {
        asm volatile("ld.relaxed.gpu.global.v2.u64 {%0, %1}, [%2];" : "=l"(a[u]), "=l"(b[u]) : "l"(p) : "memory");
        asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(c[u]) : "l"(&p->z) : "memory");
      } else {
        unsigned long long d;
        asm volatile("ld.relaxed.gpu.global.v4.u64 {%0, %1, %2, %3}, [%4];"
                     : "=l"(a[u]), "=l"(b[u]), "=l"(c[u]), "=l"(d) : "l"(p) : "memory");
      }
    }
#pragma unroll
    for (int u = 0; u < ILP; ++u) acc += a[u] ^ b[u] ^ c[u];
  }
  if (acc == 0x123456789ull) atomicAdd(out, 1ull);
}

// dependent chain: the next address depends on the value read (pure latency per thread)
__global__ void rand_chase(const ulonglong4* __restrict__ tab, uint64_t cap, uint32_t per, unsigned long long* out) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  uint64_t x = tid;
  for (uint32_t r = 0; r < per; ++r) {
    const uint64_t s = __umul64hi(mix(x + r), cap);
    const ulonglong2 v = __ldcg(reinterpret_cast<const ulonglong2*>(tab + s));
    x += v.x & 1;
  }
  if (x == 0x123456789ull) atomicAdd(out, 1ull);
}

// 128-bit CAS that fails (expects EMPTY, slot holds a key): K1b's CAS-first insert of a present key
template <int ILP>
__global__ void rand_cas(ulonglong4* tab, uint64_t cap, uint32_t per, unsigned long long* out) {
  const uint64_t tid = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  unsigned long long acc = 0;
  for (uint32_t r = 0; r < per; ++r) {
    unsigned long long lo[ILP], hi[ILP];
#pragma unroll
    for (int u = 0; u < ILP; ++u) {
      const uint64_t s = __umul64hi(mix(tid * 1315423911ull + (uint64_t)r * ILP + u), cap);
      ulonglong4* p = tab + s;
      asm volatile(
          "{\n\t.reg .b128 d, c, v;\n\t"
          "mov.b128 c, {%2, %3};\n\t"
          "mov.b128 v, {%4, %5};\n\t"
          "atom.relaxed.gpu.global.cas.b128 d, [%6], c, v;\n\t"
          "mov.b128 {%0, %1}, d;\n\t}"
          : "=l"(lo[u]), "=l"(hi[u])
          : "l"(~0ull), "l"(~0ull), "l"(1ull), "l"(2ull), "l"(p)
          : "memory");
    }
#pragma unroll
    for (int u = 0; u < ILP; ++u) acc += lo[u] ^ hi[u];
  }
  if (acc == 0x123456789ull) atomicAdd(out, 1ull);
}

int main() {
  int sms = 0;
  cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  const uint64_t max_bytes = 4ull << 30;
  ulonglong4* tab;
  unsigned long long* out;
  if (cudaMalloc(&tab, max_bytes) != cudaSuccess) { printf("alloc failed\n"); return 1; }
  cudaMalloc(&out, 8);
  cudaMemset(tab, 0x5a, max_bytes);   // every slot "present" (no EMPTY): CAS always fails
  cudaEvent_t a, b;
  cudaEventCreate(&a);
  cudaEventCreate(&b);
  const uint64_t sizes[] = {32ull << 20, 96ull << 20, 256ull << 20, 1ull << 30, 2ull << 30, 3ull << 30, 4ull << 30};
  auto run = [&](const char* name, auto launch, uint64_t ops) {
    std::vector<float> t;
    for (int rep = 0; rep < 7; ++rep) {
      cudaEventRecord(a);
      launch();
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      t.push_back(ms);
    }
    std::sort(t.begin(), t.end());
    const double ms = t[t.size() / 2];
    printf("%-44s %8.3f ms  %7.2f G sectors/s  %7.1f GB/s of 32-B sectors\n", name, ms, ops / ms / 1e6,
           ops * 32.0 / ms / 1e6);
  };
  for (uint64_t ws : sizes) {
    const uint64_t cap = ws / 32;
    printf("# working set %llu MiB\n", (unsigned long long)(ws >> 20));
    for (int bps : {4, 8, 16}) {
      const uint32_t per = 64;
      const unsigned grid = sms * bps, thr = 256;
      char nm[96];
      snprintf(nm, sizeof nm, "read ILP1 %2d blk/SM", bps);
      run(nm, [&] { rand_read<1><<<grid, thr>>>(tab, cap, per, out); }, (uint64_t)grid * thr * per);
      snprintf(nm, sizeof nm, "read ILP4 %2d blk/SM", bps);
      run(nm, [&] { rand_read<4><<<grid, thr>>>(tab, cap, per / 4, out); }, (uint64_t)grid * thr * per);
    }
    {
      const unsigned grid = sms * 8, thr = 256;
      run("read ILP8  8 blk/SM", [&] { rand_read<8><<<grid, thr>>>(tab, cap, 8, out); }, (uint64_t)grid * thr * 64);
      run("slot 2 loads ILP1 8 blk/SM", [&] { rand_slot<0, 1><<<grid, thr>>>(tab, cap, 64, out); }, (uint64_t)grid * thr * 64);
      run("slot 2 loads ILP4 8 blk/SM", [&] { rand_slot<0, 4><<<grid, thr>>>(tab, cap, 16, out); }, (uint64_t)grid * thr * 64);
      run("slot 256-bit ILP1 8 blk/SM", [&] { rand_slot<1, 1><<<grid, thr>>>(tab, cap, 64, out); }, (uint64_t)grid * thr * 64);
      run("slot 256-bit ILP4 8 blk/SM", [&] { rand_slot<1, 4><<<grid, thr>>>(tab, cap, 16, out); }, (uint64_t)grid * thr * 64);
      run("chase (latency)  8 blk/SM", [&] { rand_chase<<<grid, thr>>>(tab, cap, 16, out); }, (uint64_t)grid * thr * 16);
      run("cas128 fail ILP1 8 blk/SM", [&] { rand_cas<1><<<grid, thr>>>(tab, cap, 32, out); }, (uint64_t)grid * thr * 32);
      run("cas128 fail ILP4 8 blk/SM", [&] { rand_cas<4><<<grid, thr>>>(tab, cap, 8, out); }, (uint64_t)grid * thr * 32);
    }
  }
  // latency of one dependent round trip at low load (1 warp per SM)
  {
    const uint64_t cap = (2ull << 30) / 32;
    cudaEventRecord(a);
    rand_chase<<<sms, 32>>>(tab, cap, 256, out);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    printf("idle dependent-read latency (2 GiB set): %.0f ns\n", ms * 1e6 / 256);
  }
  printf("status: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  return 0;
}
