// arena.h — the handle's diff arena: one contiguous device virtual-address range that
// grows by mapping physical HBM on demand (CUDA virtual memory management, reached via
// cudaGetDriverEntryPoint so libckpt.so does not link libcuda).
//
// Every consolidated diff is carved at the arena top (256-B aligned) and stays at a
// fixed address for the handle's lifetime (ckpt.h: diffs are owned by the handle). Before
// each checkpoint the arena guarantees top + worst-case diff bytes are mapped, so the
// kernels never wait for the host; afterwards the top advances by the ACTUAL size. Only
// one worst-case slack is ever mapped beyond the live diffs — unlike per-checkpoint
// worst-case allocations, which would waste ~B bytes per checkpoint.
#pragma once
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>

#include <cstdint>
#include <vector>

namespace ckpt {

class DiffArena {
 public:
  bool init(int device) {
    if (!load("cuMemAddressReserve", (void**)&reserve_) || !load("cuMemAddressFree", (void**)&free_) ||
        !load("cuMemCreate", (void**)&create_) || !load("cuMemRelease", (void**)&release_) ||
        !load("cuMemMap", (void**)&map_) || !load("cuMemUnmap", (void**)&unmap_) ||
        !load("cuMemSetAccess", (void**)&access_) ||
        !load("cuMemGetAllocationGranularity", (void**)&gran_fn_))
      return false;
    prop_ = {};
    prop_.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop_.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    prop_.location.id = device;
    if (gran_fn_(&gran_, &prop_, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS || gran_ == 0) return false;
    device_ = device;
    return true;
  }

  // Reserve the virtual range once (cheap: no physical memory).
  bool reserve(uint64_t bytes) {
    reserved_ = round_up(bytes, gran_);
    return reserve_(&base_, reserved_, 0, 0, 0) == CUDA_SUCCESS;
  }

  // Make [top, top + need) mapped. Returns false when out of VA or physical memory.
  bool ensure(uint64_t need) {
    const uint64_t want = top_ + need;
    if (want <= mapped_) return true;
    if (want > reserved_) return false;
    uint64_t chunk = round_up(want - mapped_, gran_);
    const uint64_t min_chunk = round_up(1ull << 30, gran_);
    if (chunk < min_chunk) chunk = min_chunk;
    if (mapped_ + chunk > reserved_) chunk = reserved_ - mapped_;
    CUmemGenericAllocationHandle hnd;
    if (create_(&hnd, chunk, &prop_, 0) != CUDA_SUCCESS) return false;
    if (map_(base_ + mapped_, chunk, 0, hnd, 0) != CUDA_SUCCESS) {
      release_(hnd);
      return false;
    }
    CUmemAccessDesc acc = {};
    acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    acc.location.id = device_;
    acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
    if (access_(base_ + mapped_, chunk, &acc, 1) != CUDA_SUCCESS) {
      unmap_(base_ + mapped_, chunk);
      release_(hnd);
      return false;
    }
    maps_.push_back({mapped_, chunk, hnd});
    mapped_ += chunk;
    return true;
  }

  uint8_t* top_ptr() const { return reinterpret_cast<uint8_t*>(base_ + top_); }
  void commit(uint64_t bytes) { top_ += round_up(bytes, 256); }
  uint64_t mapped() const { return mapped_; }
  uint64_t used() const { return top_; }

  void release_all() {
    for (auto& m : maps_) {
      unmap_(base_ + m.off, m.size);
      release_(m.h);
    }
    maps_.clear();
    if (base_) free_(base_, reserved_);
    base_ = 0;
    mapped_ = top_ = reserved_ = 0;
  }

 private:
  static uint64_t round_up(uint64_t x, uint64_t a) { return (x + a - 1) / a * a; }
  static bool load(const char* sym, void** fn) {
    cudaDriverEntryPointQueryResult q;
    return cudaGetDriverEntryPoint(sym, fn, cudaEnableDefault, &q) == cudaSuccess &&
           q == cudaDriverEntryPointSuccess && *fn;
  }
  struct Map {
    uint64_t off, size;
    CUmemGenericAllocationHandle h;
  };
  PFN_cuMemAddressReserve_v10020 reserve_ = nullptr;
  PFN_cuMemAddressFree_v10020 free_ = nullptr;
  PFN_cuMemCreate_v10020 create_ = nullptr;
  PFN_cuMemRelease_v10020 release_ = nullptr;
  PFN_cuMemMap_v10020 map_ = nullptr;
  PFN_cuMemUnmap_v10020 unmap_ = nullptr;
  PFN_cuMemSetAccess_v10020 access_ = nullptr;
  PFN_cuMemGetAllocationGranularity_v10020 gran_fn_ = nullptr;
  CUmemAllocationProp prop_ = {};
  size_t gran_ = 0;
  int device_ = 0;
  CUdeviceptr base_ = 0;
  uint64_t reserved_ = 0, mapped_ = 0, top_ = 0;
  std::vector<Map> maps_;
};

}  // namespace ckpt
