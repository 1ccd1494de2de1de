// arena.cpp — VMM-backed device arena: the "freeing GPU capacity" half of preemption (§4.2)
// and the "reserve memory" half of swap-in (§3.4), with virtual addresses that survive
// both so a restore can scatter to the recorded addresses (SURVEY.md §7 hard part 6, NEXT-1).
//
// The VA range is reserved once (cuMemAddressReserve). Physical memory is one cuMemCreate
// allocation per slab (1 GiB, the last one smaller) mapped into the range with read/write access
// for the owning device. swap_arena_release unmaps and releases every slab (the HBM returns to the
// device's free pool; the VA stays reserved); swap_arena_reacquire creates and maps fresh slabs at
// the same addresses. Driver entry points are resolved at run time through cudart
// (cudaGetDriverEntryPoint), so libswap.so does not link libcuda and still loads on CPU-only hosts.
#include <cuda.h>
#include <cuda_runtime.h>

#include <cstring>
#include <unistd.h>
#include <string>
#include <vector>

#include "../../include/swap.h"
#include "arena.h"

namespace {

struct Drv {
  decltype(&cuMemGetAllocationGranularity) granularity = nullptr;
  decltype(&cuMemAddressReserve) reserve = nullptr;
  decltype(&cuMemAddressFree) addr_free = nullptr;
  decltype(&cuMemCreate) create = nullptr;
  decltype(&cuMemRelease) release = nullptr;
  decltype(&cuMemMap) map = nullptr;
  decltype(&cuMemUnmap) unmap = nullptr;
  decltype(&cuMemSetAccess) set_access = nullptr;
  decltype(&cuMemExportToShareableHandle) export_h = nullptr;    // optional (peer import of arenas)
  decltype(&cuMemImportFromShareableHandle) import_h = nullptr;  // optional
  bool ok = false;
};

template <class F>
bool resolve(const char* name, F* fn) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess || q != cudaDriverEntryPointSuccess ||
      !p)
    return false;
  *fn = reinterpret_cast<F>(p);
  return true;
}

const Drv& drv() {
  static Drv d = [] {
    Drv x;
    x.ok = resolve("cuMemGetAllocationGranularity", &x.granularity) && resolve("cuMemAddressReserve", &x.reserve) &&
           resolve("cuMemAddressFree", &x.addr_free) && resolve("cuMemCreate", &x.create) &&
           resolve("cuMemRelease", &x.release) && resolve("cuMemMap", &x.map) && resolve("cuMemUnmap", &x.unmap) &&
           resolve("cuMemSetAccess", &x.set_access);
    resolve("cuMemExportToShareableHandle", &x.export_h);
    resolve("cuMemImportFromShareableHandle", &x.import_h);
    return x;
  }();
  return d;
}

constexpr uint64_t kSlab = 1ull << 30;

}  // namespace

struct swap_arena {
  int device = 0;
  CUdeviceptr base = 0;
  uint64_t bytes = 0;  // rounded to the allocation granularity
  uint64_t gran = 0;
  std::vector<CUmemGenericAllocationHandle> slabs;  // one per 1-GiB slab; 0 = not mapped
  uint64_t n_mapped = 0;
  bool resident = false;  // every slab mapped
  std::string err;
};

namespace {

uint64_t n_slabs(const swap_arena* a) { return (a->bytes + kSlab - 1) / kSlab; }
uint64_t slab_size(const swap_arena* a, uint64_t i) {
  const uint64_t off = i * kSlab;
  return a->bytes - off < kSlab ? a->bytes - off : kSlab;
}

swap_status map_slab(swap_arena* a, uint64_t i) {
  if (a->slabs[i]) return SWAP_OK;
  const Drv& D = drv();
  CUmemAllocationProp prop;
  std::memset(&prop, 0, sizeof(prop));
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = a->device;
  // slabs can be exported as POSIX file descriptors (swap_arena_export: data-parallel replicas map each
  // other's arenas for the fused NVLink pull)
  prop.requestedHandleTypes = CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR;
  CUmemAccessDesc acc;
  std::memset(&acc, 0, sizeof(acc));
  acc.location = prop.location;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  const uint64_t off = i * kSlab, sz = slab_size(a, i);
  CUmemGenericAllocationHandle h;
  CUresult r = D.create(&h, sz, &prop, 0);
  if (r != CUDA_SUCCESS) {
    a->err = "cuMemCreate failed (" + std::to_string((int)r) + ") at offset " + std::to_string(off);
    return r == CUDA_ERROR_OUT_OF_MEMORY ? SWAP_ENOMEM : SWAP_ECUDA;
  }
  if ((r = D.map(a->base + off, sz, 0, h, 0)) != CUDA_SUCCESS) {
    D.release(h);
    a->err = "cuMemMap failed (" + std::to_string((int)r) + ")";
    return SWAP_ECUDA;
  }
  if ((r = D.set_access(a->base + off, sz, &acc, 1)) != CUDA_SUCCESS) {
    D.unmap(a->base + off, sz);
    D.release(h);
    a->err = "cuMemSetAccess failed (" + std::to_string((int)r) + ")";
    return SWAP_ECUDA;
  }
  a->slabs[i] = h;
  a->resident = ++a->n_mapped == n_slabs(a);
  return SWAP_OK;
}

swap_status map_all(swap_arena* a) {
  for (uint64_t i = 0; i < n_slabs(a); ++i) {
    swap_status st = map_slab(a, i);
    if (st != SWAP_OK) return st;
  }
  return SWAP_OK;
}

swap_status unmap_all(swap_arena* a) {
  const Drv& D = drv();
  swap_status st = SWAP_OK;
  for (uint64_t i = 0; i < a->slabs.size(); ++i) {
    if (!a->slabs[i]) continue;
    if (D.unmap(a->base + i * kSlab, slab_size(a, i)) != CUDA_SUCCESS) st = SWAP_ECUDA;
    if (D.release(a->slabs[i]) != CUDA_SUCCESS) st = SWAP_ECUDA;
    a->slabs[i] = 0;
  }
  a->n_mapped = 0;
  a->resident = false;
  if (st != SWAP_OK) a->err = "cuMemUnmap/cuMemRelease failed";
  return st;
}

struct CtxGuard {  // run driver calls with the device's primary context current
  int prev = -1;
  explicit CtxGuard(int dev) {
    if (cudaGetDevice(&prev) != cudaSuccess) prev = -1;
    cudaSetDevice(dev);
    cudaFree(nullptr);  // make the primary context current on this thread
  }
  ~CtxGuard() {
    if (prev >= 0) cudaSetDevice(prev);
  }
};

}  // namespace

extern "C" {

swap_status swap_arena_create(int device, uint64_t bytes, swap_arena_t** out) {
  if (!out || bytes == 0 || device < 0) return SWAP_EINVAL;
  *out = nullptr;
  int ndev = 0;
  if (cudaGetDeviceCount(&ndev) != cudaSuccess || device >= ndev) return SWAP_ECUDA;
  CtxGuard g(device);
  const Drv& D = drv();
  if (!D.ok) return SWAP_EUNSUPPORTED;
  auto* a = new (std::nothrow) swap_arena();
  if (!a) return SWAP_ENOMEM;
  a->device = device;
  CUmemAllocationProp prop;
  std::memset(&prop, 0, sizeof(prop));
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = device;
  size_t gran = 0;
  if (D.granularity(&gran, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) != CUDA_SUCCESS || gran == 0) {
    delete a;
    return SWAP_ECUDA;
  }
  a->gran = gran;
  a->bytes = (bytes + gran - 1) / gran * gran;
  a->slabs.assign(n_slabs(a), 0);
  if (D.reserve(&a->base, a->bytes, kSlab, 0, 0) != CUDA_SUCCESS) {
    delete a;
    return SWAP_ENOMEM;
  }
  swap_status st = map_all(a);
  if (st != SWAP_OK) {
    unmap_all(a);
    D.addr_free(a->base, a->bytes);
    delete a;
    return st;
  }
  *out = a;
  return SWAP_OK;
}

swap_status swap_arena_info(const swap_arena_t* a, uint64_t* dev_addr, uint64_t* bytes, int* resident) {
  if (!a) return SWAP_EINVAL;
  if (dev_addr) *dev_addr = (uint64_t)a->base;
  if (bytes) *bytes = a->bytes;
  if (resident) *resident = a->resident ? 1 : 0;
  return SWAP_OK;
}

swap_status swap_arena_release(swap_arena_t* a) {
  if (!a) return SWAP_EINVAL;
  if (a->n_mapped == 0) return SWAP_ESTATE;
  CtxGuard g(a->device);
  if (cudaDeviceSynchronize() != cudaSuccess) return SWAP_ECUDA;  // no kernel may still touch it
  return unmap_all(a);
}

swap_status swap_arena_reacquire(swap_arena_t* a) {
  if (!a) return SWAP_EINVAL;
  if (a->resident) return SWAP_ESTATE;
  CtxGuard g(a->device);
  swap_status st = map_all(a);
  if (st != SWAP_OK) unmap_all(a);
  return st;
}

swap_status swap_arena_reacquire_range(swap_arena_t* a, uint64_t offset, uint64_t bytes) {
  if (!a || offset > a->bytes || bytes > a->bytes - offset) return SWAP_EINVAL;
  if (bytes == 0) return SWAP_OK;
  CtxGuard g(a->device);
  for (uint64_t i = offset / kSlab; i <= (offset + bytes - 1) / kSlab; ++i) {
    swap_status st = map_slab(a, i);
    if (st != SWAP_OK) return st;
  }
  return SWAP_OK;
}

swap_status swap_arena_export(swap_arena_t* a, int* fds, size_t cap, size_t* n, uint64_t* slab_bytes) {
  if (!a || !n || (cap && !fds)) return SWAP_EINVAL;
  *n = n_slabs(a);
  if (slab_bytes) *slab_bytes = kSlab;
  if (!fds) return SWAP_OK;
  if (cap < *n) return SWAP_EINVAL;
  if (!a->resident) {
    a->err = "swap_arena_export needs every slab mapped (re-acquire first)";
    return SWAP_ESTATE;
  }
  const Drv& D = drv();
  if (!D.export_h) return SWAP_EUNSUPPORTED;
  CtxGuard g(a->device);
  for (uint64_t i = 0; i < *n; ++i) {
    int fd = -1;
    const CUresult r = D.export_h(&fd, a->slabs[i], CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0);
    if (r != CUDA_SUCCESS) {
      for (uint64_t k = 0; k < i; ++k) close(fds[k]);
      a->err = "cuMemExportToShareableHandle failed (" + std::to_string((int)r) + ")";
      return SWAP_ECUDA;
    }
    fds[i] = fd;
  }
  return SWAP_OK;
}

// A peer arena mapped into this process: reserved VA + imported slabs.
struct swap_arena_view {
  int device = 0;
  CUdeviceptr base = 0;
  uint64_t bytes = 0;
  struct Slab {
    CUmemGenericAllocationHandle h;
    uint64_t off, size;
  };
  std::vector<Slab> slabs;
};

void swap_arena_unimport(swap_arena_view_t* v);

swap_status swap_arena_import(int device, const int* fds, size_t n, uint64_t slab_bytes, uint64_t total_bytes,
                              swap_arena_view_t** out, uint64_t* dev_addr) {
  if (!fds || !out || !dev_addr || n == 0 || slab_bytes == 0 || total_bytes == 0 ||
      (total_bytes + slab_bytes - 1) / slab_bytes != n)
    return SWAP_EINVAL;
  *out = nullptr;
  CtxGuard g(device);
  const Drv& D = drv();
  if (!D.ok || !D.import_h) return SWAP_EUNSUPPORTED;
  auto* v = new (std::nothrow) swap_arena_view();
  if (!v) return SWAP_ENOMEM;
  v->device = device;
  v->bytes = total_bytes;
  if (D.reserve(&v->base, total_bytes, slab_bytes, 0, 0) != CUDA_SUCCESS) {
    delete v;
    return SWAP_ENOMEM;
  }
  CUmemAccessDesc acc;
  std::memset(&acc, 0, sizeof(acc));
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = device;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  for (size_t i = 0; i < n; ++i) {
    const uint64_t off = i * slab_bytes, sz = total_bytes - off < slab_bytes ? total_bytes - off : slab_bytes;
    CUmemGenericAllocationHandle h;
    void* fd_as_handle = reinterpret_cast<void*>(static_cast<uintptr_t>(fds[i]));
    if (D.import_h(&h, fd_as_handle, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR) != CUDA_SUCCESS) {
      swap_arena_unimport(v);
      return SWAP_ECUDA;
    }
    if (D.map(v->base + off, sz, 0, h, 0) != CUDA_SUCCESS) {
      D.release(h);
      swap_arena_unimport(v);
      return SWAP_ECUDA;
    }
    v->slabs.push_back(swap_arena_view::Slab{h, off, sz});
    if (D.set_access(v->base + off, sz, &acc, 1) != CUDA_SUCCESS) {
      swap_arena_unimport(v);
      return SWAP_ECUDA;
    }
  }
  *out = v;
  *dev_addr = (uint64_t)v->base;
  return SWAP_OK;
}

void swap_arena_unimport(swap_arena_view_t* v) {
  if (!v) return;
  {
    CtxGuard g(v->device);
    const Drv& D = drv();
    for (const auto& sl : v->slabs) {
      D.unmap(v->base + sl.off, sl.size);
      D.release(sl.h);
    }
    if (v->base) D.addr_free(v->base, v->bytes);
  }
  delete v;
}

const char* swap_arena_last_error(const swap_arena_t* a) { return a ? a->err.c_str() : "null arena"; }

void swap_arena_destroy(swap_arena_t* a) {
  if (!a) return;
  {
    CtxGuard g(a->device);
    cudaDeviceSynchronize();
    unmap_all(a);
    drv().addr_free(a->base, a->bytes);
  }
  delete a;
}

}  // extern "C"

namespace swarena {
uint64_t slab_bytes() { return kSlab; }
uint64_t n_slabs(const swap_arena* a) { return ::n_slabs(a); }
uint64_t slab_size(const swap_arena* a, uint64_t i) { return ::slab_size(a, i); }
bool slab_mapped(const swap_arena* a, uint64_t i) { return a->slabs[i] != 0; }
uint64_t mapped_bytes(const swap_arena* a) {
  uint64_t b = 0;
  for (uint64_t i = 0; i < a->slabs.size(); ++i)
    if (a->slabs[i]) b += ::slab_size(a, i);
  return b;
}
uint64_t slab_of(const swap_arena* a, uint64_t dev) { return (dev - a->base) / kSlab; }
swap_status map_slab(swap_arena* a, uint64_t i) { return ::map_slab(a, i); }
swap_status unmap_slab(swap_arena* a, uint64_t i) {  // caller guarantees no pending device work uses it
  if (!a->slabs[i]) return SWAP_OK;
  const Drv& D = drv();
  const bool ok = D.unmap(a->base + i * kSlab, ::slab_size(a, i)) == CUDA_SUCCESS && D.release(a->slabs[i]) == CUDA_SUCCESS;
  a->slabs[i] = 0;
  --a->n_mapped;
  a->resident = false;
  return ok ? SWAP_OK : SWAP_ECUDA;
}
bool contains(const swap_arena* a, uint64_t lo, uint64_t hi) { return lo >= a->base && hi <= a->base + a->bytes; }
bool resident(const swap_arena* a) { return a->resident; }
int device(const swap_arena* a) { return a->device; }
swap_status map_dev_range(swap_arena* a, uint64_t lo, uint64_t hi) {
  if (hi <= lo) return SWAP_OK;
  return swap_arena_reacquire_range(a, lo - a->base, hi - lo);
}
}  // namespace swarena
