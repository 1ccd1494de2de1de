// probe_tma.cu — host-link mover variants (not product code): LDG/STG with L2 fetch-size
// hints vs TMA bulk copies (cp.async.bulk) staged through shared memory, both directions.
// nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o tools/probe_tma tools/probe_tma.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <cuda_profiler_api.h>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

template <int HINT>
__device__ __forceinline__ int4 ld(const void* p) {
  int4 r;
  if (HINT == 0)
    asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  else if (HINT == 1)
    asm volatile("ld.global.nc.L1::no_allocate.L2::128B.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.L2::256B.v4.s32 {%0,%1,%2,%3}, [%4];" : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

template <int U, int HINT>
__global__ void __launch_bounds__(512) ldg_copy(const char* src, char* dst, size_t n) {
  const size_t warp = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const size_t nwarps = (gridDim.x * (size_t)blockDim.x) >> 5;
  const size_t step = (size_t)U * 512;
  for (size_t base = warp * step; base + step <= n; base += nwarps * step) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) v[u] = ld<HINT>(src + base + u * 512 + lane * 16);
#pragma unroll
    for (int u = 0; u < U; ++u) *reinterpret_cast<int4*>(dst + base + u * 512 + lane * 16) = v[u];
  }
}

__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// One elected thread per CTA drives a STAGES-deep ring: bulk load (global->smem, mbarrier
// complete_tx) then bulk store (smem->global, bulk_group).
template <int STAGES>
__global__ void tma_copy(const char* src, char* dst, size_t n, uint32_t tile) {
  extern __shared__ __align__(128) char smem[];
  __shared__ __align__(8) uint64_t bar[STAGES];
  if (threadIdx.x != 0) return;
  const size_t ntiles = n / tile;
  const size_t my = ntiles > blockIdx.x ? (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x : 0;
  for (int s = 0; s < STAGES; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar[s])));
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  auto load = [&](size_t k) {
    const int s = k % STAGES;
    const size_t t = blockIdx.x + k * gridDim.x;
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&bar[s])), "r"(tile) : "memory");
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 ::"r"(sa(smem + (size_t)s * tile)), "l"(src + t * tile), "r"(tile), "r"(sa(&bar[s])) : "memory");
  };
  for (size_t k = 0; k < my && k < STAGES; ++k) load(k);
  for (size_t k = 0; k < my; ++k) {
    const int s = k % STAGES;
    const uint32_t ph = (k / STAGES) & 1;
    asm volatile("{\n.reg .pred p;\nW%=:\nmbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n@!p bra W%=;\n}"
                 ::"r"(sa(&bar[s])), "r"(ph) : "memory");
    const size_t t = blockIdx.x + k * gridDim.x;
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(dst + t * tile),
                 "r"(sa(smem + (size_t)s * tile)), "r"(tile) : "memory");
    asm volatile("cp.async.bulk.commit_group;" ::: "memory");
    if (k >= 1 && k - 1 + STAGES < my) {
      asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory");
      load(k - 1 + STAGES);
    }
  }
  asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

typedef void (*launcher)(const char*, char*, size_t, cudaStream_t);

static float timeit(launcher f, const char* src, char* dst, size_t n, cudaStream_t s) {
  cudaEvent_t a, b;
  CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  f(src, dst, n, s);
  CK(cudaGetLastError());
  CK(cudaEventRecord(a, s));
  for (int r = 0; r < 3; ++r) f(src, dst, n, s);
  CK(cudaEventRecord(b, s));
  CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return 3.0 * n / (ms * 1e-3) / 1e9;
}

static int g_grid, g_sms;
template <int U, int H> void L_ldg(const char* s, char* d, size_t n, cudaStream_t st) { ldg_copy<U, H><<<g_grid, 512, 0, st>>>(s, d, n); }
static uint32_t g_tile;
template <int ST> void L_tma(const char* s, char* d, size_t n, cudaStream_t st) {
  size_t sm = (size_t)ST * g_tile;
  cudaFuncSetAttribute(tma_copy<ST>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  tma_copy<ST><<<g_grid, 32, sm, st>>>(s, d, n, g_tile);
}

// `probe_tma ranges`: one CE / LDG / TMA transfer of 1 GiB per direction, each in its own
// cudaProfilerStart/Stop range, for ncu --replay-mode app-range PCIe counters (profiles/r02_counters_crossover.md).
static int ranges_main() {
  const size_t n = 1ull << 30;
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  char *h, *d;
  CK(cudaHostAlloc((void**)&h, n, cudaHostAllocMapped));
  CK(cudaMalloc(&d, n));
  CK(cudaMemset(d, 3, n)); memset(h, 5, n);
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  g_grid = p.multiProcessorCount; g_tile = 16384;
  const char* names[6] = {"ce_h2d", "ce_d2h", "ldg_h2d", "stg_d2h", "tma_h2d", "tma_d2h"};
  for (int c = 0; c < 6; ++c) {
    for (int rep = 0; rep < 2; ++rep) {  // rep 0 warms up (attributes, first launch), rep 1 is profiled
      CK(cudaStreamSynchronize(s));
      if (rep) CK(cudaProfilerStart());
      switch (c) {
        case 0: CK(cudaMemcpyAsync(d, h, n, cudaMemcpyHostToDevice, s)); break;
        case 1: CK(cudaMemcpyAsync(h, d, n, cudaMemcpyDeviceToHost, s)); break;
        case 2: L_ldg<8, 0>(h, d, n, s); break;
        case 3: L_ldg<8, 0>(d, h, n, s); break;
        case 4: L_tma<4>(h, d, n, s); break;
        case 5: L_tma<4>(d, h, n, s); break;
      }
      CK(cudaStreamSynchronize(s));
      if (rep) CK(cudaProfilerStop());
    }
    printf("range %d %s %zu\n", c, names[c], n);
  }
  return 0;
}

int main(int argc, char** argv) {
  if (argc > 1 && !strcmp(argv[1], "ranges")) return ranges_main();
  size_t n = 4ull << 30;
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, 0));
  g_sms = p.multiProcessorCount;
  char *h, *d, *d2;
  CK(cudaHostAlloc((void**)&h, n, cudaHostAllocMapped));
  CK(cudaMalloc(&d, n)); CK(cudaMalloc(&d2, n));
  CK(cudaMemset(d, 3, n)); memset(h, 5, n);
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  // CE reference
  {
    cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
    for (int dir = 0; dir < 2; ++dir) {
      CK(cudaEventRecord(a, s));
      for (int r = 0; r < 3; ++r) CK(cudaMemcpyAsync(dir ? h : d, dir ? d : h, n, dir ? cudaMemcpyDeviceToHost : cudaMemcpyHostToDevice, s));
      CK(cudaEventRecord(b, s)); CK(cudaEventSynchronize(b));
      float ms; CK(cudaEventElapsedTime(&ms, a, b));
      printf("CE %s %.2f GB/s\n", dir ? "D2H" : "H2D", 3.0 * n / (ms * 1e-3) / 1e9);
    }
  }
  int grids[] = {g_sms, 2 * g_sms, 4 * g_sms};
  for (int g : grids) {
    g_grid = g;
    printf("LDG grid=%d  U8: H2D h0 %.2f h1 %.2f h2 %.2f | D2H h0 %.2f h2 %.2f\n", g,
           timeit(L_ldg<8, 0>, h, d, n, s), timeit(L_ldg<8, 1>, h, d, n, s), timeit(L_ldg<8, 2>, h, d, n, s),
           timeit(L_ldg<8, 0>, d, h, n, s), timeit(L_ldg<8, 2>, d, h, n, s));
    printf("LDG grid=%d  U4: H2D h0 %.2f h2 %.2f | U16 H2D h0 %.2f h2 %.2f\n", g,
           timeit(L_ldg<4, 0>, h, d, n, s), timeit(L_ldg<4, 2>, h, d, n, s),
           timeit(L_ldg<16, 0>, h, d, n, s), timeit(L_ldg<16, 2>, h, d, n, s));
  }
  uint32_t tiles[] = {4096, 16384, 32768};
  int tgrids[] = {g_sms, 2 * g_sms, 4 * g_sms};
  for (uint32_t t : tiles) for (int g : tgrids) {
    g_tile = t; g_grid = g;
    printf("TMA tile=%6u grid=%4d ST4: H2D %.2f D2H %.2f | ST6 H2D %.2f D2H %.2f | HBM d2d ST4 %.1f\n", t, g,
           timeit(L_tma<4>, h, d, n, s), timeit(L_tma<4>, d, h, n, s),
           t <= 16384 ? timeit(L_tma<6>, h, d, n, s) : 0.f, t <= 16384 ? timeit(L_tma<6>, d, h, n, s) : 0.f,
           timeit(L_tma<4>, d, d2, n, s));
  }
  // correctness spot check of the TMA path
  g_tile = 16384; g_grid = g_sms;
  CK(cudaMemset(d2, 0, n));
  L_tma<4>(d, d2, n, s); CK(cudaStreamSynchronize(s));
  char x[64]; CK(cudaMemcpy(x, d2 + n - 64, 64, cudaMemcpyDeviceToHost));
  printf("tma check: %d %d\n", x[0], x[63]);
  return 0;
}
