// probe_link.cu — one-off host-link probe for the B200 box (not product code).
// Measures: copy-engine H2D/D2H bandwidth (cudaMemcpyAsync, pinned), and SM-driven
// zero-copy loads/stores to mapped pinned host memory for several grid/unroll shapes.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o probe_link tools/probe_link.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

template <int U>
__global__ void zc_copy(const int4* __restrict__ src, int4* __restrict__ dst, size_t n16) {
  const size_t warp = (blockIdx.x * (size_t)blockDim.x + threadIdx.x) >> 5;
  const int lane = threadIdx.x & 31;
  const size_t nwarps = (gridDim.x * (size_t)blockDim.x) >> 5;
  const size_t step = (size_t)U * 32;
  for (size_t base = warp * step; base < n16; base += nwarps * step) {
    int4 v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      size_t i = base + u * 32 + lane;
      if (i < n16) v[u] = src[i];
    }
#pragma unroll
    for (int u = 0; u < U; ++u) {
      size_t i = base + u * 32 + lane;
      if (i < n16) dst[i] = v[u];
    }
  }
}

static float time_ce(void* dst, const void* src, size_t bytes, size_t chunk, cudaMemcpyKind k, cudaStream_t s) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  for (int w = 0; w < 2; ++w) {
    for (size_t o = 0; o < bytes; o += chunk)
      CK(cudaMemcpyAsync((char*)dst + o, (const char*)src + o, (o + chunk > bytes ? bytes - o : chunk), k, s));
  }
  CK(cudaEventRecord(a, s));
  for (size_t o = 0; o < bytes; o += chunk)
    CK(cudaMemcpyAsync((char*)dst + o, (const char*)src + o, (o + chunk > bytes ? bytes - o : chunk), k, s));
  CK(cudaEventRecord(b, s));
  CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return bytes / (ms * 1e-3) / 1e9;
}

template <int U>
static float time_zc(const void* src, void* dst, size_t bytes, int grid, int block, cudaStream_t s) {
  cudaEvent_t a, b; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b));
  size_t n16 = bytes / 16;
  zc_copy<U><<<grid, block, 0, s>>>((const int4*)src, (int4*)dst, n16);
  CK(cudaGetLastError());
  CK(cudaEventRecord(a, s));
  const int reps = 3;
  for (int r = 0; r < reps; ++r) zc_copy<U><<<grid, block, 0, s>>>((const int4*)src, (int4*)dst, n16);
  CK(cudaEventRecord(b, s));
  CK(cudaEventSynchronize(b));
  float ms; CK(cudaEventElapsedTime(&ms, a, b));
  return reps * bytes / (ms * 1e-3) / 1e9;
}

int main(int argc, char** argv) {
  size_t bytes = (argc > 1 ? strtoull(argv[1], 0, 10) : 4096ull) << 20;
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  printf("device %s SMs=%d pciBus=%d canMapHost=%d\n", p.name, p.multiProcessorCount, p.pciBusID, p.canMapHostMemory);
  void *h, *d;
  CK(cudaHostAlloc(&h, bytes, cudaHostAllocMapped | cudaHostAllocPortable));
  CK(cudaMalloc(&d, bytes));
  CK(cudaMemset(d, 1, bytes));
  for (size_t i = 0; i < bytes; i += 4096) ((char*)h)[i] = 1;
  void* hd; CK(cudaHostGetDevicePointer(&hd, h, 0));
  cudaStream_t s; CK(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
  printf("bytes=%zu MiB\n", bytes >> 20);
  size_t chunks[] = {4096, 65536, 1 << 20, 16 << 20, bytes};
  for (size_t c : chunks) {
    printf("CE chunk=%10zu H2D %.2f GB/s  D2H %.2f GB/s\n", c,
           time_ce(d, h, bytes, c, cudaMemcpyHostToDevice, s), time_ce(h, d, bytes, c, cudaMemcpyDeviceToHost, s));
  }
  int sms = p.multiProcessorCount;
  int grids[] = {sms / 4, sms / 2, sms, 2 * sms, 4 * sms};
  int blocks[] = {128, 256, 512, 1024};
  for (int g : grids) for (int bl : blocks) {
    printf("ZC grid=%4d block=%4d  U4: H2D %.2f D2H %.2f   U8: H2D %.2f D2H %.2f   U16: H2D %.2f D2H %.2f\n", g, bl,
           time_zc<4>(hd, d, bytes, g, bl, s), time_zc<4>(d, hd, bytes, g, bl, s),
           time_zc<8>(hd, d, bytes, g, bl, s), time_zc<8>(d, hd, bytes, g, bl, s),
           time_zc<16>(hd, d, bytes, g, bl, s), time_zc<16>(d, hd, bytes, g, bl, s));
  }
  // HBM-only copy for reference
  void* d2; CK(cudaMalloc(&d2, bytes));
  printf("HBM d2d kernel U8 grid=%d: %.1f GB/s (one-direction bytes)\n", 4 * sms, time_zc<8>(d, d2, bytes, 4 * sms, 512, s));
  return 0;
}
