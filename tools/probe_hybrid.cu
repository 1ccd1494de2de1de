// probe_hybrid.cu — does the host link carry more when the copy engine and SM loads/stores share it?
// (not product code). The transfer of n bytes is split: the first f*n bytes by cudaMemcpyAsync on
// stream s0, the rest by a persistent 16-B LDG/STG kernel on stream s1, both started by one event.
// Aggregate GB/s = n / max(ms0, ms1). f = 1 is the CE alone, f = 0 the SM kernel alone.
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)

__global__ void __launch_bounds__(512) sm_copy(const int4* __restrict__ src, int4* __restrict__ dst, size_t n16) {
  size_t stride = (size_t)gridDim.x * blockDim.x;
  size_t i = (size_t)blockIdx.x * blockDim.x + threadIdx.x;
  for (; i + 7 * stride < n16; i += 8 * stride) {
    int4 v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) v[u] = __ldcs(src + i + u * stride);
#pragma unroll
    for (int u = 0; u < 8; ++u) __stcs(dst + i + u * stride, v[u]);
  }
  for (; i < n16; i += stride) __stcs(dst + i, __ldcs(src + i));
}

int main() {
  size_t n = 8ull << 30;
  char *h, *d;
  CK(cudaHostAlloc((void**)&h, n, cudaHostAllocMapped)); CK(cudaMalloc(&d, n));
  char* hd; CK(cudaHostGetDevicePointer((void**)&hd, h, 0));
  int sms; CK(cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0));
  cudaStream_t s0, s1; CK(cudaStreamCreateWithFlags(&s0, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking));
  cudaEvent_t a, b0, b1; CK(cudaEventCreate(&a)); CK(cudaEventCreate(&b0)); CK(cudaEventCreate(&b1));
  const double fs[] = {1.0, 0.95, 0.9, 0.85, 0.8, 0.7, 0.5, 0.0};
  for (int dir = 0; dir < 2; ++dir)
    for (int grid_mul : {1, 2})
      for (double f : fs) {
        size_t nce = ((size_t)(f * n)) & ~(size_t)4095, nsm = n - nce;
        double best = 0;
        for (int rep = 0; rep < 3; ++rep) {
          CK(cudaDeviceSynchronize());
          CK(cudaEventRecord(a, s0)); CK(cudaStreamWaitEvent(s1, a, 0));
          if (nce) {
            if (dir == 0) CK(cudaMemcpyAsync(d, h, nce, cudaMemcpyHostToDevice, s0));
            else CK(cudaMemcpyAsync(h, d, nce, cudaMemcpyDeviceToHost, s0));
          }
          if (nsm) {
            if (dir == 0) sm_copy<<<sms * grid_mul, 512, 0, s1>>>((const int4*)(hd + nce), (int4*)(d + nce), nsm / 16);
            else sm_copy<<<sms * grid_mul, 512, 0, s1>>>((const int4*)(d + nce), (int4*)(hd + nce), nsm / 16);
            CK(cudaGetLastError());
          }
          CK(cudaEventRecord(b0, s0)); CK(cudaEventRecord(b1, s1));
          CK(cudaEventSynchronize(b0)); CK(cudaEventSynchronize(b1));
          float m0, m1; CK(cudaEventElapsedTime(&m0, a, b0)); CK(cudaEventElapsedTime(&m1, a, b1));
          double gbs = n / ((m0 > m1 ? m0 : m1) * 1e-3) / 1e9;
          if (gbs > best) best = gbs;
          if (rep == 2) printf("%s grid=%dxSM f_ce=%.2f: aggregate %.2f GB/s (ce %.1f ms, sm %.1f ms)\n", dir ? "D2H" : "H2D", grid_mul, f, best, m0, m1);
        }
      }
  return 0;
}
