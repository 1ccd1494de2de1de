// probe_ce.cu — copy-engine concurrency probe (not product code): H2D/D2H bandwidth with the
// transfer split over 1/2/4 streams, and piece sizes (how CE_PIPE should issue its copies).
#include <cstdio>
#include <cstdlib>
#include <cuda_runtime.h>
#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { fprintf(stderr, "CUDA %s line %d\n", cudaGetErrorString(e), __LINE__); exit(1);} } while (0)
int main() {
  size_t n = 8ull << 30;
  char *h, *d;
  CK(cudaHostAlloc((void**)&h, n, cudaHostAllocMapped)); CK(cudaMalloc(&d, n));
  cudaStream_t s[4]; for (auto& x : s) CK(cudaStreamCreateWithFlags(&x, cudaStreamNonBlocking));
  cudaEvent_t a, b[4]; CK(cudaEventCreate(&a)); for (auto& x : b) CK(cudaEventCreate(&x));
  size_t pieces[] = {1u << 20, 16u << 20, 256u << 20, 1u << 30};
  for (int dir = 0; dir < 2; ++dir)
    for (int ns : {1, 2, 4})
      for (size_t piece : pieces) {
        for (int rep = 0; rep < 2; ++rep) {
          CK(cudaDeviceSynchronize());
          CK(cudaEventRecord(a, s[0]));
          for (int i = 1; i < ns; ++i) CK(cudaStreamWaitEvent(s[i], a, 0));
          size_t k = 0;
          for (size_t o = 0; o < n; o += piece, ++k) {
            cudaStream_t st = s[k % ns];
            if (dir == 0) CK(cudaMemcpyAsync(d + o, h + o, piece, cudaMemcpyHostToDevice, st));
            else CK(cudaMemcpyAsync(h + o, d + o, piece, cudaMemcpyDeviceToHost, st));
          }
          for (int i = 0; i < ns; ++i) CK(cudaEventRecord(b[i], s[i]));
          float best = 0;
          for (int i = 0; i < ns; ++i) { CK(cudaEventSynchronize(b[i])); float ms; CK(cudaEventElapsedTime(&ms, a, b[i])); if (ms > best) best = ms; }
          if (rep == 1) printf("%s streams=%d piece=%5zu MiB: %.2f GB/s\n", dir ? "D2H" : "H2D", ns, piece >> 20, n / (best * 1e-3) / 1e9);
        }
      }
  // bidirectional: H2D on s0 and D2H on s1 concurrently (half each)
  CK(cudaDeviceSynchronize());
  CK(cudaEventRecord(a, s[0])); CK(cudaStreamWaitEvent(s[1], a, 0));
  CK(cudaMemcpyAsync(d, h, n / 2, cudaMemcpyHostToDevice, s[0]));
  CK(cudaMemcpyAsync(h + n / 2, d + n / 2, n / 2, cudaMemcpyDeviceToHost, s[1]));
  CK(cudaEventRecord(b[0], s[0])); CK(cudaEventRecord(b[1], s[1]));
  float m0, m1; CK(cudaEventSynchronize(b[0])); CK(cudaEventSynchronize(b[1]));
  CK(cudaEventElapsedTime(&m0, a, b[0])); CK(cudaEventElapsedTime(&m1, a, b[1]));
  printf("bidir: H2D %.2f GB/s D2H %.2f GB/s\n", n / 2 / (m0 * 1e-3) / 1e9, n / 2 / (m1 * 1e-3) / 1e9);
  return 0;
}
