// probe_smem_base.cu — where does a kernel's dynamic shared memory start (shared-window address)?
// nvcc -gencode arch=compute_100a,code=sm_100a -o tools/probe_smem_base tools/probe_smem_base.cu
#include <cstdio>
#include <cstdint>
__global__ void k(uint32_t* out) {
  extern __shared__ __align__(128) uint8_t s[];
  if (threadIdx.x == 0) out[blockIdx.x] = (uint32_t)__cvta_generic_to_shared(s);
}
int main() {
  uint32_t* d; cudaMalloc(&d, 4 * 296);
  size_t sizes[] = {1024, 100 * 1024, 200 * 1024, 227 * 1024};
  for (size_t sz : sizes) {
    cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sz);
    k<<<296, 64, sz>>>(d);
    uint32_t h[296]; cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
    uint32_t mn = ~0u, mx = 0; for (int i = 0; i < 296; ++i) { mn = h[i] < mn ? h[i] : mn; mx = h[i] > mx ? h[i] : mx; }
    printf("dyn smem %zu: base min 0x%x max 0x%x (%s)\n", sz, mn, mx, cudaGetErrorString(cudaGetLastError()));
  }
}
