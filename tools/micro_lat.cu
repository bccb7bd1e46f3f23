// Dependent-load latency: explicit shared (LDS), generic pointer into shared (LD), global L1/L2 hit.
#include <cuda_runtime.h>
#include <cstdio>
__device__ unsigned long long out[8];
__global__ void k(int* g, int n, int sel) {
  __shared__ int sm[4096];
  for (int i = threadIdx.x; i < 4096; i += blockDim.x) sm[i] = (i * 17 + 1) & 4095;
  __syncthreads();
  int* gp = sel ? sm : g;          // generic pointer (runtime-selected address space)
  int x = 0;
  long long t0 = clock64();
  for (int i = 0; i < n; ++i) x = sm[x];                   // LDS chain
  long long t1 = clock64();
  for (int i = 0; i < n; ++i) x = gp[x];                   // generic chain
  long long t2 = clock64();
  for (int i = 0; i < n; ++i) x = g[x];                    // global chain (L1 hits after first pass)
  long long t3 = clock64();
  if (threadIdx.x == 0) { out[0] = (t1 - t0) / n; out[1] = (t2 - t1) / n; out[2] = (t3 - t2) / n; out[3] = x; }
}
int main() {
  int* g; cudaMalloc(&g, 4096 * 4);
  int h[4096]; for (int i = 0; i < 4096; ++i) h[i] = (i * 17 + 1) & 4095;
  cudaMemcpy(g, h, sizeof h, cudaMemcpyHostToDevice);
  unsigned long long o[8];
  for (int sel = 0; sel < 2; ++sel) {
    k<<<1, 32>>>(g, 2000, sel); cudaDeviceSynchronize();
    k<<<1, 32>>>(g, 2000, sel); cudaDeviceSynchronize();
    cudaMemcpyFromSymbol(o, out, sizeof o);
    printf("sel=%d (generic -> %s): LDS %llu cyc | generic %llu cyc | global %llu cyc per dependent load\n", sel, sel ? "shared" : "global", o[0], o[1], o[2]);
  }
  return 0;
}
