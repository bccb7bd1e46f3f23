// global-load latency of small tables: one allocation vs 12 separate allocations (TLB)
#include <cuda_runtime.h>
#include <cstdio>
__device__ unsigned long long o[4];
__global__ void k(int* const* tabs, int nt, int* sink) {
  long long t0 = clock64();
  int s = 0;
  for (int r = 0; r < 4; ++r) {
    for (int i = 0; i < nt; ++i) s += __ldg(tabs[i] + threadIdx.x + r);
  }
  long long t1 = clock64();
  if (threadIdx.x == 0) o[0] = t1 - t0;
  if (s == 123456) *sink = s;
}
int main() {
  int* t[12]; int** dt; int* sink; cudaMalloc(&sink, 4);
  for (int i = 0; i < 12; ++i) { cudaMalloc(&t[i], 4096); cudaMemset(t[i], 0, 4096); }
  void* big; cudaMalloc(&big, 8ull << 30);   // a large allocation in between
  cudaMalloc(&dt, sizeof t); cudaMemcpy(dt, t, sizeof t, cudaMemcpyHostToDevice);
  unsigned long long h[4];
  for (int rep = 0; rep < 3; ++rep) {
    k<<<1, 128>>>(dt, 12, sink); cudaDeviceSynchronize(); cudaMemcpyFromSymbol(h, o, sizeof h);
    printf("12 tables x 4 dependent-free rounds: %llu cycles\n", h[0]);
    k<<<1, 128>>>(dt, 1, sink); cudaDeviceSynchronize(); cudaMemcpyFromSymbol(h, o, sizeof h);
    printf("1 table x 4 rounds: %llu cycles\n", h[0]);
  }
}
