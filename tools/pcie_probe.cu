// PCIe / copy-mechanism probe for the B200 box (tools/, not product code).
// Measures: DMA H2D/D2H/bidir vs size; SM zero-copy gather over mapped pinned
// memory vs grid size; many-small-copies via per-copy memcpy vs batch API vs
// zero-copy kernel; empty-kernel launch and graph replay latency.
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdlib>
#include <vector>
#include <cstdint>
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("ERR %s @%d: %s\n",#x,__LINE__,cudaGetErrorString(e)); exit(1);}}while(0)

__global__ void zc_copy(const int4* __restrict__ src, int4* __restrict__ dst, size_t n16) {
  size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x;
  size_t stride = (size_t)gridDim.x * blockDim.x;
  // 4-way unrolled to keep several 16B requests in flight per thread
  for (; i + 3 * stride < n16; i += 4 * stride) {
    int4 a = src[i], b = src[i + stride], c = src[i + 2 * stride], d = src[i + 3 * stride];
    dst[i] = a; dst[i + stride] = b; dst[i + 2 * stride] = c; dst[i + 3 * stride] = d;
  }
  for (; i < n16; i += stride) dst[i] = src[i];
}
// gather many small tensors: one warp per tensor chunk list
__global__ void zc_gather(const char* __restrict__ hostbase, char* __restrict__ devbase,
                          const int64_t* __restrict__ soff, const int64_t* __restrict__ doff,
                          const int64_t* __restrict__ nb, int n) {
  int w = (blockIdx.x * blockDim.x + threadIdx.x) >> 5, lane = threadIdx.x & 31;
  int nw = (gridDim.x * blockDim.x) >> 5;
  for (int t = w; t < n; t += nw) {
    const int4* s = (const int4*)(hostbase + soff[t]);
    int4* d = (int4*)(devbase + doff[t]);
    int64_t m = nb[t] >> 4;
    for (int64_t k = lane; k < m; k += 32) d[k] = s[k];
  }
}
__global__ void empty_k() {}

static float ms_of(cudaEvent_t a, cudaEvent_t b) { float m; cudaEventElapsedTime(&m, a, b); return m; }

int main() {
  setvbuf(stdout, NULL, _IONBF, 0);
  int dev = 0; CK(cudaSetDevice(dev));
  cudaDeviceProp p; CK(cudaGetDeviceProperties(&p, dev));
  printf("GPU %s SMs=%d pciBus=%d pciDomain=%d canMapHost=%d\n", p.name, p.multiProcessorCount, p.pciBusID, p.pciDomainID, p.canMapHostMemory);
  const size_t MAXB = (size_t)1 << 30;
  char *h, *h2, *d, *d2;
  CK(cudaHostAlloc(&h, MAXB, cudaHostAllocMapped | cudaHostAllocPortable));
  CK(cudaHostAlloc(&h2, MAXB, cudaHostAllocMapped | cudaHostAllocPortable));
  for (size_t i = 0; i < MAXB; i += 4096) { h[i] = 1; h2[i] = 2; }
  CK(cudaMalloc(&d, MAXB)); CK(cudaMalloc(&d2, MAXB));
  char *hd, *h2d; CK(cudaHostGetDevicePointer((void**)&hd, h, 0)); CK(cudaHostGetDevicePointer((void**)&h2d, h2, 0));
  cudaStream_t s1, s2; CK(cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking)); CK(cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking));
  cudaEvent_t e0, e1, e2, e3; cudaEventCreate(&e0); cudaEventCreate(&e1); cudaEventCreate(&e2); cudaEventCreate(&e3);
  // DMA sweep
  size_t sizes[] = {4096, 65536, 1 << 20, 4 << 20, 16 << 20, 64 << 20, 256 << 20, 1 << 30};
  for (size_t sz : sizes) {
    int reps = sz < (16 << 20) ? 50 : 5;
    for (int dir = 0; dir < 2; dir++) {
      cudaMemcpyAsync(dir ? h : d, dir ? d : h, sz, dir ? cudaMemcpyDeviceToHost : cudaMemcpyHostToDevice, s1);
      cudaEventRecord(e0, s1);
      for (int r = 0; r < reps; r++) cudaMemcpyAsync(dir ? h : d, dir ? d : h, sz, dir ? cudaMemcpyDeviceToHost : cudaMemcpyHostToDevice, s1);
      cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
      double t = ms_of(e0, e1) / reps;
      printf("DMA %s size=%zu  %.3f us  %.2f GB/s\n", dir ? "D2H" : "H2D", sz, t * 1e3, sz / t / 1e6);
    }
  }
  // bidirectional 256 MiB
  {
    size_t sz = 256 << 20; int reps = 5;
    CK(cudaDeviceSynchronize());
    cudaEventRecord(e0, s1); cudaStreamWaitEvent(s2, e0);
    for (int r = 0; r < reps; r++) { cudaMemcpyAsync(d, h, sz, cudaMemcpyHostToDevice, s1); cudaMemcpyAsync(h2, d2, sz, cudaMemcpyDeviceToHost, s2); }
    cudaEventRecord(e2, s2); cudaStreamWaitEvent(s1, e2); cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
    double t = ms_of(e0, e1) / reps;
    printf("DMA BIDIR 256MiB each way: %.3f ms  aggregate %.2f GB/s\n", t, 2.0 * sz / t / 1e6);
  }
  // zero-copy kernels vs grid
  int grids[] = {4, 8, 16, 32, 64, 148, 296};
  for (int g : grids) {
    size_t sz = 256 << 20; size_t n16 = sz / 16; int reps = 5;
    for (int dir = 0; dir < 2; dir++) {
      const int4* src = (const int4*)(dir ? d : hd); int4* dst = (int4*)(dir ? hd : d);
      zc_copy<<<g, 1024, 0, s1>>>(src, dst, n16);
      cudaEventRecord(e0, s1);
      for (int r = 0; r < reps; r++) zc_copy<<<g, 1024, 0, s1>>>(src, dst, n16);
      cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1)); CK(cudaGetLastError());
      double t = ms_of(e0, e1) / reps;
      printf("ZC %s grid=%d 256MiB  %.2f GB/s\n", dir ? "D2H" : "H2D", g, sz / t / 1e6);
    }
  }
  // zero-copy bidir with 2 kernels concurrently
  {
    size_t sz = 256 << 20; size_t n16 = sz / 16; int reps = 5;
    CK(cudaDeviceSynchronize());
    cudaEventRecord(e0, s1); cudaStreamWaitEvent(s2, e0);
    for (int r = 0; r < reps; r++) { zc_copy<<<32, 1024, 0, s1>>>((const int4*)hd, (int4*)d, n16); zc_copy<<<32, 1024, 0, s2>>>((const int4*)d2, (int4*)h2d, n16); }
    cudaEventRecord(e2, s2); cudaStreamWaitEvent(s1, e2); cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
    double t = ms_of(e0, e1) / reps;
    printf("ZC BIDIR 32+32 CTAs: aggregate %.2f GB/s\n", 2.0 * sz / t / 1e6);
  }
  // DMA H2D concurrently with ZC D2H
  // many small copies: 10000 x 4KiB scattered
  for (int tsz : {4096, 65536}) {
    int n = 10000; std::vector<int64_t> so(n), dofs(n), nb(n);
    for (int i = 0; i < n; i++) { so[i] = ((int64_t)((i * 7919) % n)) * tsz * 2; dofs[i] = (int64_t)i * tsz; nb[i] = tsz; }
    int64_t *dso, *ddo, *dnb; cudaMalloc(&dso, n * 8); cudaMalloc(&ddo, n * 8); cudaMalloc(&dnb, n * 8);
    cudaMemcpy(dso, so.data(), n * 8, cudaMemcpyHostToDevice); cudaMemcpy(ddo, dofs.data(), n * 8, cudaMemcpyHostToDevice); cudaMemcpy(dnb, nb.data(), n * 8, cudaMemcpyHostToDevice);
    CK(cudaDeviceSynchronize());
    cudaEventRecord(e0, s1);
    for (int i = 0; i < n; i++) cudaMemcpyAsync(d + dofs[i], h + so[i], tsz, cudaMemcpyHostToDevice, s1);
    cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
    double t = ms_of(e0, e1);
    printf("SMALL %d x %d memcpyAsync: %.3f ms %.2f GB/s\n", n, tsz, t, (double)n * tsz / t / 1e6);
    for (int g : {16, 64, 148}) {
      zc_gather<<<g, 512, 0, s1>>>(hd, d, dso, ddo, dnb, n);
      cudaEventRecord(e0, s1);
      zc_gather<<<g, 512, 0, s1>>>(hd, d, dso, ddo, dnb, n);
      cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1)); CK(cudaGetLastError());
      t = ms_of(e0, e1);
      printf("SMALL %d x %d zc_gather grid=%d: %.3f ms %.2f GB/s\n", n, tsz, g, t, (double)n * tsz / t / 1e6);
    }
  }
  // launch latency
  {
    CK(cudaDeviceSynchronize());
    cudaEventRecord(e0, s1);
    for (int i = 0; i < 1000; i++) empty_k<<<1, 32, 0, s1>>>();
    cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
    printf("empty kernel stream launch: %.3f us each\n", ms_of(e0, e1));
    cudaGraph_t gr; cudaGraphExec_t ge;
    cudaStreamBeginCapture(s1, cudaStreamCaptureModeGlobal);
    for (int i = 0; i < 100; i++) empty_k<<<1, 32, 0, s1>>>();
    cudaStreamEndCapture(s1, &gr); cudaGraphInstantiate(&ge, gr, 0);
    cudaGraphLaunch(ge, s1); CK(cudaStreamSynchronize(s1));
    cudaEventRecord(e0, s1);
    for (int i = 0; i < 10; i++) cudaGraphLaunch(ge, s1);
    cudaEventRecord(e1, s1); CK(cudaEventSynchronize(e1));
    printf("empty kernel graph node: %.3f us each\n", ms_of(e0, e1) / 1000 * 1e3);
  }
  printf("done\n");
  return 0;
}
