// Micro-benchmarks of Blackwell primitives used by the pilot kernel (tools/, not product code):
// cluster barrier round trip, TMA bulk global->shared throughput per SM, DSMEM pull latency,
// and empty-kernel / cluster-kernel launch cost. Cycle counts from clock64 in CTA 0.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
namespace cg = cooperative_groups;
#define CK(x) do{cudaError_t e=(x); if(e!=cudaSuccess){printf("ERR %s @%d: %s\n",#x,__LINE__,cudaGetErrorString(e)); return 1;}}while(0)

__device__ unsigned long long out[64];

__global__ void k_cluster_sync(int iters) {
  cg::cluster_group cl = cg::this_cluster();
  cl.sync();
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) cl.sync();
  long long t1 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) out[0] = (t1 - t0) / iters;
}
__global__ void k_syncthreads(int iters) {
  __syncthreads();
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) __syncthreads();
  long long t1 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) out[1] = (t1 - t0) / iters;
}
__device__ __forceinline__ uint32_t sa(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__global__ void k_tma(const char* src, int bytes, int chunks) {
  extern __shared__ __align__(128) unsigned char sm[];
  __shared__ __align__(8) uint64_t bar;
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sa(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();
  long long t0 = clock64();
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sa(&bar)), "r"(bytes) : "memory");
    const int cb = bytes / chunks;
    for (int c = 0; c < chunks; ++c)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                   ::"r"(sa(sm + c * cb)), "l"(src + (size_t)blockIdx.x * bytes + c * cb), "r"(cb), "r"(sa(&bar)) : "memory");
  }
  long long t1 = clock64();
  asm volatile("{\n.reg .pred P1;\nW:\nmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], 0;\n@!P1 bra W;\n}\n" ::"r"(sa(&bar)) : "memory");
  long long t2 = clock64();
  if (blockIdx.x == 0 && threadIdx.x == 0) { out[2] = t1 - t0; out[3] = t2 - t0; }
}
__global__ void k_dsmem_pull(int n) {
  __shared__ double buf[1024];
  cg::cluster_group cl = cg::this_cluster();
  for (int i = threadIdx.x; i < 1024; i += blockDim.x) buf[i] = i;
  cl.sync();
  long long t0 = clock64();
  double s = 0;
  const int C = cl.num_blocks(), r = cl.block_rank();
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    const double* rem = cl.map_shared_rank(buf, (r + 1 + (i % (C - 1 > 0 ? C - 1 : 1))) % C);
    s += rem[i % 1024];
  }
  __syncthreads();
  long long t1 = clock64();
  cl.sync();
  if (blockIdx.x == 0 && threadIdx.x == 0) { out[4] = t1 - t0; out[5] = (unsigned long long)s; }
}
__global__ void k_empty() {}

int launch_cluster(void (*k)(int), int C, int threads, int arg, size_t smem = 0) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(C); cfg.blockDim = dim3(threads); cfg.dynamicSmemBytes = smem;
  cudaLaunchAttribute at[1]; at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = C; at[0].val.clusterDim.y = 1; at[0].val.clusterDim.z = 1;
  cfg.attrs = at; cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, k, arg) != cudaSuccess;
}

int main() {
  setvbuf(stdout, NULL, _IONBF, 0);
  CK(cudaFuncSetAttribute(k_cluster_sync, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  CK(cudaFuncSetAttribute(k_dsmem_pull, cudaFuncAttributeNonPortableClusterSizeAllowed, 1));
  unsigned long long h[64];
  for (int C : {1, 2, 4, 8, 16}) {
    for (int rep = 0; rep < 2; ++rep) if (launch_cluster(k_cluster_sync, C, 256, 100)) { printf("launch fail C=%d\n", C); }
    CK(cudaDeviceSynchronize()); CK(cudaMemcpyFromSymbol(h, out, sizeof h));
    printf("cluster.sync C=%2d: %llu cycles/iter\n", C, h[0]);
  }
  k_syncthreads<<<1, 256>>>(100); CK(cudaDeviceSynchronize()); CK(cudaMemcpyFromSymbol(h, out, sizeof h));
  printf("__syncthreads 256 thr: %llu cycles/iter\n", h[1]);
  char* g; CK(cudaMalloc(&g, 64 << 20)); CK(cudaMemset(g, 1, 64 << 20));
  CK(cudaFuncSetAttribute(k_tma, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024));
  for (int bytes : {16384, 65536, 163840}) for (int chunks : {1, 8}) for (int grid : {1, 16}) {
    k_tma<<<grid, 256, bytes>>>(g, bytes, chunks); CK(cudaDeviceSynchronize());
    k_tma<<<grid, 256, bytes>>>(g, bytes, chunks); CK(cudaDeviceSynchronize());  // L2-warm
    CK(cudaMemcpyFromSymbol(h, out, sizeof h));
    printf("TMA bulk %6d B in %d chunks, grid %2d (L2 warm): issue %llu cyc, complete %llu cyc = %.1f B/cyc\n", bytes, chunks, grid, h[2], h[3], (double)bytes / h[3]);
  }
  for (int C : {2, 16}) {
    for (int rep = 0; rep < 2; ++rep) launch_cluster(k_dsmem_pull, C, 256, 512);
    CK(cudaDeviceSynchronize()); CK(cudaMemcpyFromSymbol(h, out, sizeof h));
    printf("DSMEM pull 512 doubles (256 thr) C=%2d: %llu cycles\n", C, h[4]);
  }
  // launch costs
  cudaStream_t s; CK(cudaStreamCreate(&s));
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int i = 0; i < 10; ++i) k_empty<<<1, 32, 0, s>>>();
  cudaEventRecord(a, s); for (int i = 0; i < 1000; ++i) k_empty<<<1, 32, 0, s>>>(); cudaEventRecord(b, s);
  CK(cudaEventSynchronize(b)); float ms; cudaEventElapsedTime(&ms, a, b); printf("empty launch: %.2f us each\n", ms);
  cudaEventRecord(a, s); for (int i = 0; i < 1000; ++i) launch_cluster(k_cluster_sync, 16, 256, 0); cudaEventRecord(b, s);
  CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms, a, b); printf("cluster-16 launch (0 iters): %.2f us each\n", ms);
  cudaGraph_t gr; cudaGraphExec_t ge;
  CK(cudaStreamBeginCapture(s, cudaStreamCaptureModeGlobal));
  for (int i = 0; i < 100; ++i) k_empty<<<1, 32, 0, s>>>();
  CK(cudaStreamEndCapture(s, &gr)); CK(cudaGraphInstantiate(&ge, gr, 0));
  cudaGraphLaunch(ge, s); cudaStreamSynchronize(s);
  cudaEventRecord(a, s); for (int i = 0; i < 10; ++i) cudaGraphLaunch(ge, s); cudaEventRecord(b, s);
  CK(cudaEventSynchronize(b)); cudaEventElapsedTime(&ms, a, b); printf("empty graph node: %.2f us each\n", ms * 1000 / 1000);
  return 0;
}
