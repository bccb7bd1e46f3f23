// A3 decode kernel for batches whose groups outnumber the pilot cluster's CTAs (the fused
// pilot epilogue handles the rest; pilot.cu). One CTA per (prediction b, group slot g): warp 0
// decodes the head of prediction b into shared memory (decode_dev.cuh), then the block builds
// group g. No inter-CTA dependency, no materialised path.
#include <cuda_runtime.h>
#include <cstdint>

#include "decode_dev.cuh"

namespace dyo {

constexpr int kDecThreads = 256;
constexpr int kDecTabCap2 = 8192;     // int32 words of decode tables staged in smem

struct DecSmem {
  DecHead H;
  DecGroup G;
  double ys[1];      // logits copy (O doubles, dynamic)
};

__global__ void __launch_bounds__(kDecThreads)
decode_kernel(ArchDev a, const double* __restrict__ logits, PredDev pd, int32_t* __restrict__ hist_tab,
              int32_t* __restrict__ hist_K) {
  extern __shared__ __align__(16) unsigned char dsm[];
  DecSmem& S = *reinterpret_cast<DecSmem*>(dsm);
  const int b = blockIdx.x / a.K_max, g = blockIdx.x % a.K_max;
  const double* yg = logits + (int64_t)b * a.O;
  for (int i = threadIdx.x; i < a.O; i += blockDim.x) S.ys[i] = yg[i];
  __syncthreads();
  const double* y = S.ys;
  int* tabs = reinterpret_cast<int*>(S.ys + ((a.O + 15) / 16) * 16);
  const ArchDev A = stage_decode_tables(a, tabs, kDecTabCap2);
  if (threadIdx.x < 32) head_decode_warp(A, y, S.H, threadIdx.x, b);
  __syncthreads();
  if (g == 0) write_head(A, S.H, y, pd, b, hist_K);
  if (g >= S.H.K) {
    if (threadIdx.x == 0) pd.ent_n[(int64_t)b * a.K_max + g] = 0;
    return;
  }
  build_group(A, S.H, S.G, pd, b, g, hist_tab);
}

cudaError_t launch_decode(const ArchDev& a, const double* logits, PredDev& pd, int B,
                          int32_t* hist_tab_out, int32_t* hist_K_out, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(decode_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  const size_t smem = sizeof(DecSmem) + (size_t)((a.O + 15) / 16 * 16) * sizeof(double) + (size_t)kDecTabCap2 * 4;
  decode_kernel<<<B * a.K_max, kDecThreads, smem, s>>>(a, logits, pd, hist_tab_out, hist_K_out);
  return cudaGetLastError();
}

}  // namespace dyo
