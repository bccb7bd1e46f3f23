// A3 decode kernels for batches whose groups outnumber the pilot cluster's CTAs, for the
// tensor-core batch pilot and for the traversal decode (the fused pilot epilogue handles the
// rest; pilot.cu): a head kernel (one warp per prediction) and a group kernel (one CTA per
// (prediction, group slot)). No materialised path.
#include <cuda_runtime.h>
#include <cstdint>

#include "decode_dev.cuh"

namespace dyo {

constexpr int kDecThreads = 256;
constexpr int kDecTabCap2 = 8192;     // int32 words of decode tables staged in smem

// ---- two-phase batch decode -------------------------------------------------------------
// Phase A (one warp per prediction): head decode (R4) of the fp64 logits straight from global
// memory; writes the debug copies (slots, choices, path, K, L) and the compact head (choices,
// piece starts, group starts / counts) to pd.head. Phase B (one CTA per (prediction, group
// slot)): groups past K exit at once; the others load the compact head and build their tensor
// set. Replaces the per-(prediction, group) redundant head decode + logits staging of the
// single-phase kernel for large batches (AF: 256 group slots x O = 2,576 logits).
struct HeadSmem {
  DecHead H;
};
constexpr size_t kHeadSmemBytes = (sizeof(HeadSmem) + 15) / 16 * 16;   // fp64 logits follow, 16-byte aligned

__device__ __forceinline__ int* head_of(const PredDev& pd, int b) { return pd.head + (int64_t)b * pd.head_stride; }

__global__ void __launch_bounds__(kDecThreads)
decode_head_kernel(ArchDev a, const double* __restrict__ logits, PredDev pd, int32_t* __restrict__ hist_K) {
  extern __shared__ __align__(16) unsigned char dsm[];
  HeadSmem& S = *reinterpret_cast<HeadSmem*>(dsm);
  double* ys = reinterpret_cast<double*>(dsm + kHeadSmemBytes);
  const int b = blockIdx.x, tid = threadIdx.x, lane = tid & 31;
  if (b == 0 && tid == 0) { pd.status[0] = 0; pd.status[1] = 0; }
  // the logits into shared memory in one coalesced pass (the warp's head decode would otherwise
  // chain dependent global round trips)
  const double* yg = logits + (int64_t)b * a.O;
  for (int i = tid; i < a.O; i += blockDim.x) ys[i] = yg[i];
  __syncthreads();
  if (tid < 32) head_decode_warp(a, ys, S.H, lane, b, pd.rchoices ? pd.rchoices + (int64_t)b * a.n_sites : nullptr);
  __syncthreads();
  write_head(a, S.H, ys, pd, b, hist_K);
  int* h = head_of(pd, b);
  const int ns = a.n_sites, np = a.n_pieces, K = a.K_max;
  if (tid == 0) { h[0] = S.H.L; h[1] = S.H.nk; h[2] = S.H.K; }
  int* hc = h + 3;
  for (int i = tid; i < ns; i += blockDim.x) hc[i] = S.H.choice[i];
  int* hs = hc + ns;
  for (int i = tid; i <= np; i += blockDim.x) hs[i] = S.H.start[i];
  int* hcum = hs + np + 1;
  for (int i = tid; i < S.H.nk; i += blockDim.x) hcum[i] = S.H.cum[i];
  int* hcnt = hcum + K + 1;
  for (int i = tid; i < S.H.nk; i += blockDim.x) hcnt[i] = S.H.cntc[i];
}

struct GroupSmem {
  DecHead H;
  DecGroup G;
};

__global__ void __launch_bounds__(kDecThreads)
decode_groups_kernel(ArchDev a, PredDev pd, int32_t* __restrict__ hist_tab, int tab_cap) {
  extern __shared__ __align__(16) unsigned char dsm[];
  GroupSmem& S = *reinterpret_cast<GroupSmem*>(dsm);
  const int b = blockIdx.x / a.K_max, g = blockIdx.x % a.K_max;
  const int* h = head_of(pd, b);
  const int K = h[2];
  if (g >= K) {
    if (threadIdx.x == 0) pd.ent_n[(int64_t)b * a.K_max + g] = 0;
    return;
  }
  const int ns = a.n_sites, np = a.n_pieces;
  if (threadIdx.x == 0) { S.H.L = h[0]; S.H.nk = h[1]; S.H.K = K; }
  const int* hc = h + 3;
  for (int i = threadIdx.x; i < ns; i += blockDim.x) S.H.choice[i] = hc[i];
  const int* hs = hc + ns;
  for (int i = threadIdx.x; i <= np; i += blockDim.x) S.H.start[i] = hs[i];
  const int* hcum = hs + np + 1;
  const int* hcnt = hcum + a.K_max + 1;
  const int nk = h[1];
  for (int i = threadIdx.x; i < nk; i += blockDim.x) { S.H.cum[i] = hcum[i]; S.H.cntc[i] = hcnt[i]; }
  int* tabs = reinterpret_cast<int*>(dsm + (sizeof(GroupSmem) + 15) / 16 * 16);
  const ArchDev A = stage_decode_tables(a, tabs, tab_cap);   // ends with __syncthreads()
  build_group(A, S.H, S.G, pd, b, g, hist_tab);
}

cudaError_t launch_decode(const ArchDev& a, const double* logits, PredDev& pd, int B,
                          int32_t* hist_tab_out, int32_t* hist_K_out, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  const int tab_cap = dec_table_words(a, kDecTabCap2);
  const size_t smem = (sizeof(GroupSmem) + 15) / 16 * 16 + (size_t)tab_cap * 4;
  static size_t smem_set = 0;
  if (smem > smem_set) {
    cudaError_t e = cudaFuncSetAttribute(decode_groups_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    smem_set = smem;
  }
  const size_t hsm = kHeadSmemBytes + (size_t)a.O * sizeof(double);
  static size_t hsm_set = 0;
  if (hsm > hsm_set) {
    cudaError_t e = cudaFuncSetAttribute(decode_head_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)hsm);
    if (e != cudaSuccess) return e;
    hsm_set = hsm;
  }
  decode_head_kernel<<<B, kDecThreads, hsm, s>>>(a, logits, pd, hist_K_out);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  decode_groups_kernel<<<B * a.K_max, kDecThreads, smem, s>>>(a, pd, hist_tab_out, tab_cap);
  return cudaGetLastError();
}

}  // namespace dyo
