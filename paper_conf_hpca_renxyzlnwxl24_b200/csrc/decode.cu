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
  pdl_enter();
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

// Phase B: one CTA per (prediction, group slot) - or, for the full-capacity pass, a grid-stride
// loop over the slots the first pass left pending. R = record capacity: the first pass runs with
// R = kRecSmall (~17 KB of shared memory: the whole batch fits in one wave), a group with more
// records is marked pending (ent_n = -1) and rebuilt by the kRecCap pass.
template <int R>
__global__ void __launch_bounds__(kDecThreads)
decode_groups_kernel(ArchDev a, PredDev pd, int32_t* __restrict__ hist_tab, int tab_cap, int pending_pass) {
  pdl_enter();
  extern __shared__ __align__(16) unsigned char dsm[];
  DecGroupT<R>& G = *reinterpret_cast<DecGroupT<R>*>(dsm);
  int* hw = reinterpret_cast<int*>(dsm + (sizeof(DecGroupT<R>) + 15) / 16 * 16);
  const int ns = a.n_sites, np = a.n_pieces, Km = a.K_max;
  __shared__ DecHeadDyn H;
  __shared__ int s_todo;
  if (threadIdx.x == 0) {
    H.start = hw;
    H.cum = hw + np + 1;
    H.cntc = H.cum + Km + 1;
    H.choice = H.cntc + Km;
  }
  int* tabs = hw + ((np + 1 + 2 * Km + 1 + ns + 3) / 4 * 4);
  bool staged = false;
  ArchDev A = a;
  const int n_items = pd.B * Km;
  for (int item = blockIdx.x; item < n_items; item += gridDim.x) {
    const int b = item / Km, g = item % Km;
    if (pending_pass) {
      if (threadIdx.x == 0) s_todo = pd.ent_n[(int64_t)b * Km + g] == -1;
      __syncthreads();
      const int todo = s_todo;
      __syncthreads();
      if (!todo) continue;
    }
    const int* h = head_of(pd, b);
    const int K = h[2];
    if (g >= K) {
      if (threadIdx.x == 0) pd.ent_n[(int64_t)b * Km + g] = 0;
      continue;
    }
    if (threadIdx.x == 0) { H.L = h[0]; H.nk = h[1]; H.K = K; H.b = b; }
    __syncthreads();
    const int* hc = h + 3;
    for (int i = threadIdx.x; i < ns; i += blockDim.x) H.choice[i] = hc[i];
    const int* hs = hc + ns;
    for (int i = threadIdx.x; i <= np; i += blockDim.x) H.start[i] = hs[i];
    const int* hcum = hs + np + 1;
    const int* hcnt = hcum + Km + 1;
    const int nk = h[1];
    for (int i = threadIdx.x; i < nk; i += blockDim.x) { H.cum[i] = hcum[i]; H.cntc[i] = hcnt[i]; }
    if (!staged) {
      A = stage_decode_tables(a, tabs, tab_cap);   // ends with __syncthreads()
      staged = true;
    } else {
      __syncthreads();
    }
    build_group(A, H, G, pd, b, g, hist_tab);
    __syncthreads();
  }
}

template <int R>
size_t groups_smem(const ArchDev& a, int tab_cap) {
  const int hw = (a.n_pieces + 1 + 2 * a.K_max + 1 + a.n_sites + 3) / 4 * 4;
  return (sizeof(DecGroupT<R>) + 15) / 16 * 16 + (size_t)hw * 4 + (size_t)tab_cap * 4;
}

cudaError_t launch_decode(const ArchDev& a, const double* logits, PredDev& pd, int B,
                          int32_t* hist_tab_out, int32_t* hist_K_out, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  const int tab_cap = dec_table_words(a, kDecTabCap2);
  const size_t smA = groups_smem<kRecSmall>(a, tab_cap), smB = groups_smem<kRecCap>(a, tab_cap);
  static size_t setA_d[64] = {}, setB_d[64] = {}, hsm_d[64] = {};   // per device
  const int dv = current_device();
  size_t& setA = setA_d[dv];
  size_t& setB = setB_d[dv];
  if (smA > setA) {
    cudaError_t e = cudaFuncSetAttribute(decode_groups_kernel<kRecSmall>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smA);
    if (e != cudaSuccess) return e;
    setA = smA;
  }
  if (smB > setB) {
    cudaError_t e = cudaFuncSetAttribute(decode_groups_kernel<kRecCap>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smB);
    if (e != cudaSuccess) return e;
    setB = smB;
  }
  const size_t hsm = kHeadSmemBytes + (size_t)a.O * sizeof(double);
  size_t& hsm_set = hsm_d[dv];
  if (hsm > hsm_set) {
    cudaError_t e = cudaFuncSetAttribute(decode_head_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)hsm);
    if (e != cudaSuccess) return e;
    hsm_set = hsm;
  }
  cudaError_t e = launch_pdl(decode_head_kernel, dim3(B), dim3(kDecThreads), hsm, s, a, logits, pd, hist_K_out);
  if (e != cudaSuccess) return e;
  // PredDev.B = the allocation's batch: the kernels walk B x K_max items of this call only
  PredDev pb = pd;
  pb.B = B;
  // first pass: one item per CTA while the batch fits a few CTAs per SM (MoE / LSTM: 64 x 16
  // slots, one wave); larger batches (AF: 64 x 256 slots) loop over items grid-stride, so each CTA
  // stages the decode tables once instead of once per slot
  static int sms1_d[64] = {};
  int& sms1 = sms1_d[dv];
  if (!sms1) cudaDeviceGetAttribute(&sms1, cudaDevAttrMultiProcessorCount, dv);
  const int gA = B * a.K_max < 8 * sms1 ? B * a.K_max : 8 * sms1;
  e = launch_pdl(decode_groups_kernel<kRecSmall>, dim3(gA), dim3(kDecThreads), smA, s, a, pb, hist_tab_out, tab_cap, 0);
  if (e != cudaSuccess) return e;
  static int sms_d[64] = {};
  int& sms = sms_d[dv];
  if (!sms) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dv);
  const int gB = B * a.K_max < 2 * sms ? B * a.K_max : 2 * sms;
  return launch_pdl(decode_groups_kernel<kRecCap>, dim3(gB), dim3(kDecThreads), smB, s, a, pb, hist_tab_out, tab_cap, 1);
}

}  // namespace dyo
