// A3 decode kernels for batches whose groups outnumber the pilot cluster's CTAs, for the
// tensor-core batch pilot and for the traversal decode (the fused pilot epilogue handles the
// rest; pilot.cu): a head kernel (one warp per prediction) and a group kernel (one CTA per
// (prediction, group slot)). No materialised path.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>

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

// First pass, one WARP per (prediction, group slot): the groups of <= 64 access records (the
// common case: MoE / AF / LSTM blocks) need no block barrier at all - rows, counts and signature
// sums by lane, a warp scan for the record positions, the record sort / dedup of build_group's
// warp path - so a CTA builds kDecThreads/32 groups at once instead of one. A group with more
// records is left pending (ent_n = -1) for the full-capacity block pass, exactly as before.
constexpr int kWarpRec = 64;
struct WarpGroupSmem {
  int32_t rec_t[kWarpRec];
  int32_t rec_m[kWarpRec];
  uint64_t key[kWarpRec];
};
struct WarpHead {                    // same member names as DecHead (build helpers are templated)
  int* start;
  int* cum;
  int* cntc;
  int* choice;
  int L, nk, K;
  int b;
};

__global__ void __launch_bounds__(kDecThreads)
decode_groups_warp_kernel(ArchDev a, PredDev pd, int32_t* __restrict__ hist_tab, int tab_cap, int hw_words) {
  pdl_enter();
  extern __shared__ __align__(16) unsigned char dsm[];
  const int nwarps = blockDim.x >> 5, warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  WarpGroupSmem* WG = reinterpret_cast<WarpGroupSmem*>(dsm);
  int* hw_all = reinterpret_cast<int*>(dsm + sizeof(WarpGroupSmem) * nwarps);
  int* tabs = hw_all + (size_t)hw_words * nwarps;
  const ArchDev A = stage_decode_tables(a, tabs, tab_cap);   // once per CTA (ends with a barrier)
  WarpGroupSmem& G = WG[warp];
  int* hw = hw_all + (size_t)hw_words * warp;
  const int ns = a.n_sites, np = a.n_pieces, Km = a.K_max;
  WarpHead H;
  H.start = hw;
  H.cum = hw + np + 1;
  H.cntc = H.cum + Km + 1;
  H.choice = H.cntc + Km;
  const int n_items = pd.B * Km;
  for (int item = blockIdx.x * nwarps + warp; item < n_items; item += gridDim.x * nwarps) {
    const int b = item / Km, g = item % Km;
    const int* h = head_of(pd, b);
    const int K = h[2];
    int32_t* ent_n = pd.ent_n + (int64_t)b * Km + g;
    if (g >= K) {
      if (lane == 0) *ent_n = 0;
      continue;
    }
    H.L = h[0]; H.nk = h[1]; H.K = K; H.b = b;
    const int* hc = h + 3;
    for (int i = lane; i < ns; i += 32) H.choice[i] = hc[i];
    const int* hs = hc + ns;
    for (int i = lane; i <= np; i += 32) H.start[i] = hs[i];
    const int* hcum = hs + np + 1;
    const int* hcnt = hcum + Km + 1;
    for (int i = lane; i < H.nk; i += 32) { H.cum[i] = hcum[i]; H.cntc[i] = hcnt[i]; }
    __syncwarp();
    const int s = group_start(H, g), e = group_end(H, g);
    const int nrows = e - s;
    if (lane == 0) {
      pd.grp[((int64_t)b * Km + g) * 2] = s;
      pd.grp[((int64_t)b * Km + g) * 2 + 1] = e;
    }
    // rows in contiguous chunks per lane: access counts and signature sums
    const int chunk = (nrows + 31) / 32;
    const int rs = s + lane * chunk, re = min(e, rs + chunk);
    long long sg[9] = {0, 0, 0, 0, 0, 0, 0, 0, 0};
    int cnt = 0;
    for (int r = rs; r < re; ++r) {
      const int op = row_op(A, H, r);
      if (op >= 0) {
        cnt += A.acc_ptr[op + 1] - A.acc_ptr[op];
#pragma unroll
        for (int k = 0; k < 9; ++k) sg[k] += A.op_sig[(int64_t)op * 9 + k];
      }
    }
#pragma unroll
    for (int k = 0; k < 9; ++k)
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) sg[k] += __shfl_xor_sync(0xffffffffu, sg[k], o);
    const int inc = warp_incl_scan(cnt, lane);
    const int n = __shfl_sync(0xffffffffu, inc, 31);
    if (n > kWarpRec) {                          // the full-capacity block pass builds it
      if (lane == 0) *ent_n = -1;
      __syncwarp();
      continue;
    }
    int pos = inc - cnt;
    for (int r = rs; r < re; ++r) {
      int it = 0;
      const int op = row_op(A, H, r, &it);
      if (op < 0) continue;
      for (int q = A.acc_ptr[op]; q < A.acc_ptr[op + 1]; ++q, ++pos) {
        G.rec_t[pos] = A.acc_t[q] + A.acc_s[q] * it + A.acc_sb[q] * b;   // R13 (validated at load)
        G.rec_m[pos] = A.acc_m[q];
      }
    }
    // block vector (R1) of the group: lanes 0..9
    if (lane < 10) {
      int v;
      if (lane == 0) {
        v = min(nrows, kSat);
      } else {
        long long x = 0;
#pragma unroll
        for (int k = 0; k < 9; ++k) if (k == lane - 1) x = sg[k];
        v = (int)min(x, (long long)kSat);
      }
      pd.blocks[((int64_t)b * Km + g) * 10 + lane] = v;
      hist_tab[((int64_t)b * Km + g) * 10 + lane] = v;
    }
    __syncwarp();
    // records -> tensors in first-access order with their mode union (build_group's warp path)
    uint64_t x = lane < n ? ((uint64_t)(uint32_t)G.rec_t[lane] << 32) | ((uint64_t)lane << 2) | (uint64_t)G.rec_m[lane] : ~0ull;
    uint64_t z = lane + 32 < n ? ((uint64_t)(uint32_t)G.rec_t[lane + 32] << 32) | ((uint64_t)(lane + 32) << 2) |
                                     (uint64_t)G.rec_m[lane + 32]
                               : ~0ull;
    warp_sort64(x, z, lane);
    G.key[lane] = x;
    G.key[lane + 32] = z;
    __syncwarp();
    uint64_t o[2];
#pragma unroll
    for (int hh = 0; hh < 2; ++hh) {
      const int i = lane + 32 * hh;
      o[hh] = ~0ull;
      if (i < n) {
        const uint32_t t = (uint32_t)(G.key[i] >> 32);
        if (i == 0 || (uint32_t)(G.key[i - 1] >> 32) != t) {
          const uint32_t p0 = (uint32_t)(G.key[i] & 0xffffffffu) >> 2;
          const uint32_t m0 = (uint32_t)G.key[i] & 3u;
          uint32_t mu = m0;
          for (int k = i + 1; k < n && (uint32_t)(G.key[k] >> 32) == t; ++k) mu |= (uint32_t)G.key[k] & 3u;
          o[hh] = ((uint64_t)p0 << 32) | ((uint64_t)t << 3) | (mu << 1) | (m0 & 1u);
        }
      }
    }
    warp_sort64(o[0], o[1], lane);
    const int u = __popc(__ballot_sync(0xffffffffu, o[0] != ~0ull)) + __popc(__ballot_sync(0xffffffffu, o[1] != ~0ull));
    int2* ent = pd.ent + ((int64_t)b * Km + g) * kEntCap;
#pragma unroll
    for (int hh = 0; hh < 2; ++hh) {
      const int i = lane + 32 * hh;
      if (i < u) {
        const uint32_t lo = (uint32_t)(o[hh] & 0xffffffffu);
        ent[i] = make_int2((int)(lo >> 3), (int)(((lo >> 1) & 3u) | ((lo & 1u) << 2)));
      }
    }
    if (lane == 0) *ent_n = u;
    __syncwarp();
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
  static int warp_on = -1;
  if (warp_on < 0) { const char* ev = getenv("DYO_DECODE_WARP"); warp_on = (ev && ev[0] == '0') ? 0 : 1; }
  if (warp_on) {
    // one warp per group slot (<= 64 records; larger groups pending for the block pass)
    const int hw_words = (a.n_pieces + 1 + 2 * a.K_max + 1 + a.n_sites + 3) / 4 * 4;
    const int nw = kDecThreads / 32;
    const size_t smW = sizeof(WarpGroupSmem) * nw + (size_t)hw_words * 4 * nw + (size_t)tab_cap * 4;
    static size_t setW_d[64] = {};
    if (smW > setW_d[dv]) {
      cudaError_t ee = cudaFuncSetAttribute(decode_groups_warp_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smW);
      if (ee != cudaSuccess) return ee;
      setW_d[dv] = smW;
    }
    const int items = B * a.K_max, blocks = (items + nw - 1) / nw;
    const int gW = blocks < 8 * sms1 ? blocks : 8 * sms1;
    e = launch_pdl(decode_groups_warp_kernel, dim3(gW), dim3(kDecThreads), smW, s, a, pb, hist_tab_out, tab_cap, hw_words);
  } else {
    const int gA = B * a.K_max < 8 * sms1 ? B * a.K_max : 8 * sms1;
    e = launch_pdl(decode_groups_kernel<kRecSmall>, dim3(gA), dim3(kDecThreads), smA, s, a, pb, hist_tab_out, tab_cap, 0);
  }
  if (e != cudaSuccess) return e;
  static int sms_d[64] = {};
  int& sms = sms_d[dv];
  if (!sms) cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dv);
  const int gB = B * a.K_max < 2 * sms ? B * a.K_max : 2 * sms;
  return launch_pdl(decode_groups_kernel<kRecCap>, dim3(gB), dim3(kDecThreads), smB, s, a, pb, hist_tab_out, tab_cap, 1);
}

}  // namespace dyo
