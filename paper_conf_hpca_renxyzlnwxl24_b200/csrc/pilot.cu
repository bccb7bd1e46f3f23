// K1: fused feature encode + pilot MLP forward + decode epilogue (§IV-A,
// §IV-C, §IV-B; R3, R4, R5).
//
// B200 design (one launch per prediction batch):
//  * one thread-block cluster of C CTAs per sub-batch; every stage (the three input-feature
//    layers form one stage, then each MLP layer, then the output layer) splits its output rows
//    over the cluster;
//  * at launch each CTA issues TMA bulk copies (cp.async.bulk + mbarrier complete_tx) of its
//    slice of EVERY layer's weights into shared memory - the bias rides in the row as the weight
//    of a constant-1 input - so the whole weight stream overlaps the layer chain;
//  * a warp computes 4 rows at once from one shared activation read and reduces them with a
//    transposed butterfly (6 shuffles instead of 20);
//  * a stage's outputs are PUSHED to the peer CTAs with st.async ... mbarrier::complete_tx:
//    each CTA waits on its own mbarrier for the expected bytes - no cluster barrier and no
//    DSMEM pull per stage (measured: cluster barrier ~400 cycles, 512-double pull ~1300 cycles);
//  * the encode stage (R3) is computed by each CTA straight into shared memory;
//  * epilogue: after one cluster barrier (logits visible), CTA r decodes the groups g = r mod C
//    of its samples (decode_dev.cuh) - for MoE's 16 groups on 16 CTAs, one group per CTA.
// Precision: fp32 weights, fp64 products / accumulation / activations (fp32 x fp32 is exact in
// fp64): the latency-bound GEMV chain does not notice B200's FP64 rate, and the logits meet the
// north_star's 1e-5 relative gate against the fp64 oracle with ~1e-12 to spare; decode decides
// on the fp64 logits (the oracle's precision). fp32 logits are an optional copy for the caller.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>

#include "decode_dev.cuh"
#include "pilot_common.cuh"
#include "dyo_internal.h"

namespace cg = cooperative_groups;

namespace dyo {

constexpr int kBs = 8;          // samples per cluster
constexpr int kDynCap = 227 * 1024 - 4096;   // dynamic smem cap (static smem holds the descriptors)
constexpr int kDecTabCap = 16384;             // int32 words of decode tables staged in smem
constexpr int kPilotThreads = 512;

__global__ void encode_kernel(ArchDev a, const int64_t* __restrict__ desc,
                              const int32_t* __restrict__ hist, const int32_t* __restrict__ hist_tab,
                              const int32_t* __restrict__ hist_K, int hist_B, float* __restrict__ feat) {
  const int b = blockIdx.x;
  encode_one<float>(a, desc + (int64_t)b * a.D_s, hist ? hist + (int64_t)b * a.h : nullptr, hist_tab,
                    hist_K, hist_B, feat + (int64_t)b * a.F);
}

cudaError_t launch_encode(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                          const int32_t* hist_tab, const int32_t* hist_K, int hist_B, int B, float* feat,
                          cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  encode_kernel<<<B, 128, 0, s>>>(a, desc, hist, hist_tab, hist_K, hist_B, feat);
  return cudaGetLastError();
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// Debug phase stamps (SM clock cycles of CTA 0), enabled by dyo_debug_pilot_stamps().
__device__ unsigned long long g_stamp[32];
__device__ int g_stamp_on;
__device__ __forceinline__ void stamp(int i, int on) {
  if (on && blockIdx.x == 0 && threadIdx.x == 0) g_stamp[i] = (unsigned long long)clock64();
}

// Per-launch plan (host-computed for the chosen cluster size C): stage s is staged in shared
// memory iff st_off[s] >= 0 (byte offset of the CTA's weight slice).
struct StagePlan {
  int C;
  int Bs;                 // samples per cluster
  int act_off;            // byte offset of the activation buffers
  int fuse_decode;        // 1: this kernel also decodes its samples (epilogue)
  int dec_tab_cap;        // int32 words of decode tables staged in smem by the epilogue
  int tab_off;            // >= 0: byte offset of the decode tables prefetched at launch (fused decode)
  int push_logits;        // 1: the output stage pushes its logits to every CTA (fused decode, C > 1)
  int red_off;            // batch path (BS > 1): byte offset of the DMMA tile table + K-split partials
  int wbuf;               // doubles per sample of each activation buffer: the widest stage, and the
                          // O logits when the output stage pushes them into a buffer (push_logits)
  int st_off[4 + kMaxLayers];
  int rpc[4 + kMaxLayers];      // rows per CTA of each stage
  int gsh[4 + kMaxLayers];      // log2 of the threads per row (k-split) of each stage
};

__device__ __forceinline__ float4 lds_f4(uint32_t a) {
  float4 v;
  asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];" : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w) : "r"(a));
  return v;
}
__device__ __forceinline__ double2 lds_d2(uint32_t a) {
  double2 v;
  asm volatile("ld.shared.v2.f64 {%0, %1}, [%2];" : "=d"(v.x), "=d"(v.y) : "r"(a));
  return v;
}

// fp32 -> fp64 by exponent rebias on the integer pipes (F2F.F64.F32 is a low-throughput
// conversion on this part and the GEMV converts every weight). Exact for normal numbers and
// zero; the loader flushes subnormal weights to zero (their contribution < 1.2e-38 |x|) and
// rejects non-finite ones.
__device__ __forceinline__ double f2d(float f) {
  const uint32_t u = __float_as_uint(f);
  const uint32_t e = (u >> 23) & 0xffu;
  uint32_t hi = (u & 0x80000000u) | ((e + 896u) << 20) | ((u & 0x7fffffu) >> 3);
  uint32_t lo = u << 29;
  if (e == 0) { hi = u & 0x80000000u; lo = 0; }
  return __hiloint2double((int)hi, (int)lo);
}

// Transposed butterfly reduction of 4 per-lane partial sums (rows 0..3) over the warp:
// 6 shuffles instead of 4 x 5. Lane l ends with the total of row ((l >> 4) & 1) * 2 + ((l >> 3) & 1).
__device__ __forceinline__ double warp_reduce4(double a0, double a1, double a2, double a3, int lane) {
  const bool hi16 = lane & 16;
  double k0 = hi16 ? a2 : a0, k1 = hi16 ? a3 : a1;
  k0 += __shfl_xor_sync(0xffffffffu, hi16 ? a0 : a2, 16);
  k1 += __shfl_xor_sync(0xffffffffu, hi16 ? a1 : a3, 16);
  const bool hi8 = lane & 8;
  double v = (hi8 ? k1 : k0) + __shfl_xor_sync(0xffffffffu, hi8 ? k0 : k1, 8);
  v += __shfl_xor_sync(0xffffffffu, v, 4);
  v += __shfl_xor_sync(0xffffffffu, v, 2);
  v += __shfl_xor_sync(0xffffffffu, v, 1);
  return v;
}

// ---- batch path (BS > 1): the stage as fp64 tensor-core tiles (DMMA) ------------------------
// D[row][n] = sum_k W[row][k] X[n][k] over 8-row x 8-sample tiles with mma.sync m8n8k4 f64
// (row.col): fp32 weights widen exactly, products and accumulation are fp64 - the same
// precision as the GEMV path, so the north_star gate holds for every batch. A tile never
// straddles two layers of the stage (the feature stage holds three); the bias rides as the
// weight of a constant-1 input (k == in_len). Each warp owns one tile and a K slice; K-split
// partials are summed in a fixed order (deterministic).
struct DmmaTile { int li, row0, nrows, w_off; };   // stage row of m = 0; w_off: floats from the slice base
constexpr int kDmmaMaxTiles = 512;       // host checks ceil(rows per CTA / 8) + layers <= this
constexpr int kDmmaRedBytes = kDmmaMaxTiles * 16 + 16 * 64 * 8;

template <int BS>
__device__ __forceinline__ void dmma_stage(const PilotDev& p, const StageDev& st, const float* wbase, bool staged,
                                           int r0, int r1, const double* in, double* out, int W, int nb,
                                           unsigned char* red_raw, bool last, bool act, double slope,
                                           double* __restrict__ logits64, float* __restrict__ logits32, int b0,
                                           int C, int r, uint32_t out_s, uint32_t cbar_s) {
  static_assert(BS == 8, "one 8-sample n-tile");
  DmmaTile* tiles = reinterpret_cast<DmmaTile*>(red_raw);
  double* red = reinterpret_cast<double*>(red_raw + kDmmaMaxTiles * 16);
  __shared__ int s_nt;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31, nwarps = blockDim.x >> 5;
  if (tid == 0) {
    int nt = 0, lr0 = 0;
    int64_t off = 0;                                    // floats of the staged slice before layer l
    for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l) {
      const int lr1 = lr0 + p.ly[l].out_len;
      const int a0 = max(r0, lr0), a1 = min(r1, lr1);
      for (int q = a0; q < a1 && nt < kDmmaMaxTiles; q += 8) {
        DmmaTile t;
        t.li = l;
        t.row0 = q;
        t.nrows = min(8, a1 - q);
        t.w_off = staged ? (int)(off + (int64_t)(q - a0) * p.ly[l].in_pad) : (q - lr0) * p.ly[l].in_pad;
        tiles[nt++] = t;
      }
      if (a1 > a0) off += (int64_t)(a1 - a0) * p.ly[l].in_pad;
      lr0 = lr1;
    }
    s_nt = nt;
  }
  __syncthreads();
  const int nt = s_nt;
  const int ks = nt >= nwarps ? 1 : nwarps / nt;        // warps per tile (K split)
  const int gm = lane >> 2, gk = lane & 3;              // fragment coordinates
  for (int t0 = warp / ks; t0 < nt; t0 += nwarps / ks) {
    const int part = warp % ks;
    const DmmaTile t = tiles[t0];
    const LayerDev& ly = p.ly[t.li];
    const float* wl = staged ? wbase + t.w_off : ly.W + t.w_off;
    const int nk = ly.in_pad >> 2;                      // k-steps of 4
    const int per = (nk + ks - 1) / ks;
    const int k0 = part * per, k1 = min(nk, k0 + per);
    const bool wrow_ok = gm < t.nrows;
    const float* wr = wl + (int64_t)gm * ly.in_pad + gk;
    const double* xr = in + gm * W + ly.in_off + gk;    // B fragment: sample n = gm, k = gk
    const bool xs_ok = gm < nb;
    double c0 = 0.0, c1 = 0.0, e0 = 0.0, e1 = 0.0;
    int kk = k0;
    for (; kk + 1 < k1; kk += 2) {
      const int ka = kk * 4 + gk, kb = ka + 4;
      const double wa = wrow_ok ? (double)wr[kk * 4] : 0.0, wb = wrow_ok ? (double)wr[kk * 4 + 4] : 0.0;
      const double xa = !xs_ok ? 0.0 : (ka < ly.in_len ? xr[kk * 4] : (ka == ly.in_len ? 1.0 : 0.0));
      const double xb = !xs_ok ? 0.0 : (kb < ly.in_len ? xr[kk * 4 + 4] : (kb == ly.in_len ? 1.0 : 0.0));
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c0), "+d"(c1) : "d"(wa), "d"(xa));
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(e0), "+d"(e1) : "d"(wb), "d"(xb));
    }
    if (kk < k1) {
      const int ka = kk * 4 + gk;
      const double wa = wrow_ok ? (double)wr[kk * 4] : 0.0;
      const double xa = !xs_ok ? 0.0 : (ka < ly.in_len ? xr[kk * 4] : (ka == ly.in_len ? 1.0 : 0.0));
      asm volatile("mma.sync.aligned.m8n8k4.row.col.f64.f64.f64.f64 {%0,%1}, {%2}, {%3}, {%0,%1};"
                   : "+d"(c0), "+d"(c1) : "d"(wa), "d"(xa));
    }
    c0 += e0;
    c1 += e1;
    // this thread holds D[gm][2 gk], D[gm][2 gk + 1]
    if (ks > 1) {
      red[warp * 64 + gm * 8 + 2 * gk] = c0;
      red[warp * 64 + gm * 8 + 2 * gk + 1] = c1;
    } else {
      const double v2[2] = {c0, c1};
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int m = gm, n = 2 * gk + h;
        if (m >= t.nrows || n >= nb) continue;
        double v = v2[h];
        if (act) v = v > 0.0 ? v : slope * v;
        const int row = t.row0 + m;
        if (last) {
          logits64[(int64_t)(b0 + n) * p.O + row] = v;
          if (logits32) logits32[(int64_t)(b0 + n) * p.O + row] = (float)v;
        } else {
          out[n * W + row] = v;
          const uint32_t laddr = out_s + (uint32_t)((n * W + row) * 8);
          for (int c = 0; c < C; ++c)
            if (c != r) st_async_b64(mapa_u32(laddr, c), v, mapa_u32(cbar_s, c));
        }
      }
    }
  }
  if (ks > 1) {
    __syncthreads();
    for (int e = tid; e < nt * 64; e += blockDim.x) {
      const int ti = e >> 6, m = (e >> 3) & 7, n = e & 7;
      const DmmaTile t = tiles[ti];
      if (m >= t.nrows || n >= nb) continue;
      double v = 0.0;
      for (int q = 0; q < ks; ++q) v += red[(ti * ks + q) * 64 + (e & 63)];
      if (act) v = v > 0.0 ? v : slope * v;
      const int row = t.row0 + m;
      if (last) {
        logits64[(int64_t)(b0 + n) * p.O + row] = v;
        if (logits32) logits32[(int64_t)(b0 + n) * p.O + row] = (float)v;
      } else {
        out[n * W + row] = v;
        const uint32_t laddr = out_s + (uint32_t)((n * W + row) * 8);
        for (int c = 0; c < C; ++c)
          if (c != r) st_async_b64(mapa_u32(laddr, c), v, mapa_u32(cbar_s, c));
      }
    }
  }
}

// grid = n_clusters * C (cluster dims C set at launch). Dynamic smem:
//   [mbarriers: n_stages (weights) + 2 (activation buffers)][staged weight slices]
//   [activations 2 x BS x wbuf doubles (wbuf = max_width, or O when the logits are pushed)]
// With fuse_decode the weight region is reused for the decode (DecHead / DecGroup) afterwards.
template <int BS>
__global__ void __launch_bounds__(kPilotThreads)
pilot_kernel(const __grid_constant__ ArchDev a, const PilotDev* __restrict__ pdev, const __grid_constant__ StagePlan spc,
             const float* __restrict__ feat, const int64_t* __restrict__ desc, const int32_t* __restrict__ hist,
             const int32_t* __restrict__ hist_tab, const int32_t* __restrict__ hist_K, int hist_B, int B,
             double* __restrict__ logits64, float* __restrict__ logits32, PredDev pd,
             int32_t* __restrict__ hist_tab_out, int32_t* __restrict__ hist_K_out) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  __shared__ __align__(16) PilotDev p;
  // the launch plan in shared memory: dynamically indexed parameter-bank reads (st_off[si], ...)
  // would each cost a dependent constant-cache miss per stage
  __shared__ __align__(16) StagePlan sp;
  const int tid = threadIdx.x;
  const int stamp_on = g_stamp_on;
  if (blockIdx.x == 0 && tid == 0) g_dec_stamp_on = stamp_on;
  stamp(0, stamp_on);
  {
    // descriptors: one round trip of 16-byte loads (dynamic indexing of the parameter bank in
    // the loops below would cost a dependent constant-cache miss each time)
    const int4* src = reinterpret_cast<const int4*>(pdev);
    int4* dst = reinterpret_cast<int4*>(&p);
    for (int i = tid; i < (int)(sizeof(PilotDev) / 16); i += blockDim.x) dst[i] = src[i];
    const int* ps = reinterpret_cast<const int*>(&spc);
    int* pd2 = reinterpret_cast<int*>(&sp);
    for (int i = tid; i < (int)(sizeof(StagePlan) / 4); i += blockDim.x) pd2[i] = ps[i];
  }
  const int C = spc.C;
  const int r = C > 1 ? (int)cg::this_cluster().block_rank() : 0;
  const int cluster_id = blockIdx.x / C;
  const int b0 = cluster_id * BS;
  const int nb = min(BS, B - b0);
  uint64_t* wbar = reinterpret_cast<uint64_t*>(smem_raw);           // one per stage
  uint64_t* abar = wbar + (4 + kMaxLayers);                         // two activation buffers
  double* act = reinterpret_cast<double*>(smem_raw + spc.act_off);
  if (tid == 0) {
    for (int i = 0; i < 4 + kMaxLayers; ++i) mbar_init(&wbar[i], 1);
    mbar_init(&abar[0], 1);
    mbar_init(&abar[1], 1);
    mbar_init(&abar[2], 1);                                       // decode tables
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncthreads();                       // descriptors + barrier inits visible in the CTA
  const int W = spc.wbuf;
  double* buf[2] = {act, act + BS * W};
  // ---- 0. TMA: lane si of warp 0 issues stage si's weight slice (all stages in flight at once)
  if (tid < p.n_stages && sp.st_off[tid] >= 0) {
    const int si = tid;
    const StageDev& st = p.st[si];
    const int rpc = (st.rows + C - 1) / C;
    const int r0 = r * rpc, r1 = min(st.rows, r0 + rpc);
    uint32_t bytes = 0;
    int lr0 = 0;
    for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l) {
      const int lr1 = lr0 + p.ly[l].out_len;
      const int a0 = max(r0, lr0), a1 = min(r1, lr1);
      if (a1 > a0) bytes += (uint32_t)(a1 - a0) * p.ly[l].in_pad * 4;
      lr0 = lr1;
    }
    mbar_expect_tx(&wbar[si], bytes);
    unsigned char* dst = smem_raw + sp.st_off[si];
    lr0 = 0;
    for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l) {
      const int lr1 = lr0 + p.ly[l].out_len;
      const int a0 = max(r0, lr0), a1 = min(r1, lr1);
      if (a1 > a0) {
        const uint32_t nbytes = (uint32_t)(a1 - a0) * p.ly[l].in_pad * 4;
        tma_bulk_g2s(dst, p.ly[l].W + (int64_t)(a0 - lr0) * p.ly[l].in_pad, nbytes, &wbar[si]);
        dst += nbytes;
      }
      lr0 = lr1;
    }
  }
  // the decode tables ride the same launch-time TMA stream (used only by the epilogue)
  if (sp.tab_off >= 0 && tid == 32) prefetch_dec_tables(a, reinterpret_cast<int*>(smem_raw + sp.tab_off), &abar[2]);
  // Programmatic dependent launch: everything above reads only what dyo_load_arch / dyo_load_pilot
  // wrote (descriptors, weights, decode tables), so it may overlap the previous kernel of the
  // stream; from here on (features, the history table, prediction outputs) the previous kernel's
  // writes must be visible. The next prediction may then start its own prologue.
  asm volatile("griddepcontrol.wait;" ::: "memory");
  if (blockIdx.x == 0 && tid == 0) { pd.status[0] = 0; pd.status[1] = 0; }
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
  stamp(1, stamp_on);
  // ---- 1. the sub-batch's feature vectors into buf[0] (overlaps the weight stream)
  for (int bb = 0; bb < nb; ++bb) {
    double* x = buf[0] + bb * W;
    if (feat) {
      for (int i = tid; i < p.F; i += blockDim.x) x[i] = (double)feat[(int64_t)(b0 + bb) * p.F + i];
    } else {
      encode_one<double>(a, desc + (int64_t)(b0 + bb) * a.D_s, hist ? hist + (int64_t)(b0 + bb) * a.h : nullptr,
                         hist_tab, hist_K, hist_B, x);
    }
  }
  // arm the activation barrier of stage 0's output (buffer 1) with the bytes the peers send
  if (C > 1 && tid == 0) {
    const int rows = p.st[0].rows, rpc = (rows + C - 1) / C;
    const int own = max(0, min(rows, (r + 1) * rpc) - r * rpc);
    mbar_expect_tx(&abar[1], (uint32_t)((rows - own) * nb * 8));
  }
  __syncthreads();
  stamp(2, stamp_on);

  const int warp = tid >> 5, lane = tid & 31;
  const uint32_t abar_s[2] = {smem_u32(&abar[0]), smem_u32(&abar[1])};
  for (int si = 0; si < p.n_stages; ++si) {
    const StageDev& st = p.st[si];
    const bool last = (si == p.n_stages - 1);
    const bool staged = sp.st_off[si] >= 0;
    const int rpc = sp.rpc[si];
    const int r0 = r * rpc, r1 = min(st.rows, r0 + rpc);
    const int cin = si & 1, cout = cin ^ 1;
    const double* in = buf[cin];
    double* out = buf[cout];
    // inputs of this stage: the peers' rows of stage si-1 (arrived via st.async) + own rows
    if (si > 0 && C > 1) mbar_wait(&abar[cin], ((si - 1) >> 1) & 1);
    // arm the barrier of the NEXT stage's inputs (this stage's outputs) before any peer can finish
    if (si > 0 && C > 1 && tid == 0 && (!last || sp.push_logits)) {
      const int own = max(0, r1 - r0);
      mbar_expect_tx(&abar[cout], (uint32_t)((st.rows - own) * nb * 8));
    }
    stamp(3 + 3 * si, stamp_on);
    if (staged) mbar_wait(&wbar[si], 0);
    stamp(4 + 3 * si, stamp_on);
    const uint32_t out_s = smem_u32(out);
    if constexpr (BS > 1) {
      dmma_stage<BS>(p, st, reinterpret_cast<const float*>(smem_raw + (staged ? sp.st_off[si] : 0)), staged, r0, r1,
                     in, out, W, nb, smem_raw + sp.red_off, last, st.act != 0, p.slope, logits64, logits32, b0, C, r,
                     out_s, abar_s[cout]);
      stamp(5 + 3 * si, stamp_on);
      if (!last) __syncthreads();
      continue;
    }
    // ---- k-split: G threads per output row (G = largest power of two with rows * G <= block),
    //      each accumulates a contiguous chunk of the row (16-byte weight loads, fp64 FMAs with
    //      two independent accumulators), then a log2(G)-step shuffle reduction ----
    const int gsh = sp.gsh[si], G = 1 << gsh;
    const int grp = tid >> gsh, part = tid & (G - 1);
    const int rows_per_pass = blockDim.x >> gsh;
    for (int row0 = r0; row0 < r1; row0 += rows_per_pass) {
      const int row = row0 + grp;
      const bool active = row < r1;
      double acc0[BS], acc1[BS];
#pragma unroll
      for (int bb = 0; bb < BS; ++bb) { acc0[bb] = 0.0; acc1[bb] = 0.0; }
      if (active) {
        // layer of this row (the feature stage holds up to three layers)
        int li = st.first_layer, rowl = row, lr0 = 0;
        while (rowl >= p.ly[li].out_len) { rowl -= p.ly[li].out_len; lr0 += p.ly[li].out_len; ++li; }
        const LayerDev& ly = p.ly[li];
        const float* wrow;
        if (staged) {
          int64_t off = 0;
          int l0 = 0;
          for (int l = st.first_layer; l < li; ++l) {
            const int l1 = l0 + p.ly[l].out_len;
            const int a0 = max(r0, l0), a1 = min(r1, l1);
            if (a1 > a0) off += (int64_t)(a1 - a0) * p.ly[l].in_pad;
            l0 = l1;
          }
          off += (int64_t)(row - max(r0, lr0)) * ly.in_pad;
          wrow = reinterpret_cast<const float*>(smem_raw + sp.st_off[si]) + off;
        } else {
          wrow = ly.W + (int64_t)rowl * ly.in_pad;
        }
        const int nq = ly.in_pad >> 2;                      // float4 chunks of the row
        const int nfull = ly.in_len >> 2;                   // chunks without the bias column
        // interleaved chunks: thread `part` takes q = part, part + G, ... so the G threads of a
        // row read consecutive 16-byte words (bank-conflict free); explicit shared-memory loads
        const uint32_t xin_s = smem_u32(in) + (uint32_t)ly.in_off * 8;
        if (staged) {
          const uint32_t w_s = smem_u32(wrow);
#pragma unroll 4
          for (int q = part; q < nfull; q += G) {
            const float4 w = lds_f4(w_s + (uint32_t)q * 16);
#pragma unroll
            for (int bb = 0; bb < BS; ++bb) {
              if (bb < nb) {
                const uint32_t xa = xin_s + (uint32_t)(bb * W + q * 4) * 8;
                const double2 x01 = ((ly.in_off & 1) == 0) ? lds_d2(xa) : make_double2(in[ly.in_off + bb * W + q * 4], in[ly.in_off + bb * W + q * 4 + 1]);
                const double2 x23 = ((ly.in_off & 1) == 0) ? lds_d2(xa + 16) : make_double2(in[ly.in_off + bb * W + q * 4 + 2], in[ly.in_off + bb * W + q * 4 + 3]);
                // two widenings on the F2F pipe, two by integer rebias (balances both pipes)
                acc0[bb] = fma((double)w.x, x01.x, acc0[bb]);
                acc1[bb] = fma(f2d(w.y), x01.y, acc1[bb]);
                acc0[bb] = fma((double)w.z, x23.x, acc0[bb]);
                acc1[bb] = fma(f2d(w.w), x23.y, acc1[bb]);
              }
            }
          }
        } else {
#pragma unroll 4
          for (int q = part; q < nfull; q += G) {
            const float4 w = __ldg(reinterpret_cast<const float4*>(wrow) + q);
            const double* xb = in + ly.in_off + q * 4;
#pragma unroll
            for (int bb = 0; bb < BS; ++bb) {
              if (bb < nb) {
                acc0[bb] = fma((double)w.x, xb[bb * W + 0], acc0[bb]);
                acc1[bb] = fma(f2d(w.y), xb[bb * W + 1], acc1[bb]);
                acc0[bb] = fma((double)w.z, xb[bb * W + 2], acc0[bb]);
                acc1[bb] = fma(f2d(w.w), xb[bb * W + 3], acc1[bb]);
              }
            }
          }
        }
        // the tail chunks (the remaining inputs and the bias column: weight of a constant 1)
        for (int q = nfull + part; q < nq; q += G) {
          const float4 w = staged ? lds_f4(smem_u32(wrow) + (uint32_t)q * 16) : __ldg(reinterpret_cast<const float4*>(wrow) + q);
          const float wv[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
          for (int qq = 0; qq < 4; ++qq) {
            const int kk = q * 4 + qq;
#pragma unroll
            for (int bb = 0; bb < BS; ++bb)
              if (bb < nb) acc0[bb] = fma(f2d(wv[qq]), kk < ly.in_len ? in[ly.in_off + bb * W + kk] : (kk == ly.in_len ? 1.0 : 0.0), acc0[bb]);
          }
        }
      }
#pragma unroll
      for (int bb = 0; bb < BS; ++bb) {
        double v = acc0[bb] + acc1[bb];
        for (int o = G >> 1; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
        if (!active || bb >= nb) continue;
        if (st.act) v = v > 0.0 ? v : p.slope * v;
        if (last) {
          if (part == 0) {
            logits64[(int64_t)(b0 + bb) * p.O + row] = v;
            if (logits32) logits32[(int64_t)(b0 + bb) * p.O + row] = (float)v;
          }
          if (sp.push_logits) {              // every CTA's decode reads the logits from its own smem
            if (part == 0) out[bb * W + row] = v;
            const uint32_t laddr = out_s + (uint32_t)((bb * W + row) * 8);
            for (int c = part; c < C; c += G)
              if (c != r) st_async_b64(mapa_u32(laddr, c), v, mapa_u32(abar_s[cout], c));
          }
        } else {
          if (part == 0) out[bb * W + row] = v;
          if (C > 1) {
            const uint32_t laddr = out_s + (uint32_t)((bb * W + row) * 8);
            for (int c = part; c < C; c += G)
              if (c != r) st_async_b64(mapa_u32(laddr, c), v, mapa_u32(abar_s[cout], c));
          }
        }
      }
    }
    stamp(5 + 3 * si, stamp_on);
    if (!last) __syncthreads();          // own rows of this stage visible to every warp
  }
  // ---- 2. fused decode epilogue: CTA r of the cluster decodes groups g == r (mod C) ----
  if (!sp.fuse_decode) return;
  const int cl = p.n_stages & 1;           // buffer holding the output stage's values
  if (sp.push_logits) {
    mbar_wait(&abar[cl], ((p.n_stages - 1) >> 1) & 1);   // the peers' logits rows arrived
    __syncthreads();                                       // own rows visible to every warp
  } else if (C > 1) {
    cg::this_cluster().sync();             // every CTA's logits written (release/acquire, cluster scope)
  } else {
    __syncthreads();
  }
  stamp(28, stamp_on);
  DecHead& H = *reinterpret_cast<DecHead*>(smem_raw + ((2 * (4 + kMaxLayers) + 2) * 8 + 127) / 128 * 128);
  DecGroup& Gs = *reinterpret_cast<DecGroup*>(reinterpret_cast<unsigned char*>(&H) + ((sizeof(DecHead) + 127) / 128 * 128));
  double* ys = reinterpret_cast<double*>(reinterpret_cast<unsigned char*>(&Gs) + ((sizeof(DecGroup) + 127) / 128 * 128));
  int* tabs = reinterpret_cast<int*>(ys + ((p.O + 15) / 16) * 16);
  ArchDev A;
  if (sp.tab_off >= 0) {
    mbar_wait(&abar[2], 0);
    A = dec_tables_view(a, reinterpret_cast<const int*>(smem_raw + sp.tab_off));
  } else {
    A = stage_decode_tables(a, tabs, sp.dec_tab_cap);
  }
  stamp(29, stamp_on);
  for (int bb = 0; bb < nb; ++bb) {
    const int b = b0 + bb;
    if (r >= a.K_max && r != 0) continue;
    const double* y = logits64 + (int64_t)b * p.O;
    if (sp.push_logits) {
      y = buf[cl] + bb * W;
    } else {
      __syncthreads();
      // the logits into shared memory in one coalesced pass (the argmax loops would otherwise
      // chain dependent L2 round trips)
      for (int i = tid; i < p.O; i += blockDim.x) ys[i] = y[i];
      __syncthreads();
      y = ys;
    }
    stamp(30, stamp_on);
    if (warp == 0) head_decode_warp(A, y, H, lane, b, (r == 0 && pd.rchoices) ? pd.rchoices + (int64_t)b * a.n_sites : nullptr);
    __syncthreads();
    stamp(26, stamp_on);
    if (r == 0) write_head(A, H, y, pd, b, hist_K_out);
    for (int g = r; g < a.K_max; g += C) {
      if (g >= H.K) {
        if (tid == 0) pd.ent_n[(int64_t)b * a.K_max + g] = 0;
        continue;
      }
      build_group(A, H, Gs, pd, b, g, hist_tab_out);
    }
    stamp(27, stamp_on);
  }
  if (stamp_on && blockIdx.x == 0 && tid == 0)
    for (int i = 0; i < 6; ++i) g_stamp[i < 5 ? 21 + i : 31] = g_dec_stamp[i];   // decode phases -> free slots
}

// Latency floor of the batch-1 pilot: the same launch shape, no work, n cluster barriers.
__global__ void __launch_bounds__(kPilotThreads) floor_kernel(int n_barriers) {
  for (int i = 0; i < n_barriers; ++i) cg::this_cluster().sync();
}

cudaError_t launch_floor(int C, int n_barriers, cudaStream_t s) {
  static uint64_t attr_done = 0;   // bit d: set on device d
  const uint64_t bit = 1ull << current_device();
  if (!(attr_done & bit)) {
    cudaError_t e = cudaFuncSetAttribute(floor_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(floor_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kDynCap);
    if (e != cudaSuccess) return e;
    attr_done |= bit;
  }
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(C);
  cfg.blockDim = dim3(kPilotThreads);
  cfg.dynamicSmemBytes = 160 * 1024;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeClusterDimension;
  at[0].val.clusterDim.x = C;
  at[0].val.clusterDim.y = 1;
  at[0].val.clusterDim.z = 1;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  return cudaLaunchKernelEx(&cfg, floor_kernel, n_barriers);
}

cudaError_t debug_stamps(int on, unsigned long long* out) {
  cudaError_t e = cudaMemcpyToSymbol(g_stamp_on, &on, sizeof(int));
  if (e == cudaSuccess && out) e = cudaMemcpyFromSymbol(out, g_stamp, sizeof(unsigned long long) * 32);
  return e;
}

cudaError_t launch_pilot(const ArchDev& a, const PilotDev& p, const PilotDev* p_dev, const float* feat_or_null,
                         const int64_t* desc, const int32_t* hist, const int32_t* hist_tab,
                         const int32_t* hist_K, int hist_B, int B, double* logits64, float* logits32,
                         PredDev& pd, int32_t* hist_tab_out, int32_t* hist_K_out, int* fused,
                         cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  static uint64_t attr_done = 0;   // bit d: set on device d
  const uint64_t bit = 1ull << current_device();
  if (!(attr_done & bit)) {
    for (auto fn : {pilot_kernel<1>, pilot_kernel<kBs>}) {
      cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
      if (e != cudaSuccess) return e;
      e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, kDynCap);
      if (e != cudaSuccess) return e;
    }
    attr_done |= bit;
  }
  // cluster size by weight volume (cached: cudaOccupancyMaxActiveClusters is expensive)
  int64_t wbytes = 0;
  for (int i = 0; i < p.n_stages; ++i) {
    const StageDev& st = p.st[i];
    for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l)
      wbytes += (int64_t)p.ly[l].out_len * p.ly[l].in_pad * 4;
  }
  static int64_t cached_w = -1;
  static int cached_C = 0;
  int C;
  if (wbytes == cached_w) {
    C = cached_C;
  } else {
    C = wbytes <= (64 << 10) ? 1 : (wbytes <= (512 << 10) ? 4 : 16);
    for (; C > 1; C /= 2) {
      cudaLaunchConfig_t cfg = {};
      cfg.gridDim = dim3(C);
      cfg.blockDim = dim3(kPilotThreads);
      cfg.dynamicSmemBytes = 200 * 1024;
      cudaLaunchAttribute at[1];
      at[0].id = cudaLaunchAttributeClusterDimension;
      at[0].val.clusterDim.x = C;
      at[0].val.clusterDim.y = 1;
      at[0].val.clusterDim.z = 1;
      cfg.attrs = at;
      cfg.numAttrs = 1;
      int ncl = 0;
      if (cudaOccupancyMaxActiveClusters(&ncl, pilot_kernel<kBs>, &cfg) == cudaSuccess && ncl >= 1) break;
      cudaGetLastError();
    }
    cached_w = wbytes;
    cached_C = C;
  }
  StagePlan sp{};
  sp.Bs = B < kBs ? 1 : kBs;
  // a wide pilot whose 8-sample activation buffers do not fit shared memory runs one sample per
  // cluster (the batch-1 kernel, one cluster per prediction)
  if (sp.Bs > 1 && 2 * kBs * p.max_width * (int)sizeof(double) + kDmmaRedBytes + 4096 > kDynCap) sp.Bs = 1;
  if (sp.Bs > 1) {
    // batch path: every cluster of the launch must be co-resident (one wave; measured on MoE
    // B = 64: 8 clusters of 16 CTAs -> 7 active -> two waves, 117 us; of 8 CTAs -> 74 us), so
    // halve C until the GPU holds ceil(B / 8) clusters at once. DYO_PILOT_BATCH_C overrides.
    static int bc = -1;
    if (bc < 0) { const char* e = getenv("DYO_PILOT_BATCH_C"); bc = e ? atoi(e) : 0; }
    if (bc == 1 || bc == 2 || bc == 4 || bc == 8 || bc == 16) {
      C = bc;
    } else {
      static int max_active[64][5];                // per device, per log2(C); 0 = not queried
      const int need = (B + kBs - 1) / kBs, dv = current_device();
      for (; C > 1; C /= 2) {
        int lg = 0;
        while ((1 << lg) < C) ++lg;
        int& ma = max_active[dv][lg];
        if (ma == 0) {
          cudaLaunchConfig_t cfg = {};
          cfg.gridDim = dim3(C);
          cfg.blockDim = dim3(kPilotThreads);
          cfg.dynamicSmemBytes = kDynCap;
          cudaLaunchAttribute at[1];
          at[0].id = cudaLaunchAttributeClusterDimension;
          at[0].val.clusterDim.x = C;
          at[0].val.clusterDim.y = 1;
          at[0].val.clusterDim.z = 1;
          cfg.attrs = at;
          cfg.numAttrs = 1;
          if (cudaOccupancyMaxActiveClusters(&ma, pilot_kernel<kBs>, &cfg) != cudaSuccess || ma < 1) ma = -1;
          cudaGetLastError();
        }
        if (ma >= need) break;
      }
    }
  }
  sp.C = C;
  // fuse the decode when the cluster has at least one CTA per two groups of its samples
  sp.dec_tab_cap = dec_table_words(a, kDecTabCap);
  // fuse the decode when each CTA decodes at most a few groups of its samples (traversal: the
  // host decides first, so the decode runs after it in the stand-alone kernels)
  sp.fuse_decode = (a.branch_head && !a.hp_op && sp.Bs * a.K_max <= 2 * C) ? 1 : 0;
  sp.push_logits = (sp.fuse_decode && C > 1 && sp.Bs == 1 && p.n_stages > 1) ? 1 : 0;
  sp.tab_off = -1;
  // the output stage's buffer holds O logits per sample when they are pushed (O may exceed every
  // hidden width: MoE P512 O = 544 > 512; a narrow pilot, H256, would overflow the region)
  const int o4 = (p.O + 3) / 4 * 4;
  sp.wbuf = (sp.push_logits && o4 > p.max_width) ? o4 : p.max_width;
  const int act_bytes = 2 * sp.Bs * sp.wbuf * (int)sizeof(double);
  const int base = ((2 * (4 + kMaxLayers) + 2) * 8 + 127) / 128 * 128;
  const int budget = kDynCap - act_bytes - (sp.Bs > 1 ? kDmmaRedBytes + 256 : 0);
  int off = base;
  for (int i = 0; i < p.n_stages; ++i) {
    const StageDev& st = p.st[i];
    const int rpc = (st.rows + C - 1) / C;
    sp.rpc[i] = rpc;
    int gsh = 0;
    while (gsh < 5 && rpc * (2 << gsh) <= kPilotThreads) ++gsh;
    sp.gsh[i] = gsh;
    int maxpad = 0;
    for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l) maxpad = maxpad > p.ly[l].in_pad ? maxpad : p.ly[l].in_pad;
    const int bytes = (rpc * maxpad * 4 + 127) / 128 * 128;
    if (off + bytes <= budget) {
      sp.st_off[i] = off;
      off += bytes;
    } else {
      sp.st_off[i] = -1;
    }
  }
  // the decode epilogue reuses [base, ...) after the MLP
  const int dec_bytes = (int)(((sizeof(DecHead) + 127) / 128 * 128) + ((sizeof(DecGroup) + 127) / 128 * 128) +
                              (size_t)((p.O + 15) / 16 * 16) * sizeof(double) + (size_t)sp.dec_tab_cap * 4);
  if (sp.fuse_decode && base + dec_bytes > off) off = (base + dec_bytes + 127) / 128 * 128;
  sp.act_off = off;
  size_t smem = (size_t)sp.act_off + act_bytes;
  sp.red_off = -1;
  if (sp.Bs > 1) {                        // DMMA tile table + K-split partials
    for (int i = 0; i < p.n_stages; ++i)
      if ((sp.rpc[i] + 7) / 8 + p.st[i].n_layers > kDmmaMaxTiles) return cudaErrorInvalidValue;
    sp.red_off = (int)((smem + 127) / 128 * 128);
    smem = (size_t)sp.red_off + kDmmaRedBytes;
  }
  if (sp.fuse_decode) {
    const size_t tb = (size_t)dec_table_region_words(a) * 4;
    if (smem + tb <= (size_t)kDynCap) {
      sp.tab_off = (int)((smem + 127) / 128 * 128);
      smem = (size_t)sp.tab_off + tb;
    }
  }
  if (smem > (size_t)kDynCap) return cudaErrorInvalidValue;
  const int n_clusters = (B + sp.Bs - 1) / sp.Bs;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(n_clusters * C);
  cfg.blockDim = dim3(kPilotThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[2];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = C;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  // programmatic stream serialization: the launch may begin while the stream's previous kernel
  // finishes (the kernel waits with griddepcontrol.wait before touching dependent data);
  // DYO_PILOT_PDL=0 turns it off (measurement)
  static int pdl = -1;
  if (pdl < 0) { const char* e = getenv("DYO_PILOT_PDL"); pdl = (e && e[0] == '0') ? 0 : 1; }
  attr[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[1].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 2 : 1;
  if (fused) *fused = sp.fuse_decode;
  if (sp.Bs == 1)
    return cudaLaunchKernelEx(&cfg, pilot_kernel<1>, a, p_dev, sp, feat_or_null, desc, hist, hist_tab, hist_K, hist_B,
                              B, logits64, logits32, pd, hist_tab_out, hist_K_out);
  return cudaLaunchKernelEx(&cfg, pilot_kernel<kBs>, a, p_dev, sp, feat_or_null, desc, hist, hist_tab, hist_K, hist_B,
                            B, logits64, logits32, pd, hist_tab_out, hist_K_out);
}

}  // namespace dyo
