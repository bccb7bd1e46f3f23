// K1: fused feature encode + pilot MLP forward (§IV-A, §IV-C;
// DESIGN.md R3, R5).
//
// B200 design: one thread-block cluster per sub-batch of <= kBs samples. Every stage (the
// three input-feature layers form one stage, then each MLP layer, then the output layer)
// splits its output rows across the C CTAs of the cluster; a warp owns a row, streams the
// row's fp32 weights with 16-byte loads (L2-resident across calls), reuses them for all
// samples of the sub-batch, reduces with warp shuffles, applies bias + LeakyReLU and writes
// the value into the activation buffer of every CTA of the cluster through distributed shared
// memory (DSMEM); one cluster barrier separates stages. The encode stage (R3) is computed
// redundantly by each CTA straight into its shared activation buffer (no HBM round trip).
// Precision: fp32 weights, fp64 products / accumulation / activations (an fp32 x fp32 product is
// exact in fp64); the batch-1 GEMV chain is latency-bound, so B200's FP64 pipe costs nothing
// measurable and the logits meet the north_star's 1e-5 relative gate against the fp64 oracle
// with ~1e-12 to spare; decode decisions are taken on the fp64 logits (same precision as the
// oracle). fp32 logits are an optional copy for the caller.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <cstdint>

#include "dyo_internal.h"

namespace cg = cooperative_groups;

namespace dyo {

constexpr int kBs = 8;          // samples per cluster
constexpr int kPilotThreads = 256;

template <class T>
__device__ __forceinline__ T scale_elem(int e, int v) {
  // R3: counts and idiom sums x 2^-4, dimension sums x 2^-10 (exact in fp32: v < 2^24)
  return (T)((float)v * (e < 7 ? 0.0625f : 0.0009765625f));
}

// Feature vector of one sample into x[0..F) (R3). Threads of the block cooperate.
// History table (R3): the executed block vectors of the previous dyo_pilot_predict, stored per
// prediction at [b * K_max + g] with K[b] groups each; history ids index their concatenation
// in sample order (>= 0 from the start, < 0 from the end).
template <class T>
__device__ void encode_one(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                           const int32_t* hist_tab, const int32_t* hist_K, int hist_B, T* x) {
  const int F = a.F;
  const int xs0 = 3, xa0 = 3 + a.D_s, xh0 = xa0 + 10 * a.S_max, end = xh0 + 10 * a.h;
  for (int i = threadIdx.x; i < F; i += blockDim.x) {
    float v = 0.f;
    if (i < 3) {
      v = (i == a.nn_type) ? 1.f : 0.f;
    } else if (i < xa0) {
      int64_t d = desc[i - xs0];
      d = d < 0 ? 0 : (d > kSat ? kSat : d);
      v = (float)d * 0.0009765625f;
    } else if (i < xh0) {
      int s = (i - xa0) / 10, e = (i - xa0) % 10;
      v = scale_elem<float>(e, a.seg_table[s * 10 + e]);
    } else if (i < end) {
      int k = (i - xh0) / 10, e = (i - xh0) % 10;
      if (hist && hist_B > 0) {
        int hl = 0;
        for (int b = 0; b < hist_B; ++b) hl += hist_K[b];
        const int gid = hist[k];
        int idx = gid >= 0 ? gid : hl + gid;
        if (idx >= 0 && idx < hl) {
          int b = 0;
          while (idx >= hist_K[b]) { idx -= hist_K[b]; ++b; }
          v = scale_elem<float>(e, hist_tab[((int64_t)b * a.K_max + idx) * 10 + e]);
        }
      }
    }
    x[i] = (T)v;
  }
}

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

// ---- TMA bulk copy + mbarrier helpers (sm_90+/sm_100a PTX) ----------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count));
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAIT_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}

// Per-launch plan of which stages are staged in shared memory (computed on the host for the
// chosen cluster size C): stage s is staged iff st_off[s] >= 0; st_off = byte offset of the
// CTA's weight slice (same for every rank; the slice size is bounded by st_bytes[s]).
struct StagePlan {
  int C;
  int Bs;                 // samples per cluster
  int act_off;            // byte offset of the activation buffers
  int st_off[4 + kMaxLayers];
};

// grid = n_clusters * C (cluster dims C set at launch). Dynamic smem:
//   [mbarriers][staged weight slices][activations 2 x Bs x max_width doubles]
template <int BS>
__global__ void __launch_bounds__(kPilotThreads)
pilot_kernel(ArchDev a, PilotDev p, StagePlan sp, const float* __restrict__ feat,
             const int64_t* __restrict__ desc, const int32_t* __restrict__ hist,
             const int32_t* __restrict__ hist_tab, const int32_t* __restrict__ hist_K, int hist_B, int B,
             double* __restrict__ logits64, float* __restrict__ logits32, int32_t* __restrict__ zero_status) {
  extern __shared__ __align__(128) unsigned char smem_raw[];
  cg::cluster_group cluster = cg::this_cluster();
  const int C = sp.C;
  const int r = (int)cluster.block_rank();
  const int cluster_id = blockIdx.x / C;
  const int Bs = sp.Bs;
  const int b0 = cluster_id * Bs;
  const int nb = min(Bs, B - b0);
  const int W = p.max_width;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem_raw);
  double* act = reinterpret_cast<double*>(smem_raw + sp.act_off);
  double* buf[2] = {act, act + Bs * W};

  // ---- 0. issue every staged weight slice of this CTA at once (TMA bulk, one mbarrier/stage)
  if (blockIdx.x == 0 && threadIdx.x == 0 && zero_status) { zero_status[0] = 0; zero_status[1] = 0; }
  if (threadIdx.x == 0) {
    for (int si = 0; si < p.n_stages; ++si) mbar_init(&bars[si], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int si = 0; si < p.n_stages; ++si) {
      if (sp.st_off[si] < 0) continue;
      const StageDev st = p.st[si];
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
      mbar_expect_tx(&bars[si], bytes);
      unsigned char* dst = smem_raw + sp.st_off[si];
      lr0 = 0;
      for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l) {
        const int lr1 = lr0 + p.ly[l].out_len;
        const int a0 = max(r0, lr0), a1 = min(r1, lr1);
        if (a1 > a0) {
          const uint32_t nbytes = (uint32_t)(a1 - a0) * p.ly[l].in_pad * 4;
          tma_bulk_g2s(dst, p.ly[l].W + (int64_t)(a0 - lr0) * p.ly[l].in_pad, nbytes, &bars[si]);
          dst += nbytes;
        }
        lr0 = lr1;
      }
    }
  }
  // ---- 1. encode (or load) the sub-batch's feature vectors into buf[0] (overlaps the TMA)
  for (int bb = 0; bb < nb; ++bb) {
    double* x = buf[0] + bb * W;
    if (feat) {
      for (int i = threadIdx.x; i < p.F; i += blockDim.x) x[i] = (double)feat[(int64_t)(b0 + bb) * p.F + i];
    } else {
      encode_one<double>(a, desc + (int64_t)(b0 + bb) * a.D_s, hist ? hist + (int64_t)(b0 + bb) * a.h : nullptr,
                         hist_tab, hist_K, hist_B, x);
    }
  }
  __syncthreads();

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  int cur = 0;
  for (int si = 0; si < p.n_stages; ++si) {
    const StageDev st = p.st[si];
    const bool last = (si == p.n_stages - 1);
    const bool staged = sp.st_off[si] >= 0;
    const int rpc = (st.rows + C - 1) / C;
    const int r0 = r * rpc, r1 = min(st.rows, r0 + rpc);
    const double* in = buf[cur];
    double* out = buf[cur ^ 1];
    if (staged) mbar_wait(&bars[si], 0);
    for (int row = r0 + warp; row < r1; row += nwarps) {
      int li = st.first_layer, rowl = row, lr0 = 0;
      while (rowl >= p.ly[li].out_len) { rowl -= p.ly[li].out_len; lr0 += p.ly[li].out_len; ++li; }
      const LayerDev ly = p.ly[li];
      const float* wrow;
      if (staged) {
        // byte offset of this row inside the CTA's staged slice: rows of earlier layers first
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
      double acc[BS];
#pragma unroll
      for (int bb = 0; bb < BS; ++bb) acc[bb] = 0.0;
#pragma unroll 4
      for (int k = lane * 4; k < ly.in_pad; k += 128) {
        const float4 w = staged ? *reinterpret_cast<const float4*>(wrow + k)
                                : __ldg(reinterpret_cast<const float4*>(wrow + k));
        const double wv[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          if (k + q < ly.in_len) {
#pragma unroll
            for (int bb = 0; bb < BS; ++bb)
              if (bb < nb) acc[bb] = fma(wv[q], in[bb * W + ly.in_off + k + q], acc[bb]);
          }
        }
      }
      const double bias = (double)__ldg(ly.b + rowl);
#pragma unroll
      for (int bb = 0; bb < BS; ++bb) {
        if (bb < nb) {
          double v = warp_sum(acc[bb]) + bias;
          if (st.act) v = v > 0.0 ? v : p.slope * v;
          if (last) {
            if (lane == 0) {
              logits64[(int64_t)(b0 + bb) * p.O + row] = v;
              if (logits32) logits32[(int64_t)(b0 + bb) * p.O + row] = (float)v;
            }
          } else if (lane < C) {
            double* dst = cluster.map_shared_rank(out, lane);
            dst[bb * W + row] = v;
          }
        }
      }
    }
    if (!last) {
      cluster.sync();
      cur ^= 1;
    }
  }
  // keep this CTA's shared memory alive until every peer finished its DSMEM writes
  // (the last exchange is followed by cluster.sync() above, so no further sync is needed)
}

cudaError_t launch_pilot(const ArchDev& a, const PilotDev& p, const float* feat_or_null,
                         const int64_t* desc, const int32_t* hist, const int32_t* hist_tab,
                         const int32_t* hist_K, int hist_B, int B, double* logits64, float* logits32,
                         int32_t* zero_status, int* cluster_used, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  static int attr_done = 0;
  if (!attr_done) {
    for (auto fn : {pilot_kernel<1>, pilot_kernel<kBs>}) {
      cudaError_t e = cudaFuncSetAttribute(fn, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
      if (e != cudaSuccess) return e;
      e = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
      if (e != cudaSuccess) return e;
    }
    attr_done = 1;
  }
  // cluster size by weight volume: spread the layers over enough SMs that each CTA's slice
  // streams in ~1 us; cached per (weights, max cluster) since cudaOccupancyMaxActiveClusters
  // is expensive
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
  sp.C = C;
  sp.Bs = B < kBs ? B : kBs;
  // shared memory: barriers, then staged slices while they fit, then activations
  const int act_bytes = 2 * sp.Bs * p.max_width * (int)sizeof(double);
  const int budget = 227 * 1024 - act_bytes;
  int off = (p.n_stages * 8 + 127) / 128 * 128;
  for (int i = 0; i < p.n_stages; ++i) {
    const StageDev& st = p.st[i];
    const int rpc = (st.rows + C - 1) / C;
    // worst-case slice of any rank: rpc rows of the widest layer of the stage
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
  sp.act_off = off;
  const size_t smem = (size_t)off + act_bytes;
  const int n_clusters = (B + sp.Bs - 1) / sp.Bs;
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(n_clusters * C);
  cfg.blockDim = dim3(kPilotThreads);
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeClusterDimension;
  attr[0].val.clusterDim.x = C;
  attr[0].val.clusterDim.y = 1;
  attr[0].val.clusterDim.z = 1;
  cfg.attrs = attr;
  cfg.numAttrs = 1;
  if (cluster_used) *cluster_used = C;
  if (sp.Bs == 1)
    return cudaLaunchKernelEx(&cfg, pilot_kernel<1>, a, p, sp, feat_or_null, desc, hist, hist_tab, hist_K, hist_B,
                              B, logits64, logits32, zero_status);
  return cudaLaunchKernelEx(&cfg, pilot_kernel<kBs>, a, p, sp, feat_or_null, desc, hist, hist_tab, hist_K, hist_B,
                            B, logits64, logits32, zero_status);
}

}  // namespace dyo
