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
template <class T>
__device__ void encode_one(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                           const int32_t* hist_tab, const int32_t* hist_len_p, T* x) {
  const int F = a.F;
  const int hl = hist_len_p ? *hist_len_p : 0;
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
      if (hist) {
        int gid = hist[k];
        int idx = gid >= 0 ? gid : hl + gid;
        if (idx >= 0 && idx < hl) v = scale_elem<float>(e, hist_tab[idx * 10 + e]);
      }
    }
    x[i] = (T)v;
  }
}

__global__ void encode_kernel(ArchDev a, const int64_t* __restrict__ desc,
                              const int32_t* __restrict__ hist, const int32_t* __restrict__ hist_tab,
                              const int32_t* __restrict__ hist_len, float* __restrict__ feat) {
  const int b = blockIdx.x;
  encode_one<float>(a, desc + (int64_t)b * a.D_s, hist ? hist + (int64_t)b * a.h : nullptr, hist_tab,
                    hist_len, feat + (int64_t)b * a.F);
}

cudaError_t launch_encode(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                          const int32_t* hist_tab, const int32_t* hist_len, int B, float* feat,
                          cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  encode_kernel<<<B, 128, 0, s>>>(a, desc, hist, hist_tab, hist_len, feat);
  return cudaGetLastError();
}

__device__ __forceinline__ double warp_sum(double v) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  return v;
}

// grid = n_clusters * C (cluster dims C set at launch); dynamic smem = 2 * kBs * max_width doubles
__global__ void __launch_bounds__(kPilotThreads)
pilot_kernel(ArchDev a, PilotDev p, const float* __restrict__ feat, const int64_t* __restrict__ desc,
             const int32_t* __restrict__ hist, const int32_t* __restrict__ hist_tab,
             const int32_t* __restrict__ hist_len, int B, double* __restrict__ logits64,
             float* __restrict__ logits32) {
  extern __shared__ double smem[];
  cg::cluster_group cluster = cg::this_cluster();
  const int C = (int)cluster.num_blocks();
  const int r = (int)cluster.block_rank();
  const int cluster_id = blockIdx.x / C;
  const int b0 = cluster_id * kBs;
  const int nb = min(kBs, B - b0);
  const int W = p.max_width;
  double* buf[2] = {smem, smem + kBs * W};

  // ---- encode (or load) the sub-batch's feature vectors into buf[0] ----
  for (int bb = 0; bb < nb; ++bb) {
    double* x = buf[0] + bb * W;
    if (feat) {
      for (int i = threadIdx.x; i < p.F; i += blockDim.x) x[i] = (double)feat[(int64_t)(b0 + bb) * p.F + i];
    } else {
      encode_one<double>(a, desc + (int64_t)(b0 + bb) * a.D_s, hist ? hist + (int64_t)(b0 + bb) * a.h : nullptr,
                         hist_tab, hist_len, x);
    }
  }
  __syncthreads();
  cluster.sync();

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int nwarps = blockDim.x >> 5;
  int cur = 0;
  for (int si = 0; si < p.n_stages; ++si) {
    const StageDev st = p.st[si];
    const bool last = (si == p.n_stages - 1);
    const int rpc = (st.rows + C - 1) / C;
    const int r0 = r * rpc, r1 = min(st.rows, r0 + rpc);
    const double* in = buf[cur];
    double* out = buf[cur ^ 1];
    for (int row = r0 + warp; row < r1; row += nwarps) {
      // locate the layer of this row
      int li = st.first_layer, rowl = row;
      while (rowl >= p.ly[li].out_len) { rowl -= p.ly[li].out_len; ++li; }
      const LayerDev ly = p.ly[li];
      const float* wrow = ly.W + (int64_t)rowl * ly.in_pad;
      double acc[kBs];
#pragma unroll
      for (int bb = 0; bb < kBs; ++bb) acc[bb] = 0.0;
      for (int k = lane * 4; k < ly.in_pad; k += 128) {
        const float4 w = __ldg(reinterpret_cast<const float4*>(wrow + k));
        const double wv[4] = {w.x, w.y, w.z, w.w};
#pragma unroll
        for (int q = 0; q < 4; ++q) {
          if (k + q < ly.in_len) {
#pragma unroll
            for (int bb = 0; bb < kBs; ++bb)
              if (bb < nb) acc[bb] = fma(wv[q], in[bb * W + ly.in_off + k + q], acc[bb]);
          }
        }
      }
      const double bias = (double)__ldg(ly.b + rowl);
#pragma unroll
      for (int bb = 0; bb < kBs; ++bb) {
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
}

cudaError_t launch_pilot(const ArchDev& a, const PilotDev& p, const float* feat_or_null,
                         const int64_t* desc, const int32_t* hist, const int32_t* hist_tab,
                         const int32_t* hist_len, int B, double* logits64, float* logits32,
                         int* cluster_used, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  // cluster size: enough CTAs to spread the largest stage's weights over SMs
  int64_t wbytes = 0;
  for (int i = 0; i < p.n_stages; ++i) {
    const StageDev& st = p.st[i];
    for (int l = st.first_layer; l < st.first_layer + st.n_layers; ++l)
      wbytes += (int64_t)p.ly[l].out_len * p.ly[l].in_pad * 4;
  }
  int C = wbytes <= (64 << 10) ? 1 : (wbytes <= (512 << 10) ? 4 : 16);
  static bool attr_set = false;
  const size_t smem = (size_t)2 * kBs * p.max_width * sizeof(double);
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(pilot_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(pilot_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
    if (e != cudaSuccess) return e;
    attr_set = true;
  }
  const int n_clusters = (B + kBs - 1) / kBs;
  for (;;) {
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
    int ncl = 0;
    if (C > 1 && (cudaOccupancyMaxActiveClusters(&ncl, pilot_kernel, &cfg) != cudaSuccess || ncl < 1)) {
      cudaGetLastError();
      C /= 2;
      continue;
    }
    cudaError_t e = cudaLaunchKernelEx(&cfg, pilot_kernel, a, p, feat_or_null, desc, hist, hist_tab,
                                       hist_len, B, logits64, logits32);
    if (cluster_used) *cluster_used = C;
    return e;
  }
}

}  // namespace dyo
