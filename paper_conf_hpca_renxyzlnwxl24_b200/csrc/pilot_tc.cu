// K1-TC: batched pilot forward on the 5th-generation tensor cores (§IV-C,
// L207; R3, R5; SURVEY §8(a) A2 "batch 64 on tensor cores, 3xTF32").
//
// One thread-block cluster of 16 CTAs per 64 predictions. Every MLP layer of the selected MLP
// and the output layer is a GEMM  D[out][n] = sum_k W[out][k] X[n][k]  with M = 128 output rows
// per tile (tcgen05.mma.cta_group::1.kind::tf32, A = weights from shared memory, B = the 64
// samples' activations from shared memory, D = fp32 in TMEM: lane = output row, column =
// sample). fp32 accuracy from TF32 operands by the 3xTF32 split: W = W_hi + W_lo,
// X = X_hi + X_lo (each part rounded to TF32, so the tensor core reads it exactly), and
// D = W_hi X_hi + W_hi X_lo + W_lo X_hi (the dropped W_lo X_lo is < 2^-22 |W X|).
//
// Work split (host plan, dyo_internal.h TcPlan): stage s has n_m tiles of 128 rows and its K
// split n_ks ways (n_m * n_ks <= 16); CTA r = m * n_ks + ks computes the partial product of
// tile m over K-slice ks. The partials are reduce-scattered through distributed shared memory
// (st.async into the owner CTA m * n_ks + q, which owns samples [q * 64/n_ks, ...)); the owner
// adds the bias, applies LeakyReLU, splits hi/lo and pushes the activations straight into the
// X buffers of the next stage's consumer CTAs (st.async + mbarrier complete_tx). A stage with
// more than 16 tiles (the AF output layer) gives every CTA whole tiles and needs no reduction.
//
// Warp roles: warp 0 lane 0 streams this CTA's pre-split weight chunks (host-laid-out in the
// UMMA K-major no-swizzle core-matrix layout) through a 5-slot ring with cp.async.bulk (it runs
// ahead across stages); warp 1 lane 0 issues the MMAs; warps 4-7 are the epilogue (TMEM lane
// quarter = warp % 4); all 8 warps first compute the three input-feature layers (R5) for the 64
// samples on the CUDA cores in fp64 and send them to the first stage's consumers.
// Cluster-wide progress: after stage s every CTA arrives on every CTA's `prog` mbarrier (its
// accumulator and reduce buffer are read); activations of stage s+1 are sent only after `prog`
// completes, so single X / reduce buffers are safe.
#include <cooperative_groups.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>

#include "dyo_internal.h"
#include "pilot_common.cuh"

namespace cg = cooperative_groups;

namespace dyo {

namespace {

constexpr int kThreads = 256;
constexpr int kRingBytes = kTcSlots * kTcSlotBytes;
constexpr int kXOff = kRingBytes;
constexpr int kXBytes = kTcBatch * kTcMaxKsl * 8;     // hi + lo
constexpr int kRedOff = kXOff + kXBytes;
constexpr int kRedBytes = 128 * kTcBatch * 4;
constexpr int kBarOff = kRedOff + kRedBytes;
constexpr int kScratchOff = kBarOff + 256;
constexpr int kScratchFloats = 256;                   // per warp: one sample's feature vector
constexpr int kSmemBytes = kScratchOff + 8 * kScratchFloats * 4;

__device__ __forceinline__ uint32_t tf32_rna(float x) {
  uint32_t u;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(u) : "f"(x));
  return u;
}

__device__ __forceinline__ void mbar_arrive_local(uint64_t* bar) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_remote(uint32_t raddr) {
  asm volatile("mbarrier.arrive.release.cluster.shared::cluster.b64 _, [%0];" ::"r"(raddr) : "memory");
}
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t phase) {
  asm volatile(
      "{\n"
      ".reg .pred P1;\n"
      "WAITC_%=:\n"
      "mbarrier.try_wait.parity.acquire.cluster.shared::cta.b64 P1, [%0], %1;\n"
      "@!P1 bra WAITC_%=;\n"
      "}\n" ::"r"(smem_u32(bar)),
      "r"(phase)
      : "memory");
}
__device__ __forceinline__ void st_async_b32(uint32_t raddr, uint32_t v, uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b32 [%0], %1, [%2];" ::"r"(raddr), "r"(v),
               "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void st_async_v4b32(uint32_t raddr, float a, float b, float c, float d, uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v4.b32 [%0], {%1, %2, %3, %4}, [%5];" ::"r"(raddr),
               "r"(__float_as_uint(a)), "r"(__float_as_uint(b)), "r"(__float_as_uint(c)), "r"(__float_as_uint(d)),
               "r"(rbar)
               : "memory");
}

// ---- tcgen05 ---------------------------------------------------------------------------
// Shared-memory matrix descriptor, K-major, no swizzle (canonical ((8,n),2):((1,SBO),LBO) in
// 16-byte units): lbo = byte distance between the two 16-byte K chunks of one MMA, sbo = byte
// distance between 8-row groups; version 1 (sm_100).
__device__ __forceinline__ uint64_t sdesc(uint32_t saddr, uint32_t lbo, uint32_t sbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3fffu);
  d |= (uint64_t)((lbo >> 4) & 0x3fffu) << 16;
  d |= (uint64_t)((sbo >> 4) & 0x3fffu) << 32;
  d |= (uint64_t)1 << 46;
  return d;
}
// Instruction descriptor: D f32, A/B tf32, both K-major, N = 64, M = 128.
constexpr uint32_t kIdesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(kTcBatch >> 3) << 17) | ((128u >> 4) << 24);

__device__ __forceinline__ void mma_tf32(uint32_t d_tmem, uint64_t a, uint64_t b, uint32_t acc) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(d_tmem),
      "l"(a), "l"(b), "r"(kIdesc), "r"(acc)
      : "memory");
}
__device__ __forceinline__ void mma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tc_fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void tc_fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }

__device__ __forceinline__ void tmem_ld16(uint32_t taddr, float* v) {
  uint32_t r[16];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]), "=r"(r[8]),
        "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 16; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ void tmem_ld4(uint32_t taddr, float* v) {
  uint32_t r[4];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3])
               : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 4; ++i) v[i] = __uint_as_float(r[i]);
}

// ---- plan helpers ------------------------------------------------------------------------
struct Job { int n, m[2], ks; };
__device__ __forceinline__ Job jobs_of(const TcStage& S, int r) {
  Job j{0, {0, 0}, 0};
  if (S.n_m * S.n_ks <= kTcCtas) {
    if (r < S.n_m * S.n_ks) { j.n = 1; j.m[0] = r / S.n_ks; j.ks = r % S.n_ks; }
  } else {
    for (int m = r; m < S.n_m && j.n < 2; m += kTcCtas) j.m[j.n++] = m;
  }
  return j;
}
// byte offset of X element (sample n, k) inside a K-slice buffer (K-major core matrices)
__device__ __forceinline__ uint32_t xoff(int n, int k) {
  return (uint32_t)((k >> 2) * (kTcBatch / 8 * 128) + (n >> 3) * 128 + (n & 7) * 16 + (k & 3) * 4);
}

// Send activation v of (row R of stage s's output = input R of stage s+1, sample n) to every
// consumer of stage s+1 (hi / lo TF32 parts).
__device__ __forceinline__ void send_x(const TcStage& N, int R, int n, double v, uint32_t xs, uint32_t xbar) {
  const float f = (float)v;
  const uint32_t hi = tf32_rna(f);
  const uint32_t lo = tf32_rna(f - __uint_as_float(hi));
  const int ks = R / N.ksl, k = R - ks * N.ksl;
  const uint32_t o = xoff(n, k);
  const uint32_t lo_off = (uint32_t)N.ksl * (kTcBatch * 4);
  if (N.n_m * N.n_ks <= kTcCtas) {
    for (int mm = 0; mm < N.n_m; ++mm) {
      const int c = mm * N.n_ks + ks;
      const uint32_t b = mapa_u32(xbar, c);
      st_async_b32(mapa_u32(xs + o, c), hi, b);
      st_async_b32(mapa_u32(xs + lo_off + o, c), lo, b);
    }
  } else {
    const int nc = N.n_m < kTcCtas ? N.n_m : kTcCtas;
    for (int c = 0; c < nc; ++c) {
      const uint32_t b = mapa_u32(xbar, c);
      st_async_b32(mapa_u32(xs + o, c), hi, b);
      st_async_b32(mapa_u32(xs + lo_off + o, c), lo, b);
    }
  }
}

__device__ __forceinline__ uint32_t x_bytes(const TcStage& S, int r) {
  return jobs_of(S, r).n ? (uint32_t)(kTcBatch * S.ksl * 8) : 0u;
}

}  // namespace

__global__ void __cluster_dims__(kTcCtas, 1, 1) __launch_bounds__(kThreads, 1)
pilot_tc_kernel(const __grid_constant__ ArchDev a, const PilotDev* __restrict__ pdev, const TcPlan* __restrict__ plan_g,
                const float* __restrict__ feat, const int64_t* __restrict__ desc, const int32_t* __restrict__ hist,
                const int32_t* __restrict__ hist_tab, const int32_t* __restrict__ hist_K, int hist_B, int B,
                double* __restrict__ logits64, float* __restrict__ logits32, int terms) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ TcPlan P;
  __shared__ uint32_t tmem_base_s;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int r = (int)cg::this_cluster().block_rank();
  const int b0 = (blockIdx.x / kTcCtas) * kTcBatch;
  const int nb = min(kTcBatch, B - b0);
  if (tid == 0) P = *plan_g;
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + kBarOff);
  uint64_t* empty = full + kTcSlots;
  uint64_t* xfull = empty + kTcSlots;
  uint64_t* dfull = xfull + 1;
  uint64_t* redfull = dfull + 1;
  uint64_t* prog = redfull + 1;
  const uint32_t xs = smem_u32(sm + kXOff);
  const uint32_t red_s = smem_u32(sm + kRedOff);
  __syncthreads();
  const int ns = P.n_stages;
  if (tid == 0) {
    for (int i = 0; i < kTcSlots; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(xfull, 1);
    mbar_init(dfull, 1);
    mbar_init(redfull, 1);
    mbar_init(prog, kTcCtas);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    // arm stage 0's activation and reduce buffers before any peer can send
    mbar_expect_tx(xfull, x_bytes(P.st[0], r));
    const TcStage& S0 = P.st[0];
    if (S0.n_ks > 1 && r < S0.n_m * S0.n_ks) mbar_expect_tx(redfull, (uint32_t)kRedBytes);
  }
  if (warp == 2) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 128;" ::"r"(smem_u32(&tmem_base_s)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  tc_fence_before();
  cg::this_cluster().sync();
  tc_fence_after();
  const uint32_t tmem = tmem_base_s;
  const int c0 = P.chunk_ptr[r], c1 = P.chunk_ptr[r + 1];
  // ---- weight stream: fill the ring now (overlaps the feature layers) ----
  if (tid == 0) {
    for (int i = c0; i < c1 && i < c0 + kTcSlots; ++i) {
      const TcChunk ch = P.chunks[i];
      const int slot = (i - c0) % kTcSlots;
      mbar_expect_tx(&full[slot], (uint32_t)ch.bytes);
      tma_bulk_g2s(sm + slot * kTcSlotBytes, P.blob + ch.off, (uint32_t)ch.bytes, &full[slot]);
    }
  }
  // ---- feature layers (R5) on the CUDA cores, fp64: CTA r computes features
  //      [r * fpc, (r + 1) * fpc) for all 64 samples, one sample per warp at a time ----
  {
    const int nf = P.n_feat, fpc = (nf + kTcCtas - 1) / kTcCtas;
    const int f0 = r * fpc, f1 = min(nf, f0 + fpc);
    float* xw = reinterpret_cast<float*>(sm + kScratchOff) + warp * kScratchFloats;
    const int hl = (!feat && hist && hist_B > 0) ? hist_len(hist_K, hist_B) : 0;
    const TcStage& S0 = P.st[0];
    const double slope = pdev->slope;
    for (int n = warp; n < kTcBatch; n += 8) {
      const int b = b0 + n;
      for (int i = lane; i < a.F; i += 32) {
        float v = 0.f;
        if (n < nb)
          v = feat ? feat[(int64_t)b * a.F + i]
                   : encode_elem(a, desc + (int64_t)b * a.D_s, hist ? hist + (int64_t)b * a.h : nullptr, hist_tab,
                                 hist_K, hist_B, hl, i);
        xw[i] = v;
      }
      __syncwarp();
      for (int f = f0; f < f1; ++f) {
        int li = pdev->st[0].first_layer, fl = f;
        while (fl >= pdev->ly[li].out_len) { fl -= pdev->ly[li].out_len; ++li; }
        const LayerDev& L = pdev->ly[li];
        const float* wr = L.W + (int64_t)fl * L.in_pad;
        double acc = 0.0;
        for (int k = lane; k < L.in_len; k += 32) acc = fma((double)__ldg(wr + k), (double)xw[L.in_off + k], acc);
#pragma unroll
        for (int o = 16; o > 0; o >>= 1) acc += __shfl_xor_sync(0xffffffffu, acc, o);
        acc += (double)__ldg(wr + L.in_len);                    // bias rides in the row (R5 loader)
        acc = acc > 0.0 ? acc : slope * acc;
        if (lane == 0) send_x(S0, f, n, acc, xs, smem_u32(xfull));
      }
      __syncwarp();
    }
  }
  // ---- role split ----
  if (tid == 0) {
    // TMA producer: the rest of this CTA's chunk list, gated by the ring's empty barriers
    for (int i = c0 + kTcSlots; i < c1; ++i) {
      const int q = i - c0, slot = q % kTcSlots;
      mbar_wait(&empty[slot], ((q / kTcSlots) - 1) & 1);
      const TcChunk ch = P.chunks[i];
      mbar_expect_tx(&full[slot], (uint32_t)ch.bytes);
      tma_bulk_g2s(sm + slot * kTcSlotBytes, P.blob + ch.off, (uint32_t)ch.bytes, &full[slot]);
    }
  } else if (tid == 32) {
    // MMA issuer
    int q = 0;          // chunk counter of this CTA
    for (int s = 0; s < ns; ++s) {
      const TcStage S = P.st[s];
      const Job J = jobs_of(S, r);
      mbar_wait_cluster(xfull, s & 1);
      if (J.n == 0) { mbar_arrive_local(dfull); continue; }
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      tc_fence_after();
      const uint32_t xlo = xs + (uint32_t)S.ksl * (kTcBatch * 4);
      for (int jj = 0; jj < J.n; ++jj) {
        const uint32_t d = tmem + (uint32_t)(jj * kTcBatch);
        int k0 = 0;
        while (k0 < S.ksl) {
          const TcChunk ch = P.chunks[c0 + q];
          const int slot = q % kTcSlots;
          mbar_wait(&full[slot], (q / kTcSlots) & 1);
          tc_fence_after();
          const uint32_t ahi = smem_u32(sm + slot * kTcSlotBytes);
          const uint32_t alo = ahi + (uint32_t)ch.kc * 128 * 4;
          for (int j = 0; j < ch.kc / 8; ++j) {
            const int kk = ch.k0 + 8 * j;
            const uint64_t a_hi = sdesc(ahi + (uint32_t)j * 4096u, 2048u, 128u);
            const uint64_t a_lo = sdesc(alo + (uint32_t)j * 4096u, 2048u, 128u);
            const uint64_t x_hi = sdesc(xs + (uint32_t)(kk >> 2) * 1024u, 1024u, 128u);
            const uint64_t x_lo = sdesc(xlo + (uint32_t)(kk >> 2) * 1024u, 1024u, 128u);
            const uint32_t acc0 = (k0 > 0 || j > 0) ? 1u : 0u;
            if (terms == 3) {
              mma_tf32(d, a_lo, x_hi, acc0);
              mma_tf32(d, a_hi, x_lo, 1u);
              mma_tf32(d, a_hi, x_hi, 1u);
            } else if (terms == 2) {
              mma_tf32(d, a_hi, x_lo, acc0);
              mma_tf32(d, a_hi, x_hi, 1u);
            } else if (terms == 4) {
              mma_tf32(d, a_lo, x_hi, acc0);
              mma_tf32(d, a_hi, x_hi, 1u);
            } else {
              mma_tf32(d, a_hi, x_hi, acc0);
            }
          }
          mma_commit(&empty[slot]);
          k0 += ch.kc;
          ++q;
        }
      }
      mma_commit(dfull);
    }
  } else if (warp >= 4) {
    // epilogue: thread e <-> TMEM lane e = output row e of the tile
    const int e = tid - 128;
    const uint32_t lane_base = (uint32_t)((warp & 3) * 32) << 16;
    int red_ph = 0;
    for (int s = 0; s < ns; ++s) {
      const TcStage S = P.st[s];
      const bool last = (s == ns - 1);
      const Job J = jobs_of(S, r);
      const bool owner = S.n_ks > 1 && r < S.n_m * S.n_ks;
      const float* bias = S.bias;
      mbar_wait(dfull, s & 1);
      tc_fence_after();
      float vals[kTcBatch];
      int vrow = -1, vn0 = 0, vw = 0;           // values kept for the X sends after `prog`
      if (S.n_ks == 1) {
        for (int jj = 0; jj < J.n; ++jj) {
          const int R = J.m[jj] * 128 + e;
          for (int c = 0; c < kTcBatch; c += 16) tmem_ld16(tmem + lane_base + (uint32_t)(jj * kTcBatch + c), vals + c);
          if (R < S.n_out) {
            const double bv = (double)__ldg(bias + R);
            if (last) {
              for (int n = 0; n < nb; ++n) {
                const double v = (double)vals[n] + bv;
                logits64[(int64_t)(b0 + n) * S.n_out + R] = v;
                if (logits32) logits32[(int64_t)(b0 + n) * S.n_out + R] = (float)v;
              }
            } else {
              for (int n = 0; n < kTcBatch; ++n) {
                double v = (double)vals[n] + bv;
                if (S.act) v = v > 0.0 ? v : pdev->slope * v;
                vals[n] = (float)v;
              }
              vrow = R; vn0 = 0; vw = kTcBatch;
            }
          }
        }
      } else {
        if (J.n) {
          // reduce-scatter the partial tile: columns [q w, (q+1) w) to owner m * n_ks + q
          const int w = kTcBatch / S.n_ks;
          for (int qq = 0; qq < S.n_ks; ++qq) {
            const int owner_c = J.m[0] * S.n_ks + qq;
            const uint32_t rb = mapa_u32(smem_u32(redfull), owner_c);
            for (int c = 0; c < w; c += 4) {
              float v4[4];
              tmem_ld4(tmem + lane_base + (uint32_t)(qq * w + c), v4);
              const uint32_t dst = red_s + (uint32_t)(((J.ks * 128 + e) * w + c) * 4);
              st_async_v4b32(mapa_u32(dst, owner_c), v4[0], v4[1], v4[2], v4[3], rb);
            }
          }
        }
        if (owner) {
          const int m = r / S.n_ks, qo = r % S.n_ks, w = kTcBatch / S.n_ks;
          const int R = m * 128 + e;
          mbar_wait_cluster(redfull, red_ph & 1);
          ++red_ph;
          const float* rd = reinterpret_cast<const float*>(sm + kRedOff);
          if (R < S.n_out) {
            const double bv = (double)__ldg(bias + R);
            for (int c = 0; c < w; ++c) {
              double v = bv;
              for (int k2 = 0; k2 < S.n_ks; ++k2) v += (double)rd[(k2 * 128 + e) * w + c];
              const int n = qo * w + c;
              if (last) {
                if (n < nb) {
                  logits64[(int64_t)(b0 + n) * S.n_out + R] = v;
                  if (logits32) logits32[(int64_t)(b0 + n) * S.n_out + R] = (float)v;
                }
              } else {
                if (S.act) v = v > 0.0 ? v : pdev->slope * v;
                vals[c] = (float)v;
              }
            }
            if (!last) { vrow = R; vn0 = qo * w; vw = w; }
          }
        }
      }
      if (last) break;
      // stage s consumed (TMEM read, reduce buffer read): arm stage s+1, then cluster progress
      tc_fence_before();
      asm volatile("bar.sync 1, 128;" ::: "memory");
      const TcStage N = P.st[s + 1];
      if (e == 0) {
        mbar_expect_tx(xfull, x_bytes(N, r));
        if (N.n_ks > 1 && r < N.n_m * N.n_ks) mbar_expect_tx(redfull, (uint32_t)kRedBytes);
        for (int c = 0; c < kTcCtas; ++c) mbar_arrive_remote(mapa_u32(smem_u32(prog), c));
      }
      mbar_wait_cluster(prog, s & 1);
      if (vrow >= 0)
        for (int c = 0; c < vw; ++c) send_x(N, vrow, vn0 + c, (double)vals[c], xs, smem_u32(xfull));
    }
  }
  tc_fence_before();
  __syncthreads();
  cg::this_cluster().sync();       // no CTA leaves while a peer may still address its memory
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
  }
}

cudaError_t launch_pilot_tc(const ArchDev& a, const PilotDev* p_dev, const TcPlan* plan_dev, const float* feat,
                            const int64_t* desc, const int32_t* hist, const int32_t* hist_tab, const int32_t* hist_K,
                            int hist_B, int B, double* logits64, float* logits32, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  static bool attr = false;
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(pilot_tc_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(pilot_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  const int n_clusters = (B + kTcBatch - 1) / kTcBatch;
  static int terms = -1;
  if (terms < 0) { const char* e = getenv("DYO_TC_TERMS"); terms = e ? atoi(e) : 3; }
  pilot_tc_kernel<<<n_clusters * kTcCtas, kThreads, kSmemBytes, s>>>(a, p_dev, plan_dev, feat, desc, hist, hist_tab,
                                                                    hist_K, hist_B, B, logits64, logits32, terms);
  return cudaGetLastError();
}

}  // namespace dyo
