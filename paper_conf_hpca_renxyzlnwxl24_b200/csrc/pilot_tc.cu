// K1-TC: batched pilot forward on the 5th-generation tensor cores (§IV-C,
// L207; R3, R5; SURVEY §8(a) A2 "batch 64 on tensor cores, 3xTF32").
//
// One thread-block cluster of 16 CTAs per 64 predictions. Every MLP layer of the selected MLP
// and the output layer is a GEMM  D[out][n] = sum_k W[out][k] X[n][k]  with M = 128 output rows
// per tile (tcgen05.mma.cta_group::1.kind::tf32, A = weights from shared memory, B = the 64
// samples' activations from shared memory, D = fp32 in TMEM: lane = output row, column =
// sample). Stage 0 is the three input-feature layers as one block-diagonal layer over the
// encoded features (R3/R5), which each CTA of stage 0 encodes straight into its X buffer. fp32 accuracy from TF32 operands by the 3xTF32 split: W = W_hi + W_lo,
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
// quarter = warp % 4); all 8 warps first encode the stage-0 input.
// Cluster-wide progress, two mbarriers per CTA arrived by every CTA: `progx` (its MMAs of stage s
// are done, so its X buffer may be overwritten: activations of stage s+1 are sent after it) and
// `progr` (its reduce buffer of stage s is read: partials of stage s+1 are sent after it); a
// local `tfree` keeps the next stage's MMAs off the accumulator until the epilogue has read it.
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
constexpr int kStgOff = kRedOff + kRedBytes;
constexpr int kStgBytes = 16 * 1024;                  // owner's outgoing activations (w <= 16 samples)
constexpr int kBarOff = kStgOff + kStgBytes;
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
// Wait for a phase completed by peers of the cluster: spin at CTA scope (no L1 invalidation per
// poll), then one cluster-scope acquire on the completed phase.
__device__ __forceinline__ void mbar_wait_cluster(uint64_t* bar, uint32_t phase) {
  mbar_wait(bar, phase);
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
// all 64 columns of this thread's lane (four x16 loads, one wait)
__device__ __forceinline__ void tmem_ld64(uint32_t taddr, float* v) {
  uint32_t r[64];
#pragma unroll
  for (int q = 0; q < 4; ++q)
    asm volatile(
        "tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, %15}, [%16];"
        : "=r"(r[16 * q + 0]), "=r"(r[16 * q + 1]), "=r"(r[16 * q + 2]), "=r"(r[16 * q + 3]), "=r"(r[16 * q + 4]),
          "=r"(r[16 * q + 5]), "=r"(r[16 * q + 6]), "=r"(r[16 * q + 7]), "=r"(r[16 * q + 8]), "=r"(r[16 * q + 9]),
          "=r"(r[16 * q + 10]), "=r"(r[16 * q + 11]), "=r"(r[16 * q + 12]), "=r"(r[16 * q + 13]),
          "=r"(r[16 * q + 14]), "=r"(r[16 * q + 15])
        : "r"(taddr + 16u * q));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 64; ++i) v[i] = __uint_as_float(r[i]);
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
// byte offset of X element (sample n, k) inside a K-slice buffer of ksl inputs: UMMA K-major
// no-swizzle core matrices ordered [n/8][k/4][n%8][k%4] (8-sample groups outermost, so the
// activations of 8 consecutive samples over the whole K-slice are one contiguous block)
__device__ __forceinline__ uint32_t xoff(int n, int k, int ksl) {
  return (uint32_t)((n >> 3) * (ksl * 32) + (k >> 2) * 128 + (n & 7) * 16 + (k & 3) * 4);
}

__device__ __forceinline__ uint32_t x_bytes(const TcStage& S, int r) {
  return jobs_of(S, r).n ? (uint32_t)(kTcBatch * S.ksl * 8) : 0u;
}

__device__ unsigned long long g_tc_stamp[32];
__device__ int g_tc_on;
__device__ __forceinline__ void tstamp(int i, int on) {
  if (on && blockIdx.x == 0) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_tc_stamp[i] = t;
  }
}

}  // namespace

__global__ void __cluster_dims__(kTcCtas, 1, 1) __launch_bounds__(kThreads, 1)
pilot_tc_kernel(const __grid_constant__ ArchDev a, const PilotDev* __restrict__ pdev, const TcPlan* __restrict__ plan_g,
                const float* __restrict__ feat, const int64_t* __restrict__ desc, const int32_t* __restrict__ hist,
                const int32_t* __restrict__ hist_tab, const int32_t* __restrict__ hist_K, int hist_B, int B,
                double* __restrict__ logits64, float* __restrict__ logits32) {
  extern __shared__ __align__(1024) unsigned char sm[];
  __shared__ TcPlan P;
  __shared__ uint32_t tmem_base_s;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int r = (int)cg::this_cluster().block_rank();
  const int b0 = (blockIdx.x / kTcCtas) * kTcBatch;
  const int nb = min(kTcBatch, B - b0);
  const int son = g_tc_on;
  if (tid == 0) { P = *plan_g; tstamp(0, son); }
  uint64_t* full = reinterpret_cast<uint64_t*>(sm + kBarOff);
  uint64_t* empty = full + kTcSlots;
  uint64_t* xfull = empty + kTcSlots;
  uint64_t* dfull = xfull + 1;
  uint64_t* redfull = dfull + 1;
  uint64_t* progx = redfull + 1;     // cluster: every CTA finished the MMAs of stage s (X_s free)
  uint64_t* progr = progx + 1;       // cluster: every CTA finished reading its reduce buffer of s
  uint64_t* tfree = progr + 1;       // local: the epilogue finished reading TMEM of stage s
  const uint32_t xs = smem_u32(sm + kXOff);
  const uint32_t red_s = smem_u32(sm + kRedOff);
  __syncthreads();
  const int ns = P.n_stages;
  if (tid == 0) {
    for (int i = 0; i < kTcSlots; ++i) { mbar_init(&full[i], 1); mbar_init(&empty[i], 1); }
    mbar_init(xfull, 1);
    mbar_init(dfull, 1);
    mbar_init(redfull, 1);
    mbar_init(progx, kTcCtas);
    mbar_init(progr, kTcCtas);
    mbar_init(tfree, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    // arm stage 0's reduce buffer before any peer can send (its X is this CTA's own encode)
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
  if (tid == 0) tstamp(1, son);
  // ---- weight stream: fill the ring now (overlaps the feature layers) ----
  if (tid == 0) {
    for (int i = c0; i < c1 && i < c0 + kTcSlots; ++i) {
      const TcChunk ch = P.chunks[i];
      const int slot = (i - c0) % kTcSlots;
      mbar_expect_tx(&full[slot], (uint32_t)ch.bytes);
      tma_bulk_g2s(sm + slot * kTcSlotBytes, P.blob + ch.off, (uint32_t)ch.bytes, &full[slot]);
    }
  }
  // ---- stage 0 input: the encoded feature vectors (R3) of the 64 samples, K-slice ks of this
  //      CTA, written straight into the local X buffer as TF32 hi / lo (zero past F / nb) ----
  {
    const TcStage& S0 = P.st[0];
    const Job J0 = jobs_of(S0, r);
    if (J0.n) {
      // history prefix sums in scratch (R3: history ids index the concatenated group table)
      int* pre = reinterpret_cast<int*>(sm + kScratchOff);
      const int use_hist = (!feat && hist && hist_B > 0) ? 1 : 0;
      if (use_hist && tid == 0) {
        int acc = 0;
        for (int b = 0; b < hist_B && b < 2047; ++b) { pre[b] = acc; acc += hist_K[b]; }
        pre[2047] = acc;
      }
      __syncthreads();
      const int hl = use_hist ? pre[2047] : 0;
      const int xh0 = 3 + a.D_s + 10 * a.S_max;
      const uint32_t lo_off = (uint32_t)S0.ksl * (kTcBatch * 4);
      for (int i = tid; i < kTcBatch * S0.ksl; i += kThreads) {
        const int n = i / S0.ksl, kl = i - n * S0.ksl, k = J0.ks * S0.ksl + kl;
        const int b = b0 + n;
        float v = 0.f;
        if (n < nb && k < a.F) {
          if (feat) {
            v = feat[(int64_t)b * a.F + k];
          } else if (k >= xh0 && k < xh0 + 10 * a.h) {
            // x_h by binary search over the history prefix sums (instead of a linear walk)
            if (use_hist) {
              const int kk = (k - xh0) / 10, el = (k - xh0) % 10;
              const int gid = hist[(int64_t)b * a.h + kk];
              const int idx = gid >= 0 ? gid : hl + gid;
              if (idx >= 0 && idx < hl) {
                int lo = 0, hi = min(hist_B, 2047) - 1;
                while (lo < hi) { const int mid = (lo + hi + 1) >> 1; if (pre[mid] <= idx) lo = mid; else hi = mid - 1; }
                v = scale_elem<float>(el, hist_tab[((int64_t)lo * a.K_max + (idx - pre[lo])) * 10 + el]);
              }
            }
          } else {
            v = encode_elem(a, desc + (int64_t)b * a.D_s, nullptr, hist_tab, hist_K, 0, 0, k);
          }
        }
        const uint32_t h = tf32_rna(v);
        const uint32_t l = tf32_rna(v - __uint_as_float(h));
        *reinterpret_cast<uint32_t*>(sm + kXOff + xoff(n, kl, S0.ksl)) = h;
        *reinterpret_cast<uint32_t*>(sm + kXOff + lo_off + xoff(n, kl, S0.ksl)) = l;
      }
    }
    __syncthreads();
    if (tid == 0) mbar_arrive_local(xfull);      // stage 0 input complete (local writes)
  }
  if (tid == 128) tstamp(2, son);
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
      tstamp(3 + s, son);
      if (J.n == 0) { mbar_arrive_local(dfull); continue; }
      if (s > 0) mbar_wait(tfree, (s - 1) & 1);       // accumulator of stage s-1 read
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
            const uint64_t x_hi = sdesc(xs + (uint32_t)(kk >> 2) * 128u, 128u, (uint32_t)S.ksl * 32u);
            const uint64_t x_lo = sdesc(xlo + (uint32_t)(kk >> 2) * 128u, 128u, (uint32_t)S.ksl * 32u);
            // 3xTF32: small terms first, then the dominant hi x hi
            mma_tf32(d, a_lo, x_hi, (k0 > 0 || j > 0) ? 1u : 0u);
            mma_tf32(d, a_hi, x_lo, 1u);
            mma_tf32(d, a_hi, x_hi, 1u);
          }
          mma_commit(&empty[slot]);
          k0 += ch.kc;
          ++q;
        }
      }
      mma_commit(dfull);
    }
  } else if (warp >= 4) {
    // epilogue: thread e <-> TMEM lane e = output row e of the tile. The partial tile leaves
    // straight from registers; owners reduce and push each activation as soon as it is ready.
    const int e = tid - 128;
    const uint32_t lane_base = (uint32_t)((warp & 3) * 32) << 16;
    const double slope = pdev->slope;
    const float fslope = (float)slope;
    const float* rd = reinterpret_cast<const float*>(sm + kRedOff);
    const int ql = lane & ~3;
    int red_ph = 0;
    for (int s = 0; s < ns; ++s) {
      const TcStage S = P.st[s];
      const bool last = (s == ns - 1);
      const Job J = jobs_of(S, r);
      const bool owner = S.n_ks > 1 && r < S.n_m * S.n_ks;
      const int w = kTcBatch / S.n_ks;
      mbar_wait(dfull, s & 1);
      tc_fence_after();
      if (e == 0) tstamp(11 + s, son);
      const TcStage N = P.st[last ? s : s + 1];
      float vals[kTcBatch];
      if (J.n) {
        if (S.n_ks > 1) {
          tmem_ld64(tmem + lane_base, vals);
        } else {
          for (int jj = 0; jj < J.n; ++jj) {
            tmem_ld64(tmem + lane_base + (uint32_t)(jj * kTcBatch), vals);
            const int R = J.m[jj] * 128 + e;
            if (last && R < S.n_out) {
              const double bv = (double)__ldg(S.bias + R);
#pragma unroll 1
              for (int n = 0; n < nb; ++n) {
                const double v = (double)vals[n] + bv;
                logits64[(int64_t)(b0 + n) * S.n_out + R] = v;
                if (logits32) logits32[(int64_t)(b0 + n) * S.n_out + R] = (float)v;
              }
            }
          }
        }
      }
      // the accumulator is read: the next stage's MMAs may start; X_s is free (MMAs done)
      tc_fence_before();
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (!last && e == 0) {
        mbar_expect_tx(xfull, x_bytes(N, r));           // before any peer can pass progx(s)
        mbar_arrive_local(tfree);
      }
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (!last && e < kTcCtas) mbar_arrive_remote(mapa_u32(smem_u32(progx), e));
      if (J.n && S.n_ks > 1) {
        // reduce-scatter: columns [q w, (q+1) w) of the partial tile to owner m * n_ks + q, as
        // 16-byte st.async from registers (owner's reduce buffer: [ks][c][row]); its reduce
        // buffer of the previous stage must be read (progr(s-1))
        if (s > 0) mbar_wait_cluster(progr, (s - 1) & 1);
#pragma unroll
        for (int c = 0; c < kTcBatch; c += 4) {
          const int qq = c / w, cc = c - qq * w;
          const int owner_c = J.m[0] * S.n_ks + qq;
          const uint32_t dst = mapa_u32(red_s + (uint32_t)(((J.ks * (w / 4) + cc / 4) * 128 + e) * 16), owner_c);
          st_async_v4b32(dst, vals[c], vals[c + 1], vals[c + 2], vals[c + 3], mapa_u32(smem_u32(redfull), owner_c));
        }
      }
      if (owner) {
        const int m = r / S.n_ks, qo = r % S.n_ks;
        const int R = m * 128 + e, R0 = m * 128 + (e & ~3);
        if (e == 0 && s == 1) tstamp(28, son);
        mbar_wait_cluster(redfull, red_ph & 1);
        if (e == 0 && s == 1) tstamp(29, son);
        ++red_ph;
        const float bv = R < S.n_out ? __ldg(S.bias + R) : 0.f;
        const int nsl = N.ksl;                          // K-slice of the next stage
        const int kr = R - m * 128, jq = kr / nsl, kq = (kr & ~3) - jq * nsl;   // quad's slice / first k
        const int li = lane & 3;
#pragma unroll 1
        for (int cg = 0; cg < w / 4; ++cg) {
          float4 acc4 = make_float4(0.f, 0.f, 0.f, 0.f);
          double a64[4] = {(double)bv, (double)bv, (double)bv, (double)bv};
          for (int k2 = 0; k2 < S.n_ks; ++k2) {
            const float4 p4 = *reinterpret_cast<const float4*>(rd + ((k2 * (w / 4) + cg) * 128 + e) * 4);
            if (last) { a64[0] += p4.x; a64[1] += p4.y; a64[2] += p4.z; a64[3] += p4.w; }
            else { acc4.x += p4.x; acc4.y += p4.y; acc4.z += p4.z; acc4.w += p4.w; }
          }
          if (last) {
            // logits: the partials combined in fp64
#pragma unroll
            for (int i = 0; i < 4; ++i) {
              const int n = qo * w + cg * 4 + i;
              if (R < S.n_out && n < nb) {
                logits64[(int64_t)(b0 + n) * S.n_out + R] = a64[i];
                if (logits32) logits32[(int64_t)(b0 + n) * S.n_out + R] = (float)a64[i];
              }
            }
            continue;
          }
          // fp32 (R14: an fp32-accumulating path): bias, LeakyReLU, TF32 hi / lo
          float v[4] = {acc4.x + bv, acc4.y + bv, acc4.z + bv, acc4.w + bv};
          uint32_t h[4], l[4];
#pragma unroll
          for (int i = 0; i < 4; ++i) {
            if (S.act) v[i] = v[i] > 0.f ? v[i] : fslope * v[i];
            h[i] = tf32_rna(v[i]);
            l[i] = tf32_rna(v[i] - __uint_as_float(h[i]));
          }
          // 4x4 transpose inside the quad: lane li gets sample cg*4+li of the quad's four rows
          uint32_t th[4], tl[4];
#pragma unroll
          for (int j = 0; j < 4; ++j) {
            const int snd = (li - j) & 3, src = (li + j) & 3;
            const uint32_t sh = snd == 0 ? h[0] : snd == 1 ? h[1] : snd == 2 ? h[2] : h[3];
            const uint32_t sl = snd == 0 ? l[0] : snd == 1 ? l[1] : snd == 2 ? l[2] : l[3];
            const uint32_t rh = __shfl_sync(0xffffffffu, sh, (lane & ~3) + src);
            const uint32_t rl = __shfl_sync(0xffffffffu, sl, (lane & ~3) + src);
            th[src] = rh;   // row (quad base + src)
            tl[src] = rl;
          }
          // staging: [slice j of the next stage][hi, lo][c/8][k/4][c%8][k%4] (k = row within the
          // slice); each (slice, part) block is contiguous in the consumers' X layout
          if (R - (e & 3) < S.n_out) {
            const int c = cg * 4 + li;
            const uint32_t blk = (uint32_t)((jq * 2) * w * nsl * 4);
            const uint32_t o = (uint32_t)((c >> 3) * (nsl * 32) + (kq >> 2) * 128 + (c & 7) * 16);
            *reinterpret_cast<uint4*>(sm + kStgOff + blk + o) = make_uint4(th[0], th[1], th[2], th[3]);
            *reinterpret_cast<uint4*>(sm + kStgOff + blk + (uint32_t)(w * nsl * 4) + o) = make_uint4(tl[0], tl[1], tl[2], tl[3]);
          }
        }
        if (!last) {
          // one bulk copy per (next-stage K-slice j, part, consumer) into the consumer's X at
          // samples [qo w, qo w + w), once the consumers' MMAs of this stage are done (progx)
          asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
          asm volatile("bar.sync 1, 128;" ::: "memory");
          mbar_wait_cluster(progx, s & 1);
          const int nj = (min(S.n_out - m * 128, 128) + nsl - 1) / nsl;
          const bool grid = N.n_m * N.n_ks <= kTcCtas;
          const int ncons = grid ? N.n_m : min(N.n_m, kTcCtas);
          const uint32_t bytes = (uint32_t)(w * nsl * 4);
          for (int t = e; t < nj * 2 * ncons; t += 128) {
            const int j = t / (2 * ncons), part = (t / ncons) & 1, ci = t % ncons;
            const int ks2 = (m * 128) / nsl + j;         // the slice's index in the next stage
            const int cons = grid ? ci * N.n_ks + ks2 : ci;
            const uint32_t src = smem_u32(sm + kStgOff) + (uint32_t)((j * 2 + part) * w * nsl * 4);
            const uint32_t dst = xs + (uint32_t)part * (uint32_t)(nsl * kTcBatch * 4) + (uint32_t)(qo * w / 8) * (uint32_t)(nsl * 32);
            asm volatile(
                "cp.async.bulk.shared::cluster.shared::cta.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    mapa_u32(dst, cons)),
                "r"(src), "r"(bytes), "r"(mapa_u32(smem_u32(xfull), cons))
                : "memory");
          }
        }
        if (s == 1 && (e == 0 || e == 96)) tstamp(e == 0 ? 31 : 26, son);
      }
      if (last) break;
      // reduce buffer of stage s read: arm stage s+1's, then let peers send their partials
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (e == 0 && N.n_ks > 1 && r < N.n_m * N.n_ks) mbar_expect_tx(redfull, (uint32_t)kRedBytes);
      asm volatile("bar.sync 1, 128;" ::: "memory");
      if (e == 0 && s == 1) tstamp(30, son);
      if (e < kTcCtas) mbar_arrive_remote(mapa_u32(smem_u32(progr), e));
      if (e == 0) tstamp(19 + s, son);
    }
  }
  if (tid == 128) tstamp(27, son);
  tc_fence_before();
  __syncthreads();
  cg::this_cluster().sync();       // no CTA leaves while a peer may still address its memory
  if (warp == 2) {
    tc_fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 128;" ::"r"(tmem));
  }
}

cudaError_t tc_debug_stamps(int on, unsigned long long* out) {
  cudaError_t e = cudaMemcpyToSymbol(g_tc_on, &on, sizeof(int));
  if (e == cudaSuccess && out) e = cudaMemcpyFromSymbol(out, g_tc_stamp, sizeof(unsigned long long) * 32);
  return e;
}

cudaError_t launch_pilot_tc(const ArchDev& a, const PilotDev* p_dev, const TcPlan* plan_dev, const float* feat,
                            const int64_t* desc, const int32_t* hist, const int32_t* hist_tab, const int32_t* hist_K,
                            int hist_B, int B, double* logits64, float* logits32, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  static uint64_t attr_done = 0;   // bit d: set on device d
  const uint64_t bit = 1ull << current_device();
  if (!(attr_done & bit)) {
    cudaError_t e = cudaFuncSetAttribute(pilot_tc_kernel, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(pilot_tc_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kSmemBytes);
    if (e != cudaSuccess) return e;
    attr_done |= bit;
  }
  const int n_clusters = (B + kTcBatch - 1) / kTcBatch;
  pilot_tc_kernel<<<n_clusters * kTcCtas, kThreads, kSmemBytes, s>>>(a, p_dev, plan_dev, feat, desc, hist, hist_tab,
                                                                    hist_K, hist_B, B, logits64, logits32);
  return cudaGetLastError();
}

}  // namespace dyo
