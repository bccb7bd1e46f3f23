// Device helpers shared by the pilot kernels (pilot.cu: K1 cluster GEMV path; pilot_tc.cu:
// K1-TC tensor-core batch path): feature encode (R3), mbarrier / TMA bulk copy / cluster
// st.async PTX wrappers.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "dyo_internal.h"

namespace dyo {

template <class T>
__device__ __forceinline__ T scale_elem(int e, int v) {
  // R3: counts and idiom sums x 2^-4, dimension sums x 2^-10 (exact in fp32: v < 2^24)
  return (T)((float)v * (e < 7 ? 0.0625f : 0.0009765625f));
}

// Feature vector of one sample into x[0..F) (R3). Threads of the block cooperate.
// History table (R3): the executed block vectors of the previous dyo_pilot_predict, stored per
// prediction at [b * K_max + g] with K[b] groups each; history ids index their concatenation
// in sample order (>= 0 from the start, < 0 from the end).
// Feature i of one sample (R3); hl = total groups in the history table (sum of hist_K).
__device__ __forceinline__ float encode_elem(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                                             const int32_t* hist_tab, const int32_t* hist_K, int hist_B, int hl,
                                             int i) {
  const int xs0 = 3, xa0 = 3 + a.D_s, xh0 = xa0 + 10 * a.S_max, end = xh0 + 10 * a.h;
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
      const int gid = hist[k];
      int idx = gid >= 0 ? gid : hl + gid;
      if (idx >= 0 && idx < hl) {
        int b = 0;
        while (idx >= hist_K[b]) { idx -= hist_K[b]; ++b; }
        v = scale_elem<float>(e, hist_tab[((int64_t)b * a.K_max + idx) * 10 + e]);
      }
    }
  }
  return v;
}

__device__ __forceinline__ int hist_len(const int32_t* hist_K, int hist_B) {
  int hl = 0;
  for (int b = 0; b < hist_B; ++b) hl += hist_K[b];
  return hl;
}

template <class T>
__device__ void encode_one(const ArchDev& a, const int64_t* desc, const int32_t* hist,
                           const int32_t* hist_tab, const int32_t* hist_K, int hist_B, T* x) {
  const int hl = (hist && hist_B > 0) ? hist_len(hist_K, hist_B) : 0;
  for (int i = threadIdx.x; i < a.F; i += blockDim.x)
    x[i] = (T)encode_elem(a, desc, hist, hist_tab, hist_K, hist_B, hl, i);
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


__device__ __forceinline__ uint32_t mapa_u32(uint32_t saddr, int rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(saddr), "r"(rank));
  return r;
}
// 8 / 16-byte asynchronous remote stores that signal the destination CTA's mbarrier
__device__ __forceinline__ void st_async_b64(uint32_t raddr, double v, uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.b64 [%0], %1, [%2];" ::"r"(raddr),
               "l"(__double_as_longlong(v)), "r"(rbar)
               : "memory");
}
__device__ __forceinline__ void st_async_v2b64(uint32_t raddr, double a, double b, uint32_t rbar) {
  asm volatile("st.async.shared::cluster.mbarrier::complete_tx::bytes.v2.b64 [%0], {%1, %2}, [%3];" ::"r"(raddr),
               "l"(__double_as_longlong(a)), "l"(__double_as_longlong(b)), "r"(rbar)
               : "memory");
}


}  // namespace dyo
