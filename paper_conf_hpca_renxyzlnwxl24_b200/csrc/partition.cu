// Partition labels (§IV-D, §V L203-L205 partition simulator, §VI-G;
// DESIGN.md reading R18): the execution trace of one sample (a resolved path) cut into K blocks
// that minimise the exposed migration time under the capacity H - the Sentinel-style labels the
// pilot is trained on - and the three even-split heuristics of L275.
//
//   block_tables_kernel  one warp per block start s: rows s..L-1 streamed in order, the block's
//                        tensor set kept in a shared-memory hash (first access decides read-first),
//                        need / fetch / comp of every [s, e) written as it grows
//   suffix_dp_kernel     one launch per block index j (K-2 .. 0), one thread per (s, e):
//                        f[j][s][e] = min over e' of max(0, xfer(fetch(e,e')) - comp(s,e))
//                                     + f[j+1][e][e']          (need(e, e') <= H)
//   finish_kernel        one thread: OPT and the lexicographically smallest optimal cuts, front
//                        to back (exact integer equality), or a heuristic's cuts and exposure
// Everything is integer (ns, bytes), so results equal oracle/partition.py exactly.
#include <cuda_runtime.h>
#include <cstdint>

#include "dyo_internal.h"

namespace dyo {

constexpr int kPartHash = 8192;                 // distinct tensors of one block start (smem hash)
constexpr long long kPartInf = 0x3fffffffffffffffll;

__device__ __forceinline__ long long xfer_ns(long long bytes, long long bw) { return (bytes * 1000 + bw - 1) / bw; }

__global__ void __launch_bounds__(32)
block_tables_kernel(ArchDev a, const int32_t* __restrict__ ops, const int32_t* __restrict__ its, int L, int b,
                    const long long* __restrict__ op_ns, long long* need, long long* fetch, long long* comp,
                    int* overflow) {
  __shared__ int key[kPartHash];
  const int s = blockIdx.x, lane = threadIdx.x;
  const int64_t stride = L + 1;
  for (int i = lane; i < kPartHash; i += 32) key[i] = -1;
  __syncwarp();
  long long nd = 0, ft = 0, cp = 0;
  int used = 0;
  for (int r = s; r < L; ++r) {
    const int op = ops[r];
    if (op >= 0) {
      cp += op_ns[op];
      const int q0 = a.acc_ptr[op], q1 = a.acc_ptr[op + 1];
      long long dn = 0, df = 0;
      for (int q = q0 + lane; q < q1; q += 32) {
        const int t = a.acc_t[q] + a.acc_s[q] * its[r] + a.acc_sb[q] * b;
        uint32_t h = ((uint32_t)t * 2654435761u) & (kPartHash - 1);
        bool fresh = false;
        while (true) {
          const int k = atomicCAS(&key[h], -1, t);
          if (k == -1) { fresh = true; break; }
          if (k == t) break;
          h = (h + 1) & (kPartHash - 1);
        }
        if (fresh) {
          dn += a.t_abytes[t];
          if (a.acc_m[q] & 1) df += a.t_bytes[t];
        }
        used += fresh;
      }
#pragma unroll
      for (int o = 16; o > 0; o >>= 1) {
        dn += __shfl_xor_sync(0xffffffffu, dn, o);
        df += __shfl_xor_sync(0xffffffffu, df, o);
      }
      nd += dn;
      ft += df;
      __syncwarp();
    }
    if (lane == 0) {
      need[(int64_t)s * stride + r + 1] = nd;
      fetch[(int64_t)s * stride + r + 1] = ft;
      comp[(int64_t)s * stride + r + 1] = cp;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) used += __shfl_xor_sync(0xffffffffu, used, o);
  if (lane == 0 && used > kPartHash / 2) atomicExch(overflow, 1);
}

// f layer j from layer j+1; fj1 == nullptr initialises the last block (j = K-1)
__global__ void suffix_dp_kernel(int L, const long long* __restrict__ need, const long long* __restrict__ fetch,
                                 const long long* __restrict__ comp, long long H, long long bw,
                                 const long long* __restrict__ fj1, long long* __restrict__ fj) {
  const int64_t stride = L + 1;
  const int64_t n = (int64_t)L * stride;
  for (int64_t idx = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; idx < n; idx += (int64_t)gridDim.x * blockDim.x) {
    const int s = (int)(idx / stride), e = (int)(idx % stride);
    long long best = kPartInf;
    if (e > s) {
      if (!fj1) {
        if (e == L && need[(int64_t)s * stride + L] <= H) best = 0;
      } else if (e < L) {
        const long long ce = comp[(int64_t)s * stride + e];
        for (int e2 = e + 1; e2 <= L; ++e2) {
          const long long f = fj1[(int64_t)e * stride + e2];
          if (f >= kPartInf || need[(int64_t)e * stride + e2] > H) continue;
          const long long x = xfer_ns(fetch[(int64_t)e * stride + e2], bw) - ce;
          const long long v = (x > 0 ? x : 0) + f;
          if (v < best) best = v;
        }
      }
    }
    fj[idx] = best;
  }
}

// method 0: OPT + lexicographically smallest optimal cuts from f; 1..3: the even heuristics
// (weights: operator rows, compute ns, accessed tensor bytes) and their exposure
__global__ void finish_kernel(ArchDev a, const int32_t* __restrict__ ops, const int32_t* __restrict__ its, int L, int b,
                              const long long* __restrict__ op_ns, const long long* __restrict__ need,
                              const long long* __restrict__ fetch, const long long* __restrict__ comp, long long H,
                              long long bw, const long long* __restrict__ f, int K, int method, int32_t* cuts,
                              long long* result) {
  if (threadIdx.x != 0 || blockIdx.x != 0) return;
  const int64_t stride = L + 1, lay = (int64_t)L * stride;
  if (method == 0) {
    long long opt = kPartInf;
    int c1 = -1;
    for (int c = 1; c <= L; ++c)
      if (need[c] <= H && f[c] < opt) { opt = f[c]; c1 = c; }
    if (c1 < 0) { result[0] = -1; return; }
    cuts[0] = 0;
    cuts[1] = c1;
    long long rem = opt;
    for (int j = 1; j < K; ++j) {
      const int s = cuts[j - 1], e = cuts[j];
      for (int e2 = e + 1; e2 <= L; ++e2) {
        const long long fv = f[(int64_t)j * lay + (int64_t)e * stride + e2];
        if (need[(int64_t)e * stride + e2] > H || fv >= kPartInf) continue;
        const long long x = xfer_ns(fetch[(int64_t)e * stride + e2], bw) - comp[(int64_t)s * stride + e];
        const long long st = x > 0 ? x : 0;
        if (st + fv == rem) { cuts[j + 1] = e2; rem -= st; break; }
      }
    }
    result[0] = opt;
    return;
  }
  // heuristics: prefix weights, cut j = clamp(max p with W(p) K <= W(L) j, c_{j-1} + 1, L - (K - j))
  long long tot = 0;
  for (int r = 0; r < L; ++r) {
    const int op = ops[r];
    long long w = 0;
    if (op >= 0) {
      if (method == 1) w = 1;
      else if (method == 2) w = op_ns[op];
      else
        for (int q = a.acc_ptr[op]; q < a.acc_ptr[op + 1]; ++q) w += a.t_bytes[a.acc_t[q] + a.acc_s[q] * its[r] + a.acc_sb[q] * b];
    }
    tot += w;
  }
  cuts[0] = 0;
  for (int j = 1; j < K; ++j) {
    long long pre = 0;
    int p = 0;
    for (int r = 0; r < L; ++r) {
      const int op = ops[r];
      long long w = 0;
      if (op >= 0) {
        if (method == 1) w = 1;
        else if (method == 2) w = op_ns[op];
        else
          for (int q = a.acc_ptr[op]; q < a.acc_ptr[op + 1]; ++q) w += a.t_bytes[a.acc_t[q] + a.acc_s[q] * its[r] + a.acc_sb[q] * b];
      }
      pre += w;
      if (pre * K <= tot * j) p = r + 1;
    }
    int c = p < L - (K - j) ? p : L - (K - j);
    if (c < cuts[j - 1] + 1) c = cuts[j - 1] + 1;
    cuts[j] = c;
  }
  cuts[K] = L;
  long long ex = 0;
  bool ok = true;
  for (int j = 0; j < K; ++j) ok = ok && need[(int64_t)cuts[j] * stride + cuts[j + 1]] <= H;
  for (int j = 1; j < K; ++j) {
    const long long x = xfer_ns(fetch[(int64_t)cuts[j] * stride + cuts[j + 1]], bw) - comp[(int64_t)cuts[j - 1] * stride + cuts[j]];
    ex += x > 0 ? x : 0;
  }
  result[0] = ex;
  result[1] = ok ? 1 : 0;
}

cudaError_t launch_partition(const ArchDev& a, const int32_t* ops, const int32_t* its, int L, int b,
                             const long long* op_ns, int K, int method, long long H, long long bw, long long* need,
                             long long* fetch, long long* comp, long long* f, int32_t* cuts, long long* result,
                             int* overflow, cudaStream_t s) {
  block_tables_kernel<<<L, 32, 0, s>>>(a, ops, its, L, b, op_ns, need, fetch, comp, overflow);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return e;
  const int64_t lay = (int64_t)L * (L + 1);
  if (method == 0) {
    const int grid = (int)((lay + 255) / 256 < 4096 ? (lay + 255) / 256 : 4096);
    for (int j = K - 1; j >= 0; --j) {
      suffix_dp_kernel<<<grid, 256, 0, s>>>(L, need, fetch, comp, H, bw, j == K - 1 ? nullptr : f + (j + 1) * lay, f + j * lay);
      if ((e = cudaGetLastError()) != cudaSuccess) return e;
    }
  }
  finish_kernel<<<1, 1, 0, s>>>(a, ops, its, L, b, op_ns, need, fetch, comp, H, bw, f, K, method, cuts, result);
  return cudaGetLastError();
}

}  // namespace dyo
