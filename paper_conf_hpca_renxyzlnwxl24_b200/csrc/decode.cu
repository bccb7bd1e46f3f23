// A3 decode (§IV-B; R2, R4, R6, R8), all on the device.
//
// decode_path_kernel (one CTA per prediction): block head -> rint'd slots (R4), branch head ->
//   argmax choice per site (tied sites replay, R6), the resolved path (R2) expanded in parallel
//   from the top-level pieces, the cut into groups at the cumulative counts, and the executed
//   block vector of each group (warp-reduced column sums).
// decode_sets_kernel (one CTA per group): the group's tensor accesses in order, deduplicated
//   by a shared-memory bitonic sort on (tensor, position), re-sorted by first position (R8).
// hist_compact_kernel: executed block vectors of all predictions, in order -> history table.
#include <cuda_runtime.h>
#include <cstdint>

#include "dyo_internal.h"

namespace dyo {

constexpr int kDecThreads = 256;
constexpr int kMaxPieces = 1024;
constexpr int kRecCap = 2048;      // access records per group before deduplication

__global__ void __launch_bounds__(kDecThreads)
decode_path_kernel(ArchDev a, const double* __restrict__ logits, PredDev pd) {
  const int b = blockIdx.x;
  const double* y = logits + (int64_t)b * a.O;
  __shared__ int s_start[kMaxPieces + 1];
  __shared__ int s_ngroups, s_L;
  int32_t* choices = pd.choices + (int64_t)b * a.n_sites;
  int32_t* slots = pd.slots + (int64_t)b * a.K_max * 10;

  // 1. block head -> slots (R4): n = rint(y * 2^sigma), clamped to [0, 2^24-1]
  for (int i = threadIdx.x; i < a.K_max * 10; i += blockDim.x) {
    const int e = i % 10;
    double t = y[i] * (e < 7 ? 16.0 : 1024.0);
    t = fmin(fmax(t, 0.0), (double)kSat);
    slots[i] = (int)rint(t);
  }
  // 2. branch head -> choices (argmax, lowest index on ties)
  for (int i = threadIdx.x; i < a.n_sites; i += blockDim.x) {
    const int off = a.site_logit[i];
    if (off >= 0) {
      int best = 0;
      double bv = y[off];
      for (int c = 1; c < a.site_nch[i]; ++c) {
        const double v = y[off + c];
        if (v > bv) { bv = v; best = c; }
      }
      choices[i] = best;
    }
  }
  __syncthreads();
  for (int i = threadIdx.x; i < a.n_sites; i += blockDim.x)
    if (a.site_logit[i] < 0) choices[i] = choices[a.site_tie[i]];
  __syncthreads();

  // 3. piece lengths and starts (serial: pieces are few), 4. counts of non-empty slots
  if (threadIdx.x == 0) {
    int c = 0;
    for (int p = 0; p < a.n_pieces; ++p) {
      s_start[p] = c;
      const int k = a.piece_kind[p];
      int len;
      if (k == 0) {
        len = a.piece_b[p];
      } else if (k == 1) {
        const int s = a.piece_a[p];
        len = 1 + a.arm_nops[a.site_arm_ptr[s] + choices[s]];
      } else {
        const int s = a.piece_a[p];
        const int n = a.site_lo[s] + choices[s];
        len = n * (1 + a.piece_c[p]) + 1;
      }
      c += len;
    }
    s_start[a.n_pieces] = c;
    s_L = c;
    pd.L[b] = c;
    // cut (R4): groups at cumulative counts of non-empty slots, clipped to the path
    const int L = c;
    int g = 0, C = 0;
    int32_t* grp = pd.grp + (int64_t)b * a.K_max * 2;
    for (int k = 0; k < a.K_max; ++k) {
      const int n = slots[k * 10];
      if (n == 0) continue;
      if (C >= L) break;
      grp[2 * g] = C;
      grp[2 * g + 1] = min(C + n, L);
      C += n;
      ++g;
    }
    if (g == 0 && L > 0) {
      grp[0] = 0;
      grp[1] = L;
      g = 1;
    }
    if (g > 0 && grp[2 * g - 1] < L) grp[2 * g - 1] = L;
    s_ngroups = g;
    pd.K[b] = g;
  }
  __syncthreads();
  const int L = s_L;
  if (L > a.L_max) {
    if (threadIdx.x == 0) { pd.status[0] = DYO_E_CAPACITY; pd.status[1] = L; }
    return;
  }
  // 5. path expansion (R2)
  int32_t* path = pd.path + (int64_t)b * a.L_max;
  for (int r = threadIdx.x; r < L; r += blockDim.x) {
    int lo = 0, hi = a.n_pieces - 1;
    while (lo < hi) {
      const int mid = (lo + hi + 1) >> 1;
      if (s_start[mid] <= r) lo = mid; else hi = mid - 1;
    }
    const int p = lo, q = r - s_start[p];
    const int k = a.piece_kind[p];
    int op;
    if (k == 0) {
      op = a.piece_a[p] + q;
    } else if (k == 1) {
      const int s = a.piece_a[p];
      op = q == 0 ? -1 : a.arm_first_op[a.site_arm_ptr[s] + choices[s]] + q - 1;
    } else {
      const int c = a.piece_c[p];
      const int w = q % (1 + c);
      op = w == 0 ? -1 : a.piece_b[p] + w - 1;
    }
    path[r] = op;
  }
  __syncthreads();
  // 6. executed block vectors: warp per group
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int32_t* grp = pd.grp + (int64_t)b * a.K_max * 2;
  int32_t* blocks = pd.blocks + (int64_t)b * a.K_max * 10;
  for (int g = warp; g < s_ngroups; g += blockDim.x >> 5) {
    const int s = grp[2 * g], e = grp[2 * g + 1];
    long long acc[9];
#pragma unroll
    for (int k = 0; k < 9; ++k) acc[k] = 0;
    for (int r = s + lane; r < e; r += 32) {
      const int op = path[r];
      if (op >= 0) {
#pragma unroll
        for (int k = 0; k < 9; ++k) acc[k] += a.op_sig[(int64_t)op * 9 + k];
      }
    }
#pragma unroll
    for (int k = 0; k < 9; ++k)
      for (int o = 16; o > 0; o >>= 1) acc[k] += __shfl_xor_sync(0xffffffffu, acc[k], o);
    if (lane == 0) {
      blocks[g * 10] = min(e - s, kSat);
#pragma unroll
      for (int k = 0; k < 9; ++k) blocks[g * 10 + 1 + k] = (int)min(acc[k], (long long)kSat);
    }
  }
}

__device__ void bitonic_sort_u64(uint64_t* key, int n_pow2) {
  for (int k = 2; k <= n_pow2; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < n_pow2; i += blockDim.x) {
        const int ixj = i ^ j;
        if (ixj > i) {
          const uint64_t x = key[i], z = key[ixj];
          const bool up = (i & k) == 0;
          if ((x > z) == up) { key[i] = z; key[ixj] = x; }
        }
      }
      __syncthreads();
    }
  }
}

__global__ void __launch_bounds__(kDecThreads)
decode_sets_kernel(ArchDev a, PredDev pd) {
  const int b = blockIdx.x / a.K_max, g = blockIdx.x % a.K_max;
  __shared__ uint64_t key[kRecCap];
  __shared__ int s_rowcnt[kDecThreads + 1];
  __shared__ int s_n, s_u;
  int32_t* ent_n = pd.ent_n + (int64_t)b * a.K_max + g;
  if (g >= pd.K[b] || pd.status[0] != 0) {
    if (threadIdx.x == 0) *ent_n = 0;
    return;
  }
  const int32_t* grp = pd.grp + ((int64_t)b * a.K_max + g) * 2;
  const int s = grp[0], e = grp[1];
  const int32_t* path = pd.path + (int64_t)b * a.L_max;
  // each thread takes a contiguous chunk of rows; exclusive scan of their access counts
  const int nrows = e - s;
  const int chunk = (nrows + blockDim.x - 1) / blockDim.x;
  const int rs = s + threadIdx.x * chunk, re = min(e, rs + chunk);
  int cnt = 0;
  for (int r = rs; r < re; ++r) {
    const int op = path[r];
    if (op >= 0) cnt += a.acc_ptr[op + 1] - a.acc_ptr[op];
  }
  s_rowcnt[threadIdx.x] = cnt;
  __syncthreads();
  if (threadIdx.x == 0) {
    int c = 0;
    for (int i = 0; i < blockDim.x; ++i) { const int v = s_rowcnt[i]; s_rowcnt[i] = c; c += v; }
    s_n = c;
  }
  __syncthreads();
  const int n = s_n;
  if (n > kRecCap) {
    if (threadIdx.x == 0) { *ent_n = 0; atomicCAS(&pd.status[0], 0, DYO_E_CAPACITY); pd.status[1] = n; }
    return;
  }
  int pos = s_rowcnt[threadIdx.x];
  for (int r = rs; r < re; ++r) {
    const int op = path[r];
    if (op < 0) continue;
    for (int q = a.acc_ptr[op]; q < a.acc_ptr[op + 1]; ++q, ++pos)
      key[pos] = ((uint64_t)a.acc_t[q] << 32) | ((uint64_t)pos << 2) | (uint64_t)a.acc_m[q];
  }
  int np2 = 1;
  while (np2 < n) np2 <<= 1;
  for (int i = n + threadIdx.x; i < np2; i += blockDim.x) key[i] = ~0ull;
  __syncthreads();
  bitonic_sort_u64(key, np2);
  // runs of equal tensor: first record = first access; union of modes (R8)
  // results are written into the upper part of key[] by position order afterwards
  __shared__ uint64_t out_key[kRecCap];
  __shared__ int s_flag[kRecCap];
  for (int i = threadIdx.x; i < n; i += blockDim.x)
    s_flag[i] = (i == 0 || (key[i] >> 32) != (key[i - 1] >> 32)) ? 1 : 0;
  __syncthreads();
  for (int i = threadIdx.x; i < np2; i += blockDim.x) out_key[i] = ~0ull;
  __syncthreads();
  for (int i = threadIdx.x; i < n; i += blockDim.x) {
    if (!s_flag[i]) continue;
    const uint32_t t = (uint32_t)(key[i] >> 32);
    const uint32_t p0 = (uint32_t)(key[i] & 0xffffffffu) >> 2;
    const uint32_t m0 = (uint32_t)key[i] & 3u;
    uint32_t mu = m0;
    for (int k = i + 1; k < n && (uint32_t)(key[k] >> 32) == t; ++k) mu |= (uint32_t)key[k] & 3u;
    const uint32_t rd = m0 & 1u;
    // sort key by first position; payload tensor / mode / read-first
    out_key[i] = ((uint64_t)p0 << 32) | ((uint64_t)t << 3) | (mu << 1) | rd;
  }
  __syncthreads();
  bitonic_sort_u64(out_key, np2);
  if (threadIdx.x == 0) {
    int u = 0;
    while (u < n && out_key[u] != ~0ull) ++u;
    s_u = u;
  }
  __syncthreads();
  const int u = s_u;
  if (u > kEntCap) {
    if (threadIdx.x == 0) { *ent_n = 0; atomicCAS(&pd.status[0], 0, DYO_E_CAPACITY); pd.status[1] = u; }
    return;
  }
  int2* ent = pd.ent + ((int64_t)b * a.K_max + g) * kEntCap;
  for (int i = threadIdx.x; i < u; i += blockDim.x) {
    const uint32_t lo = (uint32_t)(out_key[i] & 0xffffffffu);
    ent[i] = make_int2((int)(lo >> 3), (int)(((lo >> 1) & 3u) | ((lo & 1u) << 2)));
  }
  if (threadIdx.x == 0) *ent_n = u;
}

__global__ void hist_compact_kernel(ArchDev a, PredDev pd, int B, int32_t* tab, int32_t* len) {
  __shared__ int s_off[65];
  if (threadIdx.x == 0) {
    int c = 0;
    for (int b = 0; b < B; ++b) { s_off[b] = c; c += pd.K[b]; }
    s_off[B] = c;
    *len = c;
  }
  __syncthreads();
  for (int b = 0; b < B; ++b) {
    const int K = pd.K[b];
    for (int i = threadIdx.x; i < K * 10; i += blockDim.x)
      tab[(int64_t)(s_off[b]) * 10 + i] = pd.blocks[(int64_t)b * a.K_max * 10 + i];
  }
}

cudaError_t launch_decode(const ArchDev& a, const double* logits, PredDev& pd, int B,
                          int32_t* hist_tab_out, int32_t* hist_len_out, cudaStream_t s) {
  if (B <= 0) return cudaSuccess;
  cudaMemsetAsync(pd.status, 0, 2 * sizeof(int32_t), s);
  decode_path_kernel<<<B, kDecThreads, 0, s>>>(a, logits, pd);
  decode_sets_kernel<<<B * a.K_max, kDecThreads, 0, s>>>(a, pd);
  hist_compact_kernel<<<1, 256, 0, s>>>(a, pd, B, hist_tab_out, hist_len_out);
  return cudaGetLastError();
}

}  // namespace dyo
