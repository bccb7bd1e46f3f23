// Device-side decode of one prediction (§IV-B; R2, R4, R6, R8).
// Shared by the fused pilot kernel's epilogue (pilot.cu) and the stand-alone decode kernel
// (decode.cu, used when a batch has more groups than the pilot cluster has CTAs).
//
//   head_decode_warp  one warp, no block barriers: block head -> non-empty counts (ballot
//                     compaction), branch head -> argmax choices (tied sites replay), piece
//                     lengths -> warp scan -> piece starts (the resolved path is never stored),
//                     counts -> warp scan -> group starts, K.
//   build_group       group g: its rows' operators (binary search over the piece starts),
//                     executed block vector and tensor set W_g (R8): access records
//                     keyed (tensor, position) -> sort -> first record per tensor + mode union
//                     -> sort by first position. <= 64 records: one warp, registers + shuffles;
//                     more: the whole block with shared-memory bitonic sorts.
#pragma once
#include <cuda_runtime.h>
#include <cstdint>

#include "dyo_device.cuh"
#include "dyo_internal.h"

namespace dyo {

constexpr int kMaxPieces = 1024;
constexpr int kRecCap = 2048;          // access records per group before deduplication

struct DecHead {
  int start[kMaxPieces + 1];           // piece start rows; start[n_pieces] = L
  int cum[256 + 1];                    // start row of each group
  int cntc[256];                       // non-empty counts in slot order
  int choice[kMaxSites];
  int L, nk, K;
};

struct DecGroup {
  uint64_t key[kRecCap];
  uint64_t key2[kRecCap];
  int warp_tmp[32];
  long long sum_tmp[32];
  unsigned long long sig[9];
  int n, u;
};

// Copy the small decode tables (sites, arms, pieces) into shared memory `buf` (int32 words,
// capacity cap) and return an ArchDev whose pointers refer to the copies; tables that do not
// fit stay in global memory. All threads of the block call it; ends with __syncthreads().
__device__ __forceinline__ ArchDev stage_decode_tables(const ArchDev& a, int* buf, int cap) {
  const int n_arms = a.n_arms;
  ArchDev s = a;
  int off = 0;
  auto take = [&](const int32_t* src, int n) -> const int32_t* {
    if (off + n > cap) return src;
    int* dst = buf + off;
    for (int i = threadIdx.x; i < n; i += blockDim.x) dst[i] = src[i];
    off += n;
    return dst;
  };
  s.site_logit = take(a.site_logit, a.n_sites);
  s.site_nch = take(a.site_nch, a.n_sites);
  s.site_tie = take(a.site_tie, a.n_sites);
  s.site_lo = take(a.site_lo, a.n_sites);
  s.site_arm_ptr = take(a.site_arm_ptr, a.n_sites);
  s.site_rev = take(a.site_rev, a.n_sites);
  s.piece_kind = take(a.piece_kind, a.n_pieces);
  s.piece_a = take(a.piece_a, a.n_pieces);
  s.piece_b = take(a.piece_b, a.n_pieces);
  s.piece_c = take(a.piece_c, a.n_pieces);
  s.arm_nops = take(a.arm_nops, n_arms);
  s.arm_first_op = take(a.arm_first_op, n_arms);
  __syncthreads();
  return s;
}

__device__ __forceinline__ int warp_incl_scan(int v, int lane) {
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, v, o);
    if (lane >= o) v += y;
  }
  return v;
}

// Decode the head of logits y (fp64, R4) into H. Called by ONE warp; __syncwarp() at the end.
// b = index of the prediction in its batch (selects the host traversal's choices when the
// arch has no branch head).
static __device__ void head_decode_warp(const ArchDev& a, const double* __restrict__ y, DecHead& H, int lane, int b) {
  // 1. block-head counts of every slot; compact the non-empty ones in slot order
  int nk = 0;
  for (int k0 = 0; k0 < a.K_max; k0 += 32) {
    const int k = k0 + lane;
    int n = 0;
    if (k < a.K_max) {
      double t = y[10 * k] * 16.0;
      t = fmin(fmax(t, 0.0), (double)kSat);
      n = (int)rint(t);
    }
    const unsigned m = __ballot_sync(0xffffffffu, n != 0);
    if (n != 0) H.cntc[nk + __popc(m & ((1u << lane) - 1))] = n;
    nk += __popc(m);
  }
  // 2. branch head: argmax per free site (lowest index on ties), then tied sites; without a
  //    branch head the choices are the host traversal's
  if (a.forced) {
    for (int i = lane; i < a.n_sites; i += 32) H.choice[i] = a.forced[(int64_t)b * a.n_sites + i];
  }
  for (int i = lane; i < a.n_sites && !a.forced; i += 32) {
    const int off = a.site_logit[i];
    if (off >= 0) {
      int best = 0;
      double bv = y[off];
      const int nch = a.site_nch[i];
      for (int c = 1; c < nch; ++c) {
        const double v = y[off + c];
        if (v > bv) { bv = v; best = c; }
      }
      H.choice[i] = best;
    }
  }
  __syncwarp();
  for (int i = lane; i < a.n_sites && !a.forced; i += 32)
    if (a.site_logit[i] < 0) H.choice[i] = H.choice[a.site_tie[i]];   // tie targets are free sites
  __syncwarp();
  // 3. piece lengths -> exclusive scan -> piece starts (R2)
  int carry = 0;
  for (int p0 = 0; p0 < a.n_pieces; p0 += 32) {
    const int p = p0 + lane;
    int len = 0;
    if (p < a.n_pieces) {
      const int k = a.piece_kind[p];
      if (k == 0) {
        len = a.piece_b[p];
      } else if (k == 1) {
        const int s = a.piece_a[p];
        len = 1 + a.arm_nops[a.site_arm_ptr[s] + H.choice[s]];
      } else {
        const int s = a.piece_a[p];
        len = (a.site_lo[s] + H.choice[s]) * (1 + a.piece_c[p]) + 1;
      }
    }
    const int inc = warp_incl_scan(len, lane);
    if (p < a.n_pieces) H.start[p] = carry + inc - len;
    carry += __shfl_sync(0xffffffffu, inc, 31);
  }
  const int L = carry;
  // 4. cut (R4): group starts = exclusive scan of the compacted counts; K = groups inside the path
  __syncwarp();
  int c2 = 0, K = 0;
  for (int k0 = 0; k0 < nk; k0 += 32) {
    const int k = k0 + lane;
    const int v = k < nk ? H.cntc[k] : 0;
    const int inc = warp_incl_scan(v, lane);
    const int st = c2 + inc - v;
    if (k < nk) H.cum[k] = st;
    K += __popc(__ballot_sync(0xffffffffu, k < nk && st < L));
    c2 += __shfl_sync(0xffffffffu, inc, 31);
  }
  if (nk == 0 && L > 0) K = 1;
  if (lane == 0) {
    H.start[a.n_pieces] = L;
    H.L = L;
    H.nk = nk;
    H.K = K;
  }
  __syncwarp();
}

__device__ __forceinline__ int group_start(const DecHead& H, int g) { return H.nk == 0 ? 0 : H.cum[g]; }
__device__ __forceinline__ int group_end(const DecHead& H, int g) {
  if (H.nk == 0 || g == H.K - 1) return H.L;                    // last group absorbs the remainder
  return min(H.cum[g] + H.cntc[g], H.L);
}

// Operator of path row r (-1 for a control row); *it = iteration index of its loop for the
// per-iteration tensors (R13; 0 outside loops, counted down in a reversed loop).
__device__ __forceinline__ int row_op(const ArchDev& a, const DecHead& H, int r, int* it = nullptr) {
  int lo = 0, hi = a.n_pieces - 1;
  while (lo < hi) {
    const int mid = (lo + hi + 1) >> 1;
    if (H.start[mid] <= r) lo = mid; else hi = mid - 1;
  }
  const int p = lo, q = r - H.start[p];
  const int k = a.piece_kind[p];
  if (k == 0) return a.piece_a[p] + q;
  if (k == 1) {
    const int s = a.piece_a[p];
    return q == 0 ? -1 : a.arm_first_op[a.site_arm_ptr[s] + H.choice[s]] + q - 1;
  }
  const int c = a.piece_c[p];
  const int w = q % (1 + c);
  if (it) {
    const int s = a.piece_a[p];
    const int i = q / (1 + c);
    *it = a.site_rev[s] ? (a.site_lo[s] + H.choice[s] - 1 - i) : i;
  }
  return w == 0 ? -1 : a.piece_b[p] + w - 1;
}

// Build group g of prediction b. All threads of the block must call it (uniform arguments).
// Writes blocks / hist / grp / ent / ent_n for (b, g).
static __device__ void build_group(const ArchDev& a, const DecHead& H, DecGroup& G, PredDev& pd, int b, int g,
                            int32_t* __restrict__ hist_tab) {
  const int tid = threadIdx.x, NT = blockDim.x, lane = tid & 31, warp = tid >> 5;
  const int s = group_start(H, g), e = group_end(H, g);
  const int nrows = e - s;
  if (tid == 0) {
    pd.grp[((int64_t)b * a.K_max + g) * 2] = s;
    pd.grp[((int64_t)b * a.K_max + g) * 2 + 1] = e;
  }
  if (tid < 9) G.sig[tid] = 0;
  __syncthreads();
  // rows split in contiguous chunks; per-thread access counts and signature sums
  const int chunk = (nrows + NT - 1) / NT;
  const int rs = s + tid * chunk, re = min(e, rs + chunk);
  long long sg[9] = {0, 0, 0, 0, 0, 0, 0, 0, 0};
  int cnt = 0;
  for (int r = rs; r < re; ++r) {
    const int op = row_op(a, H, r);
    if (op >= 0) {
      cnt += a.acc_ptr[op + 1] - a.acc_ptr[op];
#pragma unroll
      for (int k = 0; k < 9; ++k) sg[k] += a.op_sig[(int64_t)op * 9 + k];
    }
  }
  // block sums of the nine signature columns (no 64-bit shared atomics: CAS spin loops)
  for (int k = 0; k < 9; ++k) {
    const long long v = block_sum64(sg[k], G.sum_tmp);
    if (tid == 0) G.sig[k] = (unsigned long long)v;
  }
  int total = 0;
  int pos = block_scan(cnt, G.warp_tmp, &total);   // includes __syncthreads (sig sums done)
  if (tid == 0) {
    int32_t* bv = pd.blocks + ((int64_t)b * a.K_max + g) * 10;
    int32_t* hv = hist_tab + ((int64_t)b * a.K_max + g) * 10;
    const int c0 = min(nrows, kSat);
    bv[0] = c0;
    hv[0] = c0;
    for (int k = 0; k < 9; ++k) {
      const int v = (int)min((long long)G.sig[k], (long long)kSat);
      bv[1 + k] = v;
      hv[1 + k] = v;
    }
  }
  int32_t* ent_n = pd.ent_n + (int64_t)b * a.K_max + g;
  int2* ent = pd.ent + ((int64_t)b * a.K_max + g) * kEntCap;
  if (total > kRecCap) {
    if (tid == 0) { *ent_n = 0; atomicCAS(&pd.status[0], 0, DYO_E_CAPACITY); pd.status[1] = total; }
    __syncthreads();
    return;
  }
  const int n = total;
  for (int r = rs; r < re; ++r) {
    int it = 0;
    const int op = row_op(a, H, r, &it);
    if (op < 0) continue;
    for (int q = a.acc_ptr[op]; q < a.acc_ptr[op + 1]; ++q, ++pos) {
      const uint32_t t = (uint32_t)(a.acc_t[q] + a.acc_s[q] * it + a.acc_sb[q] * b);   // R13 (validated at load)
      G.key[pos] = ((uint64_t)t << 32) | ((uint64_t)pos << 2) | (uint64_t)a.acc_m[q];
    }
  }
  __syncthreads();
  if (n <= 64) {
    // ---- warp path: registers + shuffles, no block barriers ----
    if (warp == 0) {
      uint64_t x = lane < n ? G.key[lane] : ~0ull;
      uint64_t z = lane + 32 < n ? G.key[lane + 32] : ~0ull;
      warp_sort64(x, z, lane);
      G.key[lane] = x;
      G.key[lane + 32] = z;
      __syncwarp();
      uint64_t o[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int i = lane + 32 * h;
        o[h] = ~0ull;
        if (i < n) {
          const uint32_t t = (uint32_t)(G.key[i] >> 32);
          if (i == 0 || (uint32_t)(G.key[i - 1] >> 32) != t) {
            const uint32_t p0 = (uint32_t)(G.key[i] & 0xffffffffu) >> 2;
            const uint32_t m0 = (uint32_t)G.key[i] & 3u;
            uint32_t mu = m0;
            for (int k = i + 1; k < n && (uint32_t)(G.key[k] >> 32) == t; ++k) mu |= (uint32_t)G.key[k] & 3u;
            o[h] = ((uint64_t)p0 << 32) | ((uint64_t)t << 3) | (mu << 1) | (m0 & 1u);
          }
        }
      }
      warp_sort64(o[0], o[1], lane);
      const int u = __popc(__ballot_sync(0xffffffffu, o[0] != ~0ull)) + __popc(__ballot_sync(0xffffffffu, o[1] != ~0ull));
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int i = lane + 32 * h;
        if (i < u) {
          const uint32_t lo = (uint32_t)(o[h] & 0xffffffffu);
          ent[i] = make_int2((int)(lo >> 3), (int)(((lo >> 1) & 3u) | ((lo & 1u) << 2)));
        }
      }
      if (lane == 0) *ent_n = u;
    }
    __syncthreads();
    return;
  }
  // ---- block path ----
  block_sort_u64(G.key, n);
  int np2 = 1;
  while (np2 < n) np2 <<= 1;
  for (int i = tid; i < np2; i += NT) G.key2[i] = ~0ull;
  __syncthreads();
  for (int i = tid; i < n; i += NT) {
    const uint32_t t = (uint32_t)(G.key[i] >> 32);
    if (i > 0 && (uint32_t)(G.key[i - 1] >> 32) == t) continue;
    const uint32_t p0 = (uint32_t)(G.key[i] & 0xffffffffu) >> 2;
    const uint32_t m0 = (uint32_t)G.key[i] & 3u;
    uint32_t mu = m0;
    for (int k = i + 1; k < n && (uint32_t)(G.key[k] >> 32) == t; ++k) mu |= (uint32_t)G.key[k] & 3u;
    G.key2[i] = ((uint64_t)p0 << 32) | ((uint64_t)t << 3) | (mu << 1) | (m0 & 1u);
  }
  __syncthreads();
  block_sort_u64(G.key2, n);
  int flag = 0;
  for (int i = tid; i < n; i += NT) flag += G.key2[i] != ~0ull ? 1 : 0;
  int u = 0;
  block_scan(flag, G.warp_tmp, &u);
  if (u > kEntCap) {
    if (tid == 0) { *ent_n = 0; atomicCAS(&pd.status[0], 0, DYO_E_CAPACITY); pd.status[1] = u; }
    __syncthreads();
    return;
  }
  for (int i = tid; i < u; i += NT) {
    const uint32_t lo = (uint32_t)(G.key2[i] & 0xffffffffu);
    ent[i] = make_int2((int)(lo >> 3), (int)(((lo >> 1) & 3u) | ((lo & 1u) << 2)));
  }
  if (tid == 0) *ent_n = u;
  __syncthreads();
}

// Debug copies of prediction b (slots, choices, path, K, L) + the history K; one block.
static __device__ void write_head(const ArchDev& a, const DecHead& H, const double* __restrict__ y, PredDev& pd, int b,
                           int32_t* __restrict__ hist_K) {
  for (int i = threadIdx.x; i < a.K_max * 10; i += blockDim.x) {
    const int e = i % 10;
    double t = y[i] * (e < 7 ? 16.0 : 1024.0);
    t = fmin(fmax(t, 0.0), (double)kSat);
    pd.slots[(int64_t)b * a.K_max * 10 + i] = (int)rint(t);
  }
  for (int i = threadIdx.x; i < a.n_sites; i += blockDim.x) pd.choices[(int64_t)b * a.n_sites + i] = H.choice[i];
  if (H.L <= a.L_max)
    for (int r = threadIdx.x; r < H.L; r += blockDim.x) pd.path[(int64_t)b * a.L_max + r] = row_op(a, H, r);
  if (threadIdx.x == 0) {
    pd.K[b] = H.K;
    pd.L[b] = H.L;
    hist_K[b] = H.K;
  }
}

}  // namespace dyo
