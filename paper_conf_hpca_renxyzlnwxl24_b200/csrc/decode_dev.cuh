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

// debug phase stamps of the decode (SM clock; one CTA of the fused pilot epilogue)
static __device__ unsigned long long g_dec_stamp[8];
static __device__ int g_dec_stamp_on;
#define DSTAMP(i) do { if (g_dec_stamp_on && blockIdx.x == 0 && threadIdx.x == 0) g_dec_stamp[i] = (unsigned long long)clock64(); } while (0)

constexpr int kMaxPieces = 1024;
constexpr int kRecCap = 2048;          // access records per group before deduplication

struct DecHead {
  int start[kMaxPieces + 1];           // piece start rows; start[n_pieces] = L
  int cum[256 + 1];                    // start row of each group
  int cntc[256];                       // non-empty counts in slot order
  int choice[kMaxSites];
  int L, nk, K;
  int b;                               // the prediction (host-resolved paths, R16)
};

// Head of a prediction with runtime-sized arrays (the stand-alone group kernel carves them from
// dynamic shared memory: n_pieces + 1, K_max + 1, K_max and n_sites ints) - same member names
// as DecHead, so the templated group build takes either.
struct DecHeadDyn {
  int* start;
  int* cum;
  int* cntc;
  int* choice;
  int L, nk, K;
  int b;
};

// Group-build scratch for at most R access records (R a power of two).
template <int R>
struct DecGroupT {
  int32_t rec_t[R];                    // access records in row order (position = index)
  int32_t rec_m[R];                    // mode bits (R = 1, W = 2)
  int32_t first[R];                    // 1 at the first position of each tensor, then its scan
  int32_t ht_key[2 * R];               // open-addressing table: tensor -> first position, mode union
  int32_t ht_pos[2 * R];
  int32_t ht_mode[2 * R];
  int warp_tmp[32];
  long long sig_w[32][9];              // per-warp signature partial sums
  unsigned long long sig[9];
  int n, u;
};
using DecGroup = DecGroupT<kRecCap>;
constexpr int kRecSmall = 64;          // the high-occupancy first pass of the group kernel

// Copy the small decode tables (sites, arms, pieces) into shared memory `buf` (int32 words,
// capacity cap) and return an ArchDev whose pointers refer to the copies; tables that do not
// fit stay in global memory. All threads of the block call it; ends with __syncthreads().
// One flat pass over all tables with every load of a thread issued before its stores, so the
// copy costs one global round trip instead of one per table.
// int32 words stage_decode_tables needs for every table (capped; host and device)
__host__ __device__ inline int dec_table_words(const ArchDev& a, int cap) {
  const int need = 6 * a.n_sites + 4 * a.n_pieces + 2 * a.n_arms;
  return need < cap ? need : cap;
}

// The twelve small decode tables (sites, pieces, arms) in a fixed order; host and device.
constexpr int kDecTabs = 12;
__host__ __device__ inline const int32_t* dec_table(const ArchDev& a, int k, int* len) {
  switch (k) {
    case 0: *len = a.n_sites; return a.site_logit;
    case 1: *len = a.n_sites; return a.site_nch;
    case 2: *len = a.n_sites; return a.site_tie;
    case 3: *len = a.n_sites; return a.site_lo;
    case 4: *len = a.n_sites; return a.site_arm_ptr;
    case 5: *len = a.n_sites; return a.site_rev;
    case 6: *len = a.n_pieces; return a.piece_kind;
    case 7: *len = a.n_pieces; return a.piece_a;
    case 8: *len = a.n_pieces; return a.piece_b;
    case 9: *len = a.n_pieces; return a.piece_c;
    case 10: *len = a.n_arms; return a.arm_nops;
    default: *len = a.n_arms; return a.arm_first_op;
  }
}
// int32 words of the prefetched table region: every table padded to 16 bytes
__host__ __device__ inline int dec_table_region_words(const ArchDev& a) {
  int w = 0;
  for (int k = 0; k < kDecTabs; ++k) {
    int n = 0;
    dec_table(a, k, &n);
    w += (n + 3) / 4 * 4;
  }
  return w;
}
// One thread: bulk-copy (TMA) every table into `region` (16-byte aligned shared memory) and arm
// `bar` with the bytes. The tables are 256-byte aligned slab carvings, so rounding a copy up to
// 16 bytes stays inside the allocation.
__device__ __forceinline__ void prefetch_dec_tables(const ArchDev& a, int* region, uint64_t* bar) {
  uint32_t bytes = 0;
  for (int k = 0; k < kDecTabs; ++k) {
    int n = 0;
    dec_table(a, k, &n);
    bytes += (uint32_t)((n + 3) / 4 * 16);
  }
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"((uint32_t)__cvta_generic_to_shared(bar)),
               "r"(bytes) : "memory");
  int off = 0;
  for (int k = 0; k < kDecTabs; ++k) {
    int n = 0;
    const int32_t* src = dec_table(a, k, &n);
    const uint32_t nb = (uint32_t)((n + 3) / 4 * 16);
    if (nb)
      asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       (uint32_t)__cvta_generic_to_shared(region + off)),
                   "l"(src), "r"(nb), "r"((uint32_t)__cvta_generic_to_shared(bar))
                   : "memory");
    off += (n + 3) / 4 * 4;
  }
}
// The ArchDev view whose decode tables point into the prefetched region.
__device__ __forceinline__ ArchDev dec_tables_view(const ArchDev& a, const int* region) {
  ArchDev s = a;
  int off = 0, n = 0;
  auto nx = [&](int k) { dec_table(a, k, &n); const int32_t* p = region + off; off += (n + 3) / 4 * 4; return p; };
  s.site_logit = nx(0); s.site_nch = nx(1); s.site_tie = nx(2); s.site_lo = nx(3); s.site_arm_ptr = nx(4);
  s.site_rev = nx(5); s.piece_kind = nx(6); s.piece_a = nx(7); s.piece_b = nx(8); s.piece_c = nx(9);
  s.arm_nops = nx(10); s.arm_first_op = nx(11);
  return s;
}

__device__ __forceinline__ ArchDev stage_decode_tables(const ArchDev& a, int* buf, int cap) {
  constexpr int NTAB = 12;
  const int32_t* src[NTAB] = {a.site_logit, a.site_nch, a.site_tie, a.site_lo, a.site_arm_ptr, a.site_rev,
                              a.piece_kind, a.piece_a, a.piece_b, a.piece_c, a.arm_nops, a.arm_first_op};
  const int len[NTAB] = {a.n_sites, a.n_sites, a.n_sites, a.n_sites, a.n_sites, a.n_sites,
                         a.n_pieces, a.n_pieces, a.n_pieces, a.n_pieces, a.n_arms, a.n_arms};
  int beg[NTAB];
  int off = 0, nt = 0;
  bool fits = true;
#pragma unroll
  for (int k = 0; k < NTAB; ++k) {       // tables are staged in order while they fit
    beg[k] = off;
    fits = fits && (off + len[k] <= cap);
    if (fits) { off += len[k]; nt = k + 1; }
  }
  const int NT = blockDim.x;
  for (int i0 = 0; i0 < off; i0 += 8 * NT) {
    int v[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int i = i0 + u * NT + (int)threadIdx.x;
      v[u] = 0;
      if (i < off) {
        const int32_t* ptr = src[0];
        int b0 = 0;
#pragma unroll
        for (int q = 1; q < NTAB; ++q)
          if (q < nt && i >= beg[q]) { ptr = src[q]; b0 = beg[q]; }
        v[u] = __ldg(ptr + (i - b0));
      }
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const int i = i0 + u * NT + (int)threadIdx.x;
      if (i < off) buf[i] = v[u];
    }
  }
  ArchDev s = a;
  s.site_logit = nt > 0 ? buf + beg[0] : a.site_logit;
  s.site_nch = nt > 1 ? buf + beg[1] : a.site_nch;
  s.site_tie = nt > 2 ? buf + beg[2] : a.site_tie;
  s.site_lo = nt > 3 ? buf + beg[3] : a.site_lo;
  s.site_arm_ptr = nt > 4 ? buf + beg[4] : a.site_arm_ptr;
  s.site_rev = nt > 5 ? buf + beg[5] : a.site_rev;
  s.piece_kind = nt > 6 ? buf + beg[6] : a.piece_kind;
  s.piece_a = nt > 7 ? buf + beg[7] : a.piece_a;
  s.piece_b = nt > 8 ? buf + beg[8] : a.piece_b;
  s.piece_c = nt > 9 ? buf + beg[9] : a.piece_c;
  s.arm_nops = nt > 10 ? buf + beg[10] : a.arm_nops;
  s.arm_first_op = nt > 11 ? buf + beg[11] : a.arm_first_op;
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
// Raw block-head element i (R4): rint(y * 2^sigma), sigma = 4 (elements 0..6) or 10, clamped.
__device__ __forceinline__ int slot_int(const double* __restrict__ y, int i) {
  const int e = i % 10;
  double t = y[i] * (e < 7 ? 16.0 : 1024.0);
  t = fmin(fmax(t, 0.0), (double)kSat);
  return (int)rint(t);
}

// Exact-match memo lookup (R15), one warp: key = (raw block head, raw choices);
// a hit replaces H.choice with the memoised actual choices. rch (may be null) receives the raw
// choices (the key half a later dyo_report needs); only the CTA given rch counts the hit.
__device__ __forceinline__ void memo_lookup_warp(const ArchDev& a, const double* __restrict__ y, DecHead& H, int lane,
                                                 int32_t* __restrict__ rch) {
  const int ns = a.n_sites;
  if (rch)
    for (int i = lane; i < ns; i += 32) rch[i] = H.choice[i];
  if (a.memo_live <= 0 || a.forced) return;
  const int KW = 10 * a.K_max;
  uint64_t h = 0;
  for (int i = lane; i < KW; i += 32) h += memo_mix((uint64_t)i, slot_int(y, i));
  for (int i = lane; i < ns; i += 32) h += memo_mix((uint64_t)(KW + i), H.choice[i]);
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) h += __shfl_xor_sync(0xffffffffu, h, o);
  if (h == 0) h = 1;
  int slot = (int)(h & (uint64_t)a.memo_mask), hit = -1;
  for (int probe = 0; probe <= a.memo_mask; ++probe) {
    const int e = a.memo_index[slot];
    if (e == -1) break;
    if (e >= 0 && a.memo_hash[e] == h) {
      const int32_t* k = a.memo_key + (int64_t)e * (KW + ns);
      bool same = true;
      for (int i = lane; i < KW; i += 32) same = same && k[i] == slot_int(y, i);
      for (int i = lane; i < ns; i += 32) same = same && k[KW + i] == H.choice[i];
      if (__all_sync(0xffffffffu, same)) { hit = e; break; }
    }
    slot = (slot + 1) & a.memo_mask;
  }
  __syncwarp();
  if (hit >= 0) {
    for (int i = lane; i < ns; i += 32) H.choice[i] = a.memo_val[(int64_t)hit * ns + i];
    if (lane == 0 && a.memo_hits && rch) atomicAdd(a.memo_hits, 1ull);   // one decoding CTA counts
  }
  __syncwarp();
}

static __device__ void head_decode_warp(const ArchDev& a, const double* __restrict__ y, DecHead& H, int lane, int b,
                                        int32_t* __restrict__ rch = nullptr) {
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
  DSTAMP(0);
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
  memo_lookup_warp(a, y, H, lane, rch);
  DSTAMP(1);
  // 3. piece lengths -> exclusive scan -> piece starts (R2); a host-resolved path (nested
  //    sites, R16) brings its own length
  int carry = 0;
  if (a.hp_len) carry = a.hp_len[b];
  for (int p0 = 0; p0 < a.n_pieces && !a.hp_len; p0 += 32) {
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
  DSTAMP(2);
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
    H.b = b;
  }
  __syncwarp();
}

template <class HT>
__device__ __forceinline__ int group_start(const HT& H, int g) { return H.nk == 0 ? 0 : H.cum[g]; }
template <class HT>
__device__ __forceinline__ int group_end(const HT& H, int g) {
  if (H.nk == 0 || g == H.K - 1) return H.L;                    // last group absorbs the remainder
  return min(H.cum[g] + H.cntc[g], H.L);
}

// Operator of path row r (-1 for a control row); *it = iteration index of its loop for the
// per-iteration tensors (R13; 0 outside loops, counted down in a reversed loop).
template <class HT>
__device__ __forceinline__ int row_op(const ArchDev& a, const HT& H, int r, int* it = nullptr) {
  if (a.hp_op) {                                               // host-resolved path (R16)
    const int64_t i = (int64_t)H.b * a.L_max + r;
    if (it) *it = a.hp_it[i];
    return a.hp_op[i];
  }
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
// Writes blocks / hist / grp / ent / ent_n for (b, g). With R < kRecCap a group of more than R
// records is left pending (ent_n = -1) for the full-capacity pass.
template <class HT, int R>
static __device__ void build_group(const ArchDev& a, const HT& H, DecGroupT<R>& G, PredDev& pd, int b, int g,
                            int32_t* __restrict__ hist_tab) {
  const int tid = threadIdx.x, NT = blockDim.x, lane = tid & 31, warp = tid >> 5;
  const int s = group_start(H, g), e = group_end(H, g);
  const int nrows = e - s;
  if (tid == 0) {
    pd.grp[((int64_t)b * a.K_max + g) * 2] = s;
    pd.grp[((int64_t)b * a.K_max + g) * 2 + 1] = e;
  }
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
  // the nine signature sums: warp shuffles, then one pass over the per-warp partials (a single
  // barrier, shared with the scan below; no 64-bit shared atomics: CAS spin loops)
  const int nw = (NT + 31) >> 5;
#pragma unroll
  for (int k = 0; k < 9; ++k) {
    long long v = sg[k];
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    if (lane == 0) G.sig_w[warp][k] = v;
  }
  DSTAMP(3);
  int total = 0;
  int pos = block_scan(cnt, G.warp_tmp, &total);   // its barriers also publish sig_w
  DSTAMP(4);
  if (tid < 9) {
    long long v = 0;
    for (int w = 0; w < nw; ++w) v += G.sig_w[w][tid];
    G.sig[tid] = (unsigned long long)v;
  }
  int32_t* ent_n = pd.ent_n + (int64_t)b * a.K_max + g;
  int2* ent = pd.ent + ((int64_t)b * a.K_max + g) * kEntCap;
  if (total > R) {
    if (tid == 0) {
      if (R < kRecCap) {
        *ent_n = -1;                                   // pending: the full-capacity pass builds it
      } else {
        *ent_n = 0;
        atomicCAS(&pd.status[0], 0, DYO_E_CAPACITY);
        pd.status[1] = total;
      }
    }
    __syncthreads();
    return;
  }
  const int n = total;
  for (int r = rs; r < re; ++r) {
    int it = 0;
    const int op = row_op(a, H, r, &it);
    if (op < 0) continue;
    for (int q = a.acc_ptr[op]; q < a.acc_ptr[op + 1]; ++q, ++pos) {
      G.rec_t[pos] = a.acc_t[q] + a.acc_s[q] * it + a.acc_sb[q] * b;   // R13 (validated at load)
      G.rec_m[pos] = a.acc_m[q];
    }
  }
  // hash-table size (power of two >= 2n) and its initialisation ride the same barrier
  int hsz = 64;
  while (hsz < 2 * n) hsz <<= 1;
  if (n > 64) {
    for (int i = tid; i < hsz; i += NT) { G.ht_key[i] = -1; G.ht_pos[i] = 0x7fffffff; G.ht_mode[i] = 0; }
    for (int i = tid; i < n; i += NT) G.first[i] = 0;
  }
  __syncthreads();
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
  DSTAMP(5);
  if (n <= 64) {
    // ---- warp path: registers + shuffles, no block barriers ----
    if (warp == 0) {
      uint64_t x = lane < n ? ((uint64_t)(uint32_t)G.rec_t[lane] << 32) | ((uint64_t)lane << 2) | (uint64_t)G.rec_m[lane] : ~0ull;
      uint64_t z = lane + 32 < n ? ((uint64_t)(uint32_t)G.rec_t[lane + 32] << 32) | ((uint64_t)(lane + 32) << 2) |
                                       (uint64_t)G.rec_m[lane + 32]
                                 : ~0ull;
      warp_sort64(x, z, lane);
      uint64_t* key = reinterpret_cast<uint64_t*>(G.ht_key);   // scratch (unused on this path)
      key[lane] = x;
      key[lane + 32] = z;
      __syncwarp();
      uint64_t o[2];
#pragma unroll
      for (int h = 0; h < 2; ++h) {
        const int i = lane + 32 * h;
        o[h] = ~0ull;
        if (i < n) {
          const uint32_t t = (uint32_t)(key[i] >> 32);
          if (i == 0 || (uint32_t)(key[i - 1] >> 32) != t) {
            const uint32_t p0 = (uint32_t)(key[i] & 0xffffffffu) >> 2;
            const uint32_t m0 = (uint32_t)key[i] & 3u;
            uint32_t mu = m0;
            for (int k = i + 1; k < n && (uint32_t)(key[k] >> 32) == t; ++k) mu |= (uint32_t)key[k] & 3u;
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
  // ---- block path: tensor -> (first position, mode union) in an open-addressing table
  //      (32-bit shared atomics: CAS / min / or, order-independent), then the first positions
  //      are flagged and one exclusive scan gives every tensor its slot in first-access order ----
  const int mask = hsz - 1;
  for (int i = tid; i < n; i += NT) {
    const int t = G.rec_t[i];
    int h = (int)(((uint32_t)t * 2654435761u) >> 7) & mask;
    for (;;) {
      const int old = atomicCAS(&G.ht_key[h], -1, t);
      if (old == -1 || old == t) {
        atomicMin(&G.ht_pos[h], i);
        atomicOr(&G.ht_mode[h], G.rec_m[i]);
        break;
      }
      h = (h + 1) & mask;
    }
  }
  __syncthreads();
  for (int h = tid; h < hsz; h += NT)
    if (G.ht_key[h] >= 0) G.first[G.ht_pos[h]] = h + 1;     // slot + 1 at the tensor's first position
  __syncthreads();
  int u = 0;
  for (int i0 = 0; i0 < n; i0 += NT) {
    const int i = i0 + tid;
    const int f = i < n ? G.first[i] : 0;
    int tot = 0;
    const int idx = u + block_scan(f ? 1 : 0, G.warp_tmp, &tot);
    if (f && idx < kEntCap) {
      const int h = f - 1;
      const int m0 = G.rec_m[i];
      ent[idx] = make_int2(G.ht_key[h], (G.ht_mode[h] & 3) | ((m0 & 1) << 2));
    }
    u += tot;
  }
  if (u > kEntCap) {
    if (tid == 0) { *ent_n = 0; atomicCAS(&pd.status[0], 0, DYO_E_CAPACITY); pd.status[1] = u; }
    __syncthreads();
    return;
  }
  if (tid == 0) *ent_n = u;
  __syncthreads();
}

// Debug copies of prediction b (slots, choices, path, K, L) + the history K; one block.
static __device__ void write_head(const ArchDev& a, const DecHead& H, const double* __restrict__ y, PredDev& pd, int b,
                           int32_t* __restrict__ hist_K) {
  for (int i = threadIdx.x; i < a.K_max * 10; i += blockDim.x) pd.slots[(int64_t)b * a.K_max * 10 + i] = slot_int(y, i);
  for (int i = threadIdx.x; i < a.n_sites; i += blockDim.x) pd.choices[(int64_t)b * a.n_sites + i] = H.choice[i];
  if (H.L <= a.L_max && !a.hp_op)
    for (int r = threadIdx.x; r < H.L; r += blockDim.x) pd.path[(int64_t)b * a.L_max + r] = row_op(a, H, r);
  if (threadIdx.x == 0) {
    pd.K[b] = H.K;
    pd.L[b] = H.L;
    hist_K[b] = H.K;
  }
}

}  // namespace dyo
