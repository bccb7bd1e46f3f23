// K2: the double-buffered evict/prefetch planner (§IV-E, §V;
// DESIGN.md R7-R12). Integer-only and deterministic (every ordering decision is a sort on a
// unique key; atomics only count or fill order-free buckets), so it is bit-exact with
// oracle/plan.py.
//
// Launch sequence of one dyo_plan (one stream, no host round trip):
//   plan_prep_kernel     (1 CTA)   group list of the plan, entry bases (block scans)
//   bucket kernels       (grid)    every entry's next occurrence of its tensor: entries are
//                                  bucketed per tensor, each bucket sorted by group (one warp per
//                                  tensor) - replaces a sequential reverse sweep over the groups
//   plan_kernel          (1 CTA)   the transitions, sequential, parallel inside
//   plan_export_kernel   (grid)    records -> pinned host mirrors (api.cpp)
//
// plan_kernel keeps, per half, the list of its valid tensors in ascending offset as 16-byte
// records carrying everything the candidate scan needs (offset, aligned size, id, transient /
// next-use-reads / dirty flags, next-use group), so a transition touches the half's list in a
// few coalesced passes (one contiguous chunk per thread, one block scan per pass) and its W_j
// through shared memory:
//   A  load W_j, classify KEEP / CARRY / ALLOC / FETCH (R8), need, feasibility (R7)
//   B  scan the half: dead (R9) / live candidates, live bytes
//   C  RETAIN with live bytes > room only: radix select of the prefix cut over the keys
//      (next-use distance, aligned size, id) - the north_star's "top-k over sizes and reuse
//      distance" as a threshold, no full sort (R10)
//   D  kept list + EVICT keys (block scan compaction), gaps between kept tensors
//   E  placement keys (CARRY by id, ALLOC by id, FETCH by host offset) rank-sorted; first fit
//      (R11) by one warp, a run of equal sizes at a time (exact: a run fills the gaps in address
//      order), compaction by exclusive prefix sums when a run does not fit
//   F  records + per-tensor state; CARRY tombstones the source record of the other half
//   G  rebuild the half's list: merge of the kept (offset order) and placed tensors
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>

#include "dyo_device.cuh"
#include "dyo_internal.h"

namespace dyo {

constexpr int NT = kPlanThreads;                  // 1024
constexpr uint64_t kInfD = 0xFFFFull;
constexpr int kInwSmemWords = 8192;               // smem W_j bitmap for T <= 2^18
constexpr int kEvSmem = 8192;                     // EVICT keys sorted in shared memory up to this

__device__ unsigned long long g_pstamp[64];
__device__ int g_pstamp_j = -1;
#define PSTAMP(i) do { if (j == pstamp_j && tid == 0) g_pstamp[i] = (unsigned long long)clock64(); } while (0)

// ---- small block primitives (1024 threads) --------------------------------------------
// Exclusive scan of one int64 per thread; *total = sum. tmp: 32 long longs. Three barriers.
__device__ __forceinline__ long long scan64(long long v, long long* tmp, long long* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  long long x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const long long y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) tmp[w] = x;
  __syncthreads();
  if (w == 0) {
    long long s = tmp[lane];
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const long long y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    tmp[lane] = s;
  }
  __syncthreads();
  const long long base = w > 0 ? tmp[w - 1] : 0;
  *total = tmp[31];
  __syncthreads();
  return base + x - v;
}

// Sums of four int64 per thread over the block (every thread gets them). Two barriers.
__device__ __forceinline__ void sum4(long long v[4], long long (*tmp)[4]) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
#pragma unroll
  for (int q = 0; q < 4; ++q)
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) v[q] += __shfl_xor_sync(0xffffffffu, v[q], o);
  if (lane == 0)
#pragma unroll
    for (int q = 0; q < 4; ++q) tmp[w][q] = v[q];
  __syncthreads();
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    long long s = 0;
    for (int i = 0; i < 32; ++i) s += tmp[i][q];
    v[q] = s;
  }
  __syncthreads();
}

__device__ __forceinline__ bool bit_get(const uint32_t* b, int t) { return (b[t >> 5] >> (t & 31)) & 1u; }

// ---- 0. group list + entry bases -------------------------------------------------------
__global__ void __launch_bounds__(NT, 1)
plan_prep_kernel(ArchDev a, PredDev pd, int b0, int nb, PlanScratch sc, PlanOut out, int max_groups) {
  __shared__ long long tmp[32];
  __shared__ int s_fail;
  const int tid = threadIdx.x;
  int* status = out.status;
  if (tid == 0) {
    s_fail = 0;
    if (pd.status[0] != 0) { status[0] = pd.status[0]; status[2] = pd.status[1]; s_fail = 1; }
  }
  __syncthreads();
  if (s_fail) { if (tid == 0) sc.Kt[0] = -1; return; }
  // groups per prediction -> group list (nb <= 1024: one prediction per thread)
  const int Kb = tid < nb ? pd.K[b0 + tid] : 0;
  long long Kt = 0;
  const long long gb = scan64(Kb, tmp, &Kt);
  if (Kt > max_groups) {
    if (tid == 0) { status[0] = DYO_E_CAPACITY; status[2] = (int)Kt; sc.Kt[0] = -1; }
    return;
  }
  for (int k = 0; k < Kb; ++k) { sc.grp_b[gb + k] = b0 + tid; sc.grp_k[gb + k] = k; }
  __syncthreads();
  // entry bases: a contiguous chunk of groups per thread, one scan
  const int per = (int)((Kt + NT - 1) / NT);
  const int g0 = min((int)Kt, tid * per), g1 = min((int)Kt, g0 + per);
  long long c = 0;
  for (int g = g0; g < g1; ++g) c += pd.ent_n[sc.grp_b[g] * a.K_max + sc.grp_k[g]];
  long long tot = 0;
  long long base = scan64(c, tmp, &tot);
  if (tot > out.cap_ent) {
    if (tid == 0) { status[0] = DYO_E_CAPACITY; status[2] = (int)tot; sc.Kt[0] = -1; }
    return;
  }
  for (int g = g0; g < g1; ++g) {
    sc.ebase[g] = base;
    out.hdr[g].o_ent = base;
    base += pd.ent_n[sc.grp_b[g] * a.K_max + sc.grp_k[g]];
  }
  if (tid == 0) sc.Kt[0] = (int)Kt;
}

// ---- bucket kernels: next occurrence of every entry's tensor ---------------------------
__global__ void bucket_init_kernel(ArchDev a, PlanScratch sc) {
  for (int t = blockIdx.x * blockDim.x + threadIdx.x; t < a.T; t += gridDim.x * blockDim.x) {
    sc.bcnt[t] = 0;
    sc.bfill[t] = 0;
    sc.first[t] = -1;
    sc.first_rd[t] = 0;
    sc.au[t] = (int32_t)(a.t_abytes[t] / a.align);
  }
}

__device__ __forceinline__ const int2* group_entries(const ArchDev& a, const PredDev& pd, const PlanScratch& sc, int g,
                                                     int* n) {
  const int64_t slot = (int64_t)sc.grp_b[g] * a.K_max + sc.grp_k[g];
  *n = pd.ent_n[slot];
  return pd.ent + slot * kEntCap;
}

// one block per group (grid-stride)
__global__ void bucket_count_kernel(ArchDev a, PredDev pd, PlanScratch sc) {
  const int Kt = sc.Kt[0];
  for (int g = blockIdx.x; g < Kt; g += gridDim.x) {
    int n;
    const int2* ent = group_entries(a, pd, sc, g, &n);
    for (int e = threadIdx.x; e < n; e += blockDim.x) atomicAdd(&sc.bcnt[ent[e].x], 1);
  }
}

// exclusive scan of the bucket counts (one CTA, a contiguous chunk of tensors per thread)
__global__ void __launch_bounds__(NT, 1) bucket_scan_kernel(ArchDev a, PlanScratch sc) {
  __shared__ long long tmp[32];
  if (sc.Kt[0] < 0) return;
  const int T = a.T, per = (T + NT - 1) / NT;
  const int t0 = min(T, (int)threadIdx.x * per), t1 = min(T, t0 + per);
  long long c = 0;
  for (int t = t0; t < t1; ++t) c += sc.bcnt[t];
  long long tot = 0;
  long long base = scan64(c, tmp, &tot);
  for (int t = t0; t < t1; ++t) {
    const int v = sc.bcnt[t];
    sc.bcnt[t] = (int)base;
    base += v;
  }
  if (threadIdx.x == 0) sc.bcnt[T] = (int)tot;
}

__global__ void bucket_fill_kernel(ArchDev a, PredDev pd, PlanScratch sc) {
  const int Kt = sc.Kt[0];
  for (int g = blockIdx.x; g < Kt; g += gridDim.x) {
    int n;
    const int2* ent = group_entries(a, pd, sc, g, &n);
    for (int e = threadIdx.x; e < n; e += blockDim.x) {
      const int t = ent[e].x;
      sc.bkey[sc.bcnt[t] + atomicAdd(&sc.bfill[t], 1)] = (g << 10) | e;
    }
  }
}

// one warp per tensor: sort its bucket by group (keys are unique: a tensor appears once per
// group), then every entry learns the next group holding the tensor and whether that
// occurrence reads it first; the tensor learns its first occurrence in the plan
__global__ void bucket_sort_kernel(ArchDev a, PredDev pd, PlanScratch sc) {
  if (sc.Kt[0] < 0) return;
  const int lane = threadIdx.x & 31;
  const int warps = (gridDim.x * blockDim.x) >> 5;
  for (int t = (blockIdx.x * blockDim.x + threadIdx.x) >> 5; t < a.T; t += warps) {
    const int lo = sc.bcnt[t], hi = sc.bcnt[t + 1], n = hi - lo;
    if (n == 0) continue;
    auto rd_of = [&](int key) {
      const int g = key >> 10, e = key & 1023;
      const int64_t slot = (int64_t)sc.grp_b[g] * a.K_max + sc.grp_k[g];
      return (uint8_t)((pd.ent[slot * kEntCap + e].y >> 2) & 1);
    };
    auto emit = [&](int key, int next_key) {
      const int g = key >> 10, e = key & 1023;
      const int64_t gi = sc.ebase[g] + e;
      sc.nxt[gi] = next_key < 0 ? -1 : (next_key >> 10);
      sc.nxt_rd[gi] = next_key < 0 ? 0 : rd_of(next_key);
    };
    if (n <= 32) {
      // bitonic sort of <= 32 keys in registers
      int k = lane < n ? sc.bkey[lo + lane] : 0x7fffffff;
#pragma unroll
      for (int kk = 2; kk <= 32; kk <<= 1)
#pragma unroll
        for (int jj = kk >> 1; jj > 0; jj >>= 1) {
          const int p = __shfl_xor_sync(0xffffffffu, k, jj);
          const bool up = (lane & kk) == 0, lower = (lane & jj) == 0;
          k = (lower == up) ? min(k, p) : max(k, p);
        }
      const int nk = __shfl_down_sync(0xffffffffu, k, 1);
      if (lane < n) emit(k, lane + 1 < n ? nk : -1);
      if (lane == 0) { sc.first[t] = k >> 10; sc.first_rd[t] = rd_of(k); }
    } else {
      // rank sort into bsort (each lane ranks n / 32 of the keys)
      for (int i = lane; i < n; i += 32) {
        const int k = sc.bkey[lo + i];
        int r = 0;
        for (int q = 0; q < n; ++q) r += sc.bkey[lo + q] < k;
        sc.bsort[lo + r] = k;
      }
      __syncwarp();
      for (int i = lane; i < n; i += 32) emit(sc.bsort[lo + i], i + 1 < n ? sc.bsort[lo + i + 1] : -1);
      if (lane == 0) { sc.first[t] = sc.bsort[lo] >> 10; sc.first_rd[t] = rd_of(sc.bsort[lo]); }
    }
  }
}

// ---- the sequential planner ------------------------------------------------------------
struct PlanSmem {
  int32_t e_t[kEntCap];
  int8_t e_mode[kEntCap];
  int8_t e_rd[kEntCap];
  int8_t e_cls[kEntCap];
  uint64_t pkey[kEntCap];        // placement sort keys
  int32_t p_t[kEntCap];          // placed tensors in placement order
  int32_t p_a[kEntCap];          // their aligned sizes (units)
  int32_t p_off[kEntCap];        // their new offsets (units)
  int32_t p_cls[kEntCap];
  int32_t q_off[kEntCap];        // placed offsets sorted ascending (rebuild merge)
  int32_t q_idx[kEntCap];        // placement index of q_off[k]
  int32_t q_cnt[kEntCap];        // kept tensors below q_off[k]
  uint32_t hist[256];
  uint32_t hcnt[256];
  long long tmp[32];
  long long tmp4[32][4];
};

__device__ __forceinline__ uint64_t live_key(int4 r, int j) {
  const uint64_t d = r.w < 0 ? kInfD : (uint64_t)(r.w - j);
  return (d << 48) | ((uint64_t)r.y << 20) | (uint64_t)(r.z & kRecIdMask);
}

// 0 skip (tombstone), 1 keep (in W_j), 2 dead, 3 live
__device__ __forceinline__ int rec_kind(int4 r, const uint32_t* inw) {
  if (r.z & kRecTomb) return 0;
  const int t = r.z & kRecIdMask;
  if (bit_get(inw, t)) return 1;
  const bool dead = (r.w < 0 && (r.z & kRecTransient)) || (r.w >= 0 && !(r.z & kRecNxRd));
  return dead ? 2 : 3;
}

__device__ __forceinline__ bool rec_evicted(int4 r, int k, int rule, uint64_t thresh, int j) {
  return k == 2 || (k == 3 && (rule == 0 || (rule == 2 && live_key(r, j) >= thresh)));
}

__global__ void __launch_bounds__(NT, 1)
plan_kernel(ArchDev a, PredDev pd, int policy, PlanState in, PlanState st, PlanScratch sc, PlanOut out,
            int inw_smem) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PlanSmem& S = *reinterpret_cast<PlanSmem*>(smem_raw);
  uint64_t* evs = reinterpret_cast<uint64_t*>(smem_raw + (sizeof(PlanSmem) + 15) / 16 * 16);   // kEvSmem keys
  uint32_t* inw = inw_smem ? reinterpret_cast<uint32_t*>(evs + kEvSmem) : sc.inw;
  const int T = a.T;
  const int64_t AL = a.align;
  const int Hu = (int)(a.H / AL);
  int* status = out.status;
  const int tid = threadIdx.x, lane = tid & 31;
  const int Kt = sc.Kt[0];
  if (Kt < 0) return;                              // prep failed (status already set)
  const int nwords = (T + 31) >> 5;

  // ---- 1. work copy of the committed state (transactional, R7), R9, next uses of the plan
  for (int t = tid; t < T; t += NT) {
    st.loc[t] = in.loc[t];
    st.off[t] = in.off[t];
    st.dirty[t] = (a.t_flags[t] & 1) ? 0 : in.dirty[t];
    st.pw[t] = in.pw[t];
    st.prev[t] = in.prev[t];
    st.pos[t] = in.pos[t];
  }
  for (int w = tid; w < nwords; w += NT) inw[w] = 0u;
  __shared__ int s_n[2], s_sel[2];
  if (tid == 0) {
    st.prev_n[0] = in.prev_n[0];
    for (int h = 0; h < 2; ++h) { s_n[h] = in.rl_meta[h]; s_sel[h] = in.rl_meta[2 + h]; }
  }
  __syncthreads();
  for (int h = 0; h < 2; ++h) {
    const int4* src = in.rl[h][s_sel[h]];
    int4* dst = st.rl[h][s_sel[h]];
    for (int i = tid; i < s_n[h]; i += NT) {
      int4 r = src[i];
      const int t = r.z & kRecIdMask;
      if (r.z & kRecTransient) r.z &= ~kRecDirty;            // R9: transient contents end
      r.w = sc.first[t];
      r.z = (r.z & ~kRecNxRd) | (sc.first_rd[t] ? kRecNxRd : 0);
      dst[i] = r;
    }
  }
  __syncthreads();

  __shared__ long long c_ev, c_mv, c_ca, c_al, c_fe;
  __shared__ int s_np, s_compact, s_nkept, s_nev, s_ng, s_nmove;
  __shared__ unsigned long long s_thresh;
  if (tid == 0) { c_ev = c_mv = c_ca = c_al = c_fe = 0; }
  const int pstamp_j = g_pstamp_j;
  const int64_t G0 = in.G[0];

  for (int j = 0; j < Kt; ++j) {
    PSTAMP(0);
    const int m = (int)((G0 + j) & 1);
    int n;
    const int2* ent = group_entries(a, pd, sc, j, &n);
    const int64_t eb = sc.ebase[j];
    PlanHdr& hd = out.hdr[j];
    // ---- A. W_j, classes, need (R7, R8)
    long long v4[4] = {0, 0, 0, 0};                 // need units, carries, allocs, fetches
    if (tid < n) {
      const int2 en = ent[tid];
      const int t = en.x, md = en.y & 3, rd = (en.y >> 2) & 1;
      const int l = st.loc[t];
      const int c = l == m ? C_KEEP : (l == 1 - m && rd ? C_CARRY : (rd ? C_FETCH : C_ALLOC));
      S.e_t[tid] = t;
      S.e_mode[tid] = (int8_t)md;
      S.e_rd[tid] = (int8_t)rd;
      S.e_cls[tid] = (int8_t)c;
      sc.wnx[t] = sc.nxt[eb + tid];
      sc.wfl[t] = (uint8_t)(sc.nxt_rd[eb + tid] | ((md & 2) ? 2 : 0));
      atomicOr(&inw[t >> 5], 1u << (t & 31));
      v4[0] = sc.au[t];
      v4[1] = c == C_CARRY;
      v4[2] = c == C_ALLOC;
      v4[3] = c == C_FETCH;
    }
    sum4(v4, S.tmp4);
    const long long need_u = v4[0];
    const int nc = (int)v4[1], na = (int)v4[2], nf = (int)v4[3];
    if (need_u > Hu) {
      if (tid == 0) { status[0] = DYO_E_BUDGET; status[1] = j; status[2] = 0; }
      return;
    }
    const long long room = Hu - need_u;
    PSTAMP(1);
    // ---- B. candidates of half m: dead (R9) / live, live bytes
    const int nm = s_n[m];
    int4* recs = st.rl[m][s_sel[m]];
    const int per = (nm + NT - 1) / NT;
    const int i0 = min(nm, tid * per), i1 = min(nm, i0 + per);
    long long live_u = 0;
    {
      long long w4[4] = {0, 0, 0, 0};
      for (int i = i0; i < i1; ++i) {
        const int4 r = recs[i];
        if (rec_kind(r, inw) == 3) w4[0] += r.y;
      }
      sum4(w4, S.tmp4);
      live_u = w4[0];
    }
    // eviction rule: 0 evict every live candidate (PAPER), 1 keep all (RETAIN, fits), 2 cut
    const int rule = policy == 0 ? 0 : (live_u <= room ? 1 : 2);
    PSTAMP(2);
    // ---- C. RETAIN prefix cut by radix select: the smallest key K* whose prefix sum of
    //      aligned sizes (keys ascending) exceeds the room; keys >= K* are evicted
    if (rule == 2) {
      long long cnt = 0;
      for (int i = i0; i < i1; ++i) cnt += rec_kind(recs[i], inw) == 3;
      long long nlive = 0;
      long long kb = scan64(cnt, S.tmp, &nlive);
      for (int i = i0; i < i1; ++i) {
        const int4 r = recs[i];
        if (rec_kind(r, inw) == 3) sc.keys[kb++] = live_key(r, j);
      }
      __syncthreads();
      uint64_t prefix = 0, mask = 0;
      long long cum = 0;                             // units of the keys below the prefix
      const int kper = (int)((nlive + NT - 1) / NT);
      const int k0 = min((int)nlive, tid * kper), k1 = min((int)nlive, k0 + kper);
      for (int shift = 56; shift >= 0; shift -= 8) {
        if (tid < 256) { S.hist[tid] = 0; S.hcnt[tid] = 0; }
        __syncthreads();
        for (int k = k0; k < k1; ++k) {
          const uint64_t key = sc.keys[k];
          if ((key & mask) == prefix) {
            const int dg = (int)((key >> shift) & 255);
            atomicAdd(&S.hist[dg], (uint32_t)((key >> 20) & ((1u << 28) - 1)));
            atomicAdd(&S.hcnt[dg], 1u);
          }
        }
        __syncthreads();
        if (tid < 32) {
          // 8 bins per lane: the first digit whose cumulative units exceed the room
          long long loc[8];
          long long s = 0;
#pragma unroll
          for (int q = 0; q < 8; ++q) { s += S.hist[lane * 8 + q]; loc[q] = s; }
          long long incl = s;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const long long y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
          }
          const long long excl = incl - s;
          int found = 256;
          long long below = 0;                       // units of this lane's bins under `found`
#pragma unroll
          for (int q = 7; q >= 0; --q)
            if (cum + excl + loc[q] > room) { found = lane * 8 + q; below = q ? loc[q - 1] : 0; }
          const unsigned bal = __ballot_sync(0xffffffffu, found < 256);
          const int src = __ffs(bal) - 1;
          const int dg = __shfl_sync(0xffffffffu, found, src);
          const long long add = __shfl_sync(0xffffffffu, excl + below, src);
          if (lane == 0) {
            S.tmp[0] = dg;
            S.tmp[1] = add;
            S.tmp[2] = S.hcnt[dg];
          }
        }
        __syncthreads();
        const int dg = (int)S.tmp[0];
        cum += S.tmp[1];
        prefix |= (uint64_t)dg << shift;
        mask |= 255ull << shift;
        const int bcount = (int)S.tmp[2];
        __syncthreads();
        if (bcount == 1) break;
      }
      // the threshold: the unique key under the prefix (keys are unique)
      for (int k = k0; k < k1; ++k) {
        const uint64_t key = sc.keys[k];
        if ((key & mask) == prefix) s_thresh = key;
      }
      __syncthreads();
    }
    const uint64_t thresh = rule == 2 ? s_thresh : 0;
    PSTAMP(3);
    // ---- D. kept list (offset order) and EVICT keys (host offset, id, writeback)
    {
      long long ck = 0, ce = 0;
      for (int i = i0; i < i1; ++i) {
        const int4 r = recs[i];
        const int k = rec_kind(r, inw);
        if (k == 0) continue;
        if (rec_evicted(r, k, rule, thresh, j)) ++ce; else ++ck;
      }
      long long nk = 0, ne = 0;
      long long bk = scan64(ck, S.tmp, &nk);
      long long be = scan64(ce, S.tmp, &ne);
      if (c_ev + ne > out.cap_rec) {
        if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_ev + ne); }
        return;
      }
      uint64_t* ekeys = ne <= kEvSmem ? evs : sc.keys;
      for (int i = i0; i < i1; ++i) {
        const int4 r = recs[i];
        const int k = rec_kind(r, inw);
        if (k == 0) continue;
        if (rec_evicted(r, k, rule, thresh, j)) {
          const int t = r.z & kRecIdMask;
          const uint64_t wb = (k == 3 && (r.z & kRecDirty)) ? 1 : 0;
          ekeys[be++] = ((uint64_t)(a.t_host[t] / AL) << 21) | ((uint64_t)t << 1) | wb;
        } else {
          sc.kept[bk++] = r;
        }
      }
      if (tid == 0) { s_nkept = (int)nk; s_nev = (int)ne; }
      __syncthreads();
    }
    const int nkept = s_nkept, nev = s_nev;
    PSTAMP(4);
    // gaps of half m between the kept tensors
    {
      const int kper = (nkept + 1 + NT - 1) / NT;
      const int q0 = min(nkept + 1, tid * kper), q1 = min(nkept + 1, q0 + kper);
      int prev_end = 0;
      if (q0 > 0 && q0 <= nkept) { const int4 r = sc.kept[q0 - 1]; prev_end = r.x + r.y; }
      long long cg = 0;
      int pe = prev_end;
      for (int q = q0; q < q1; ++q) {
        const int ge = q == nkept ? Hu : sc.kept[q].x;
        if (ge > pe) ++cg;
        if (q < nkept) { const int4 r = sc.kept[q]; pe = r.x + r.y; }
      }
      long long ng = 0;
      long long bg = scan64(cg, S.tmp, &ng);
      pe = prev_end;
      for (int q = q0; q < q1; ++q) {
        const int ge = q == nkept ? Hu : sc.kept[q].x;
        if (ge > pe) { sc.gap_s[bg] = pe; sc.gap_e[bg] = ge; ++bg; }
        if (q < nkept) { const int4 r = sc.kept[q]; pe = r.x + r.y; }
      }
      if (tid == 0) s_ng = (int)ng;
    }
    // ---- E. placement order: CARRY by id, ALLOC by id, FETCH by (host offset, id)
    if (tid == 0) s_np = 0;
    __syncthreads();
    if (tid < n && S.e_cls[tid] != C_KEEP) {
      const int c = S.e_cls[tid], t = S.e_t[tid];
      const uint64_t rank = c == C_CARRY ? 0 : (c == C_ALLOC ? 1 : 2);
      const uint64_t mid = c == C_FETCH ? (uint64_t)(a.t_host[t] / AL) : 0;
      S.pkey[atomicAdd(&s_np, 1)] = (rank << 62) | (mid << 20) | (uint64_t)t;
    }
    __syncthreads();
    const int np = s_np;
    if (tid < np) {
      const uint64_t k = S.pkey[tid];
      int r = 0;
      for (int q = 0; q < np; ++q) r += S.pkey[q] < k;
      const int t = (int)(k & kRecIdMask);
      S.p_t[r] = t;
      S.p_a[r] = sc.au[t];
      S.p_cls[r] = (int)(k >> 62);
    }
    __syncthreads();
    PSTAMP(5);
    // first fit by warp 0 (R11): a run of equal aligned sizes fills the gaps in address order
    if (tid < 32) {
      const int ng = s_ng;
      bool fail = false;
      int i = 0;
      while (i < np && !fail) {
        const int asz = S.p_a[i];
        int r = 1;
        while (i + r < np && S.p_a[i + r] == asz) ++r;
        int left = r, done = 0;
        for (int g0 = 0; g0 < ng && left > 0; g0 += 32) {
          const int g = g0 + lane;
          const int gs = g < ng ? sc.gap_s[g] : 0;
          const int cap = g < ng ? (sc.gap_e[g] - gs) / asz : 0;
          int incl = cap;
#pragma unroll
          for (int o = 1; o < 32; o <<= 1) {
            const int y = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += y;
          }
          const int excl = incl - cap;
          const int take = max(0, min(cap, left - excl));
          for (int q = 0; q < take; ++q) S.p_off[i + done + excl + q] = gs + q * asz;
          if (take > 0) sc.gap_s[g] = gs + take * asz;
          const int got = min(__shfl_sync(0xffffffffu, incl, 31), left);
          left -= got;
          done += got;
        }
        __syncwarp();
        if (left > 0) fail = true;
        i += r;
      }
      if (lane == 0) s_compact = fail ? 1 : 0;
    }
    __syncthreads();
    const int compact = s_compact;
    if (compact) {
      // exclusive prefix sums over [kept in offset order | placed in placement order]
      const int kper = (nkept + NT - 1) / NT;
      const int q0 = min(nkept, tid * kper), q1 = min(nkept, q0 + kper);
      long long cu = 0;
      for (int q = q0; q < q1; ++q) cu += sc.kept[q].y;
      long long tot = 0;
      long long base = scan64(cu, S.tmp, &tot);
      for (int q = q0; q < q1; ++q) {
        const int4 r = sc.kept[q];
        sc.newoff[r.z & kRecIdMask] = (int)base;
        base += r.y;
      }
      if (tid == 0) {
        long long c = tot;
        for (int p = 0; p < np; ++p) { S.p_off[p] = (int)c; c += S.p_a[p]; }
      }
      __syncthreads();
    }
    PSTAMP(6);
    // ---- F. records
    if (c_ca + nc > out.cap_rec || c_al + na > out.cap_rec || c_fe + nf > out.cap_rec ||
        c_mv + nkept > out.cap_rec) {
      if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_mv + nkept); }
      return;
    }
    // EVICT, sorted by (host offset, id)
    {
      uint64_t* ekeys = nev <= kEvSmem ? evs : sc.keys;
      if (nev <= NT) {
        uint64_t k = 0;
        int r = 0;
        if (tid < nev) {
          k = ekeys[tid];
          for (int q = 0; q < nev; ++q) r += ekeys[q] < k;
        }
        __syncthreads();
        if (tid < nev) ekeys[r] = k;
        __syncthreads();
      } else {
        block_sort_u64(ekeys, nev);                   // bitonic (smem up to kEvSmem, else global)
      }
      long long d2h = 0;
      for (int k = tid; k < nev; k += NT) {
        const uint64_t key = ekeys[k];
        const int t = (int)((key >> 1) & kRecIdMask);
        const int wb = (int)(key & 1);
        dyo_evict_rec r;
        r.t = t;
        r.src = (int64_t)m * a.H + st.off[t];
        r.host_off = a.t_host[t];
        r.bytes = a.t_bytes[t];
        r.writeback = wb;
        out.ev[c_ev + k] = r;
        if (wb) d2h += r.bytes;
        st.loc[t] = -1;
        st.dirty[t] = 0;
      }
      long long s4[4] = {d2h, 0, 0, 0};
      sum4(s4, S.tmp4);
      if (tid == 0) hd.d2h = s4[0];
    }
    // MOVE (compaction only): kept tensors whose offset changed, in kept (= destination) order
    long long d2d = 0, h2d = 0;
    if (compact) {
      const int kper = (nkept + NT - 1) / NT;
      const int q0 = min(nkept, tid * kper), q1 = min(nkept, q0 + kper);
      long long cm = 0;
      for (int q = q0; q < q1; ++q) { const int4 r = sc.kept[q]; cm += sc.newoff[r.z & kRecIdMask] != r.x; }
      long long nmv = 0;
      long long bm = scan64(cm, S.tmp, &nmv);
      for (int q = q0; q < q1; ++q) {
        const int4 r = sc.kept[q];
        const int t = r.z & kRecIdMask;
        const int no = sc.newoff[t];
        if (no != r.x) {
          dyo_move_rec mv;
          mv.t = t;
          mv.src = (int64_t)m * a.H + (int64_t)r.x * AL;
          mv.dst = (int64_t)m * a.H + (int64_t)no * AL;
          mv.bytes = a.t_bytes[t];
          out.mv[c_mv + bm++] = mv;
          d2d += mv.bytes;
          st.off[t] = (int64_t)no * AL;
        }
      }
      if (tid == 0) s_nmove = (int)nmv;
    } else if (tid == 0) {
      s_nmove = 0;
    }
    // CARRY / ALLOC / FETCH + placed state (loc, off, dirty); carried sources tombstoned
    for (int p = tid; p < np; p += NT) {
      const int t = S.p_t[p];
      // a copy valid in the other half (CARRY source, or overwritten by an ALLOC) stops being
      // valid there (R1): its record is dropped at that half's next rebuild
      if (st.loc[t] == 1 - m) st.rl[1 - m][s_sel[1 - m]][st.pos[t]].z |= kRecTomb;
      const int64_t dst = (int64_t)m * a.H + (int64_t)S.p_off[p] * AL;
      const int c = S.p_cls[p];
      const int64_t nbytes = a.t_bytes[t];
      if (c == 0) {
        dyo_carry_rec r;
        r.t = t;
        r.src = (int64_t)(1 - m) * a.H + st.off[t];
        r.dst = dst;
        r.bytes = nbytes;
        r.late = st.pw[t] ? 1 : 0;
        out.ca[c_ca + p] = r;
        d2d += nbytes;
      } else if (c == 1) {
        dyo_alloc_rec r;
        r.t = t;
        r.dst = dst;
        r.bytes = nbytes;
        out.al[c_al + p - nc] = r;
        st.dirty[t] = 0;
      } else {
        dyo_fetch_rec r;
        r.t = t;
        r.host_off = a.t_host[t];
        r.dst = dst;
        r.bytes = nbytes;
        out.fe[c_fe + p - nc - na] = r;
        h2d += nbytes;
        st.dirty[t] = 0;
      }
      st.loc[t] = (int8_t)m;
      st.off[t] = (int64_t)S.p_off[p] * AL;
    }
    __syncthreads();
    // entry records (placement of every W_j tensor); block j writes: dirty
    if (tid < n) {
      const int t = S.e_t[tid];
      dyo_entry_rec r;
      r.t = t;
      r.mode = S.e_mode[tid];
      r.needs_fetch = S.e_rd[tid];
      r.dst = (int64_t)m * a.H + st.off[t];
      out.ent[eb + tid] = r;
      if (S.e_mode[tid] & 2) st.dirty[t] = 1;
    }
    {
      long long s4[4] = {d2d, h2d, 0, 0};
      sum4(s4, S.tmp4);
      if (tid == 0) { hd.d2d = s4[0]; hd.h2d = s4[1]; }
    }
    // previous-group written flags (late carries, R8)
    const int pn = st.prev_n[0];
    for (int i = tid; i < pn; i += NT) st.pw[st.prev[i]] = 0;
    __syncthreads();
    if (tid < n) {
      const int t = S.e_t[tid];
      st.pw[t] = (S.e_mode[tid] & 2) ? 1 : 0;
      st.prev[tid] = t;
    }
    PSTAMP(7);
    // ---- G. rebuild the half's list: kept (offset order, updated) merged with the placed
    //      tensors sorted by their new offsets
    if (tid < np) {
      const int o = S.p_off[tid];
      int r = 0;
      for (int q = 0; q < np; ++q) r += S.p_off[q] < o;
      S.q_off[r] = o;
      S.q_idx[r] = tid;
      S.q_cnt[r] = nkept;                             // default: every kept tensor is below
    }
    __syncthreads();
    const int sel_new = 1 - s_sel[m];
    int4* dst = st.rl[m][sel_new];
    {
      const int kper = (nkept + NT - 1) / NT;
      const int q0 = min(nkept, tid * kper), q1 = min(nkept, q0 + kper);
      auto lower = [&](int o) {                        // placed offsets below o
        int lo = 0, hi = np;
        while (lo < hi) { const int mid = (lo + hi) >> 1; if (S.q_off[mid] < o) lo = mid + 1; else hi = mid; }
        return lo;
      };
      int lb_prev = 0;
      if (q0 > 0 && q0 < nkept) {
        const int4 r = sc.kept[q0 - 1];
        lb_prev = lower(compact ? sc.newoff[r.z & kRecIdMask] : r.x);
      }
      for (int q = q0; q < q1; ++q) {
        int4 r = sc.kept[q];
        const int t = r.z & kRecIdMask;
        if (compact) r.x = sc.newoff[t];
        if (bit_get(inw, t)) {                         // KEEP: this occurrence updates the record
          const uint8_t fl = sc.wfl[t];
          r.w = sc.wnx[t];
          r.z = (r.z & ~kRecNxRd) | ((fl & 1) ? kRecNxRd : 0) | ((fl & 2) ? kRecDirty : 0);
        }
        const int lb = lower(r.x);
        for (int k = (q == 0 ? 0 : lb_prev); k < lb; ++k) S.q_cnt[k] = q;
        lb_prev = lb;
        dst[q + lb] = r;
        st.pos[t] = q + lb;
      }
    }
    __syncthreads();
    if (tid < np) {
      const int p = S.q_idx[tid];
      const int t = S.p_t[p];
      const uint8_t fl = sc.wfl[t];
      int4 r;
      r.x = S.p_off[p];
      r.y = S.p_a[p];
      r.z = t | ((a.t_flags[t] & 1) ? kRecTransient : 0) | ((fl & 1) ? kRecNxRd : 0) | (st.dirty[t] ? kRecDirty : 0);
      r.w = sc.wnx[t];
      dst[tid + S.q_cnt[tid]] = r;
      st.pos[t] = tid + S.q_cnt[tid];
    }
    if (tid < n) { const int t = S.e_t[tid]; atomicAnd(&inw[t >> 5], ~(1u << (t & 31))); }
    // ---- header
    if (tid == 0) {
      s_n[m] = nkept + np;
      s_sel[m] = sel_new;
      st.prev_n[0] = n;
      hd.half = m;
      hd.n_ent = n;
      hd.n_evict = nev;
      hd.n_move = s_nmove;
      hd.n_carry = nc;
      hd.n_alloc = na;
      hd.n_fetch = nf;
      hd.need = need_u * AL;
      hd.o_evict = c_ev;
      hd.o_move = c_mv;
      hd.o_carry = c_ca;
      hd.o_alloc = c_al;
      hd.o_fetch = c_fe;
      c_ev += nev;
      c_mv += s_nmove;
      c_ca += nc;
      c_al += na;
      c_fe += nf;
    }
    __syncthreads();
    PSTAMP(8);
  }
  if (tid == 0) {
    st.G[0] = G0 + Kt;
    for (int h = 0; h < 2; ++h) { st.rl_meta[h] = s_n[h]; st.rl_meta[2 + h] = s_sel[h]; }
    out.counts[0] = Kt;
    out.counts[1] = (int)c_ev;
    out.counts[2] = (int)c_mv;
    out.counts[3] = (int)c_ca;
    out.counts[4] = (int)c_al;
    out.counts[5] = (int)c_fe;
    status[0] = 0;
  }
}

cudaError_t plan_debug_stamps(int j, unsigned long long* out) {
  cudaError_t e = cudaMemcpyToSymbol(g_pstamp_j, &j, sizeof(int));
  if (e == cudaSuccess && out) e = cudaMemcpyFromSymbol(out, g_pstamp, sizeof(unsigned long long) * 64);
  return e;
}

// 8-byte words of the record arrays, grid-stride over all six lists
__global__ void plan_export_kernel(PlanOut d, PlanOut h) {
  if (d.status[0] != 0) return;
  const int K = d.counts[0];
  const int64_t n[6] = {(int64_t)K * (int64_t)(sizeof(PlanHdr) / 8), (int64_t)d.counts[1] * 5, (int64_t)d.counts[2] * 4,
                        (int64_t)d.counts[3] * 5, (int64_t)d.counts[4] * 3, (int64_t)d.counts[5] * 4};
  const uint64_t* src[6] = {reinterpret_cast<const uint64_t*>(d.hdr), reinterpret_cast<const uint64_t*>(d.ev),
                            reinterpret_cast<const uint64_t*>(d.mv), reinterpret_cast<const uint64_t*>(d.ca),
                            reinterpret_cast<const uint64_t*>(d.al), reinterpret_cast<const uint64_t*>(d.fe)};
  uint64_t* dst[6] = {reinterpret_cast<uint64_t*>(h.hdr), reinterpret_cast<uint64_t*>(h.ev),
                      reinterpret_cast<uint64_t*>(h.mv), reinterpret_cast<uint64_t*>(h.ca),
                      reinterpret_cast<uint64_t*>(h.al), reinterpret_cast<uint64_t*>(h.fe)};
  const int64_t stride = (int64_t)gridDim.x * blockDim.x;
  for (int l = 0; l < 6; ++l)
    for (int64_t i = (int64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n[l]; i += stride) dst[l][i] = src[l][i];
}

cudaError_t launch_plan_export(const PlanOut& d, const PlanOut& h, cudaStream_t s) {
  static_assert(sizeof(PlanHdr) % 8 == 0 && sizeof(dyo_evict_rec) == 40 && sizeof(dyo_move_rec) == 32 &&
                sizeof(dyo_carry_rec) == 40 && sizeof(dyo_alloc_rec) == 24 && sizeof(dyo_fetch_rec) == 32, "record layout");
  plan_export_kernel<<<64, 256, 0, s>>>(d, h);
  return cudaGetLastError();
}

cudaError_t launch_plan(const ArchDev& a, const PredDev& pd, int b0, int nb, int policy,
                        PlanState& in, PlanState& work, PlanScratch& sc, PlanOut& out,
                        int max_groups, cudaStream_t s) {
  static uint64_t attr_done = 0;                   // bit d: set on device d
  const uint64_t bit = 1ull << current_device();
  const size_t base = (sizeof(PlanSmem) + 15) / 16 * 16 + (size_t)kEvSmem * 8;
  const int inw_smem = a.T <= kInwSmemWords * 32 ? 1 : 0;
  const size_t smem = base + (inw_smem ? (size_t)kInwSmemWords * 4 : 0);
  if (!(attr_done & bit)) {
    cudaError_t e = cudaFuncSetAttribute(plan_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(base + (size_t)kInwSmemWords * 4));
    if (e != cudaSuccess) return e;
    attr_done |= bit;
  }
  if (nb > NT) return cudaErrorInvalidValue;
  plan_prep_kernel<<<1, NT, 0, s>>>(a, pd, b0, nb, sc, out, max_groups);
  const int grid = 296;
  bucket_init_kernel<<<grid, 256, 0, s>>>(a, sc);
  bucket_count_kernel<<<grid, 256, 0, s>>>(a, pd, sc);
  bucket_scan_kernel<<<1, NT, 0, s>>>(a, sc);
  bucket_fill_kernel<<<grid, 256, 0, s>>>(a, pd, sc);
  bucket_sort_kernel<<<grid * 2, 256, 0, s>>>(a, pd, sc);
  plan_kernel<<<1, NT, smem, s>>>(a, pd, policy, in, work, sc, out, inw_smem);
  return cudaGetLastError();
}

}  // namespace dyo
