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

int pdl_enabled() {
  static int v = -1;
  if (v < 0) { const char* e = getenv("DYO_PDL"); v = (e && e[0] == '0') ? 0 : 1; }
  return v;
}

constexpr int NT = kPlanThreads;                  // 1024
constexpr uint64_t kInfD = 0xFFFFull;
constexpr int kInwSmemWords = 8192;               // smem W_j bitmap for T <= 2^18

__device__ unsigned long long g_pstamp[64];
__device__ int g_pstamp_j = -1;
#define PSTAMP(i) do { if (j == pstamp_j && tid == 0) g_pstamp[i] = (unsigned long long)clock64(); } while (0)

// ---- small block primitives (1024 threads) --------------------------------------------
// Exclusive scan of one int64 per thread (any multiple of 32 threads up to 1024); *total = sum.
// tmp: 32 long longs. Three barriers.
__device__ __forceinline__ long long scan64(long long v, long long* tmp, long long* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  long long x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const long long y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  const int nw = blockDim.x >> 5;
  if (lane == 31) tmp[w] = x;
  __syncthreads();
  if (w == 0) {
    long long s = lane < nw ? tmp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const long long y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < nw) tmp[lane] = s;
  }
  __syncthreads();
  const long long base = w > 0 ? tmp[w - 1] : 0;
  *total = tmp[nw - 1];
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
  const int nw = blockDim.x >> 5;
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    long long s = 0;
    for (int i = 0; i < nw; ++i) s += tmp[i][q];
    v[q] = s;
  }
  __syncthreads();
}

__device__ __forceinline__ bool bit_get(const uint32_t* b, int t) { return (b[t >> 5] >> (t & 31)) & 1u; }

// ---- 0. group list + entry bases -------------------------------------------------------
__global__ void __launch_bounds__(NT, 1)
plan_prep_kernel(ArchDev a, PredDev pd, int b0, int nb, PlanScratch sc, PlanOut out, int max_groups) {
  pdl_enter();
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
  pdl_enter();
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
  pdl_enter();
  const int Kt = sc.Kt[0];
  for (int g = blockIdx.x; g < Kt; g += gridDim.x) {
    int n;
    const int2* ent = group_entries(a, pd, sc, g, &n);
    for (int e = threadIdx.x; e < n; e += blockDim.x) atomicAdd(&sc.bcnt[ent[e].x], 1);
  }
}

// exclusive scan of the bucket counts (one CTA, a contiguous chunk of tensors per thread)
__global__ void __launch_bounds__(NT, 1) bucket_scan_kernel(ArchDev a, PlanScratch sc) {
  pdl_enter();
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
  pdl_enter();
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
  pdl_enter();
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
// 512 threads; each holds its contiguous chunk of the half's records in registers (up to RPT)
// across the passes of a transition, so the half's list costs one coalesced global read per
// transition; larger halves re-read their chunk in RPT-record windows (same code, same order).
// Every W_j entry's per-tensor state is gathered into shared memory in one round trip (phase A)
// and everything after it that concerns W_j (placement, records, rebuild) reads shared memory.
constexpr int kPlanBig = 512;                     // planner threads (large halves)
constexpr int kPlanSmall = 128;                   // small problems: fewer warps per barrier
constexpr int RPT = 16;                           // records per thread kept in registers
constexpr int kHash = 2048;                       // W_j: tensor -> entry (open addressing)
constexpr int kGapSmem = 4096;                    // gaps in shared memory up to this
constexpr int kEvSort = 1024;                     // EVICT keys rank-sorted in shared memory up to this

struct PlanSmem {
  // W_j entries (index e < n) and their gathered state
  int32_t e_t[kEntCap];
  int32_t e_off[kEntCap];        // offset units in its half (valid when loc >= 0)
  int32_t e_pos[kEntCap];        // record index in its half's list
  int32_t e_au[kEntCap];
  int32_t e_nx[kEntCap];         // next use after this group (-1)
  int32_t e_newoff[kEntCap];     // offset units in half m after the transition
  int64_t e_host[kEntCap];
  int64_t e_bytes[kEntCap];
  int8_t e_mode[kEntCap];
  int8_t e_rd[kEntCap];
  int8_t e_cls[kEntCap];
  int8_t e_loc[kEntCap];
  uint8_t e_fl[kEntCap];         // bit 0 transient, 1 pw (written by the previous group), 2 dirty, 3 next use reads
  // placement
  alignas(16) uint64_t pkey[kEntCap];
  int32_t pidx[kEntCap];         // entry of pkey[k]
  int32_t p_e[kEntCap];          // entry of placed tensor p (placement order)
  int32_t p_off[kEntCap];
  alignas(16) int32_t p_au[kEntCap];   // aligned size of placed p (units)
  int32_t run_st[kEntCap + 1];   // starts of the runs of equal aligned size in placement order
  int32_t gcum[kGapSmem + 1];    // inclusive prefix of the gap capacities of one run
  alignas(16) int32_t q_off[kEntCap];  // placed offsets ascending (rebuild merge)
  int32_t q_idx[kEntCap];
  int32_t q_cnt[kEntCap];
  // tensor -> entry of W_j
  int32_t h_key[kHash];
  int32_t h_val[kHash];
  // previous group (late carries; pw bits to clear)
  int32_t prev_t[kEntCap];
  // gaps of half m
  int32_t gap_s[kGapSmem];
  int32_t gap_e[kGapSmem];
  // EVICT sort: key (host units, id, writeback) + payload (offset units)
  alignas(16) uint64_t ev_key[kEvSort];
  int32_t ev_off[kEvSort];
  uint32_t hist[256];
  uint32_t hcnt[256];
  long long tmp[32];
  long long tmp4[32][4];
};

// Rank of k among keys[0, n) (count of smaller keys), 16-byte shared-memory loads; keys unique.
__device__ __forceinline__ int rank_u64(const uint64_t* keys, int n, uint64_t k) {
  int r = 0, x = 0;
  const ulonglong2* k2 = reinterpret_cast<const ulonglong2*>(keys);
#pragma unroll 4
  for (; x + 1 < n; x += 2) {
    const ulonglong2 v = k2[x >> 1];
    r += (v.x < k) + (v.y < k);
  }
  if (x < n) r += keys[x] < k;
  return r;
}
__device__ __forceinline__ int rank_i32(const int32_t* keys, int n, int k) {
  int r = 0, x = 0;
  const int4* k4 = reinterpret_cast<const int4*>(keys);
#pragma unroll 4
  for (; x + 3 < n; x += 4) {
    const int4 v = k4[x >> 2];
    r += (v.x < k) + (v.y < k) + (v.z < k) + (v.w < k);
  }
  for (; x < n; ++x) r += keys[x] < k;
  return r;
}

__device__ __forceinline__ uint32_t hash_t(int t) { return ((uint32_t)t * 2654435761u) >> 21; }   // 11 bits

__device__ __forceinline__ int hash_find(const PlanSmem& S, int t) {
  uint32_t h = hash_t(t);
  while (true) {
    const int k = S.h_key[h];
    if (k == t) return S.h_val[h];
    if (k < 0) return -1;
    h = (h + 1) & (kHash - 1);
  }
}

// exclusive max-scan of one int per thread (values >= 0); *total = max. tmp: 32 long longs.
__device__ __forceinline__ int scanmax(int v, long long* tmp, int* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x = max(x, y);
  }
  const int ex_w = __shfl_up_sync(0xffffffffu, x, 1);
  if (lane == 31) tmp[w] = x;
  __syncthreads();
  if (w == 0) {
    int s = lane < nw ? (int)tmp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s = max(s, y);
    }
    if (lane < nw) tmp[lane] = s;
  }
  __syncthreads();
  const int before = w > 0 ? (int)tmp[w - 1] : 0;
  *total = (int)tmp[nw - 1];
  __syncthreads();
  return max(before, lane > 0 ? ex_w : 0);
}

__device__ __forceinline__ uint64_t live_key(int4 r, int j) {
  const uint64_t d = r.w < 0 ? kInfD : (uint64_t)(r.w - j);
  return (d << 48) | ((uint64_t)r.y << 20) | (uint64_t)(r.z & kRecIdMask);
}

// 0 skip (tombstone), 1 keep (in W_j), 2 dead, 3 live
__device__ __forceinline__ int rec_kind(int4 r, const uint32_t* inw) {
  if (r.z & kRecTomb) return 0;
  const int t = r.z & kRecIdMask;
  if (bit_get(inw, t)) return 1;
  // R9: only a transient tensor can be dead (no later access, or written first next)
  const bool dead = (r.z & kRecTransient) && (r.w < 0 || !(r.z & kRecNxRd));
  return dead ? 2 : 3;
}

__device__ __forceinline__ bool rec_evicted(int4 r, int k, int rule, uint64_t thresh, int j) {
  return k == 2 || (k == 3 && (rule == 0 || (rule == 2 && live_key(r, j) >= thresh)));
}

// Iterate this thread's records [i0, i1) in order: from registers R when the chunk fits RPT
// (one window, loaded in phase B), else in RPT-record windows re-read into R from global
// memory. BODY sees `r` and `gi`.
#define FOR_RECS(BODY)                                                                          \
  for (int w0_ = i0; w0_ < i1; w0_ += RPT) {                                                   \
    if (!regmode) {                                                                             \
      _Pragma("unroll") for (int u_ = 0; u_ < RPT; ++u_) if (w0_ + u_ < i1) R[u_] = recs[w0_ + u_]; \
    }                                                                                           \
    _Pragma("unroll") for (int u_ = 0; u_ < RPT; ++u_) if (w0_ + u_ < i1) {                     \
      const int4 r = R[u_]; const int gi = w0_ + u_; (void)gi; BODY                             \
    }                                                                                           \
  }

template <int PNT>
__global__ void __launch_bounds__(PNT, 1)
plan_kernel(ArchDev a, PredDev pd, int policy, PlanState in, PlanState st, PlanScratch sc, PlanOut out,
            int inw_smem) {
  pdl_enter();
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PlanSmem& S = *reinterpret_cast<PlanSmem*>(smem_raw);
  uint32_t* inw = inw_smem ? reinterpret_cast<uint32_t*>(smem_raw + (sizeof(PlanSmem) + 15) / 16 * 16) : sc.inw;
  const int T = a.T;
  const int64_t AL = a.align;
  const int Hu = (int)(a.H / AL);
  int* status = out.status;
  const int tid = threadIdx.x, lane = tid & 31;
  const int Kt = sc.Kt[0];
  if (Kt < 0) return;                              // prep failed (status already set)
  const int nwords = (T + 31) >> 5;

  // ---- 1. work copy of the committed state (transactional, R7), R9, next uses of the plan
  for (int t = tid; t < T; t += PNT) {
    st.loc[t] = in.loc[t];
    st.off[t] = in.off[t];
    st.dirty[t] = (a.t_flags[t] & 1) ? 0 : in.dirty[t];
    st.pw[t] = in.pw[t];
    st.pos[t] = in.pos[t];
  }
  for (int w = tid; w < nwords; w += PNT) inw[w] = 0u;
  for (int h = tid; h < kHash; h += PNT) S.h_key[h] = -1;
  __shared__ int s_n[2], s_sel[2], s_prev_n, s_prev_share;
  const bool share_on = (policy & 2) != 0;        // R20
  if (tid == 0) {
    s_prev_n = in.prev_n[0];
    s_prev_share = 0;      // a plan's last transition never SHAREs (no next group): nothing pinned at j = 0
    for (int h = 0; h < 2; ++h) { s_n[h] = in.rl_meta[h]; s_sel[h] = in.rl_meta[2 + h]; }
  }
  __syncthreads();
  for (int i = tid; i < s_prev_n; i += PNT) S.prev_t[i] = in.prev[i];
  for (int h = 0; h < 2; ++h) {
    const int4* src = in.rl[h][s_sel[h]];
    int4* dst = st.rl[h][s_sel[h]];
    for (int i = tid; i < s_n[h]; i += PNT) {
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
  __shared__ int s_np, s_compact, s_ng, s_nmove;
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
    // ---- A. W_j: gather every entry's state in one round trip; classes; need (R7, R8)
    long long v4[4] = {0, 0, 0, 0};                 // need units, carries, allocs, fetches
#pragma unroll
    for (int q = 0; q < kEntCap / PNT; ++q) {
      const int e = tid + q * PNT;
      if (e < n) {
        const int2 en = ent[e];
        const int t = en.x, md = en.y & 3, rd = (en.y >> 2) & 1;
        const int l = st.loc[t];
        const int64_t off = st.off[t];
        const int pos = st.pos[t];
        const int pw = st.pw[t], dirty = st.dirty[t], tf = a.t_flags[t];
        const int au = sc.au[t];
        const int64_t host = a.t_host[t], bytes = a.t_bytes[t];
        const int nx = sc.nxt[eb + e];
        const int nxrd = sc.nxt_rd[eb + e];
        // R20 (policy bit 2): a tensor valid in the other half that the next group also holds
        // stays there (SHARE); nx == j + 1 <=> t is in W_{j+1} of this plan
        const int c = l == m ? C_KEEP
                    : (l == 1 - m && share_on && nx == j + 1) ? C_SHARE
                    : (l == 1 - m && rd ? C_CARRY : (rd ? C_FETCH : C_ALLOC));
        S.e_t[e] = t;
        S.e_off[e] = (int)(off / AL);
        S.e_pos[e] = pos;
        S.e_au[e] = au;
        S.e_nx[e] = nx;
        S.e_newoff[e] = (int)(off / AL);
        S.e_host[e] = host;
        S.e_bytes[e] = bytes;
        S.e_mode[e] = (int8_t)md;
        S.e_rd[e] = (int8_t)rd;
        S.e_cls[e] = (int8_t)c;
        S.e_loc[e] = (int8_t)l;
        S.e_fl[e] = (uint8_t)((tf & 1) | (pw ? 2 : 0) | (dirty ? 4 : 0) | (nxrd ? 8 : 0));
        atomicOr(&inw[t >> 5], 1u << (t & 31));
        uint32_t h = hash_t(t);
        while (atomicCAS(&S.h_key[h], -1, t) != -1) h = (h + 1) & (kHash - 1);
        S.h_val[h] = e;
        v4[0] += c == C_SHARE ? 0 : au;               // a SHARE'd tensor takes no room in half m
        v4[1] += (c == C_CARRY) + ((long long)(c == C_SHARE) << 32);
        v4[2] += c == C_ALLOC;
        v4[3] += c == C_FETCH;
      }
    }
    sum4(v4, S.tmp4);
    const long long need_u = v4[0];
    const int nc = (int)(v4[1] & 0xffffffffll), na = (int)v4[2], nf = (int)v4[3];
    const int nsh = (int)(v4[1] >> 32);
    if (need_u > Hu) {
      if (tid == 0) { status[0] = DYO_E_BUDGET; status[1] = j; status[2] = 0; }
      return;
    }
    const long long room = Hu - need_u;
    PSTAMP(1);
    // ---- B. the half's records (registers), live bytes, kept / evicted counts per rule
    const int nm = s_n[m];
    const int4* recs = st.rl[m][s_sel[m]];
    const int per = (nm + PNT - 1) / PNT;
    const int i0 = min(nm, tid * per), i1 = min(nm, i0 + per);
    const bool regmode = per <= RPT;
    int4 R[RPT];
    if (regmode) {
#pragma unroll
      for (int u = 0; u < RPT; ++u)
        if (i0 + u < i1) R[u] = recs[i0 + u];
    }
    long long live_u = 0;
    {
      long long w4[4] = {0, 0, 0, 0};
      FOR_RECS(if (rec_kind(r, inw) == 3) w4[0] += r.y;)
      sum4(w4, S.tmp4);
      live_u = w4[0];
    }
    // eviction rule: 0 evict every live candidate (PAPER), 1 keep all (RETAIN, fits), 2 cut
    const int rule = (policy & 1) == 0 ? 0 : (live_u <= room ? 1 : 2);
    PSTAMP(2);
    // ---- C. RETAIN prefix cut by radix select: the smallest key K* whose prefix sum of
    //      aligned sizes (keys ascending) exceeds the room; keys >= K* are evicted
    if (rule == 2) {
      long long cnt = 0;
      FOR_RECS(cnt += rec_kind(r, inw) == 3;)
      long long nlive = 0;
      long long kb = scan64(cnt, S.tmp, &nlive);
      if (nlive <= 256) {
        // few live candidates: rank selection in shared memory (keys are unique, so the ranks
        // are a permutation): sizes in key order, one block scan, the first rank whose prefix
        // exceeds the room -> its key is the threshold (the same K* as the radix select below)
        uint64_t* keys = S.ev_key;                      // free until phase D
        uint64_t* sorted = S.pkey;                      // free until phase E
        int32_t* szs = S.gap_s;                         // free until phase D
        FOR_RECS(if (rec_kind(r, inw) == 3) keys[kb++] = live_key(r, j);)
        __syncthreads();
        const int nl = (int)nlive;
        for (int i = tid; i < nl; i += PNT) {
          const uint64_t k = keys[i];
          const int rk = rank_u64(keys, nl, k);
          sorted[rk] = k;
          szs[rk] = (int32_t)((k >> 20) & ((1u << 28) - 1));
        }
        __syncthreads();
        const int per_k = (nl + PNT - 1) / PNT;
        const int r0 = min(nl, tid * per_k), r1 = min(nl, r0 + per_k);
        long long ls = 0;
        for (int q = r0; q < r1; ++q) ls += szs[q];
        long long tot = 0;
        long long c = scan64(ls, S.tmp, &tot);
        if (c <= room)                                  // exactly one thread's chunk crosses the room
          for (int q = r0; q < r1; ++q) {
            c += szs[q];
            if (c > room) { s_thresh = sorted[q]; break; }
          }
        __syncthreads();
      } else {
      FOR_RECS(if (rec_kind(r, inw) == 3) sc.keys[kb++] = live_key(r, j);)
      __syncthreads();
      uint64_t prefix = 0, mask = 0;
      long long cum = 0;                             // units of the keys below the prefix
      const int kper = (int)((nlive + PNT - 1) / PNT);
      const int k0 = min((int)nlive, tid * kper), k1 = min((int)nlive, k0 + kper);
      for (int shift = 56; shift >= 0; shift -= 8) {
        for (int hb = tid; hb < 256; hb += PNT) { S.hist[hb] = 0; S.hcnt[hb] = 0; }
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
      for (int k = k0; k < k1; ++k) {               // the unique key under the prefix
        const uint64_t key = sc.keys[k];
        if ((key & mask) == prefix) s_thresh = key;
      }
      __syncthreads();
      }
    }
    const uint64_t thresh = rule == 2 ? s_thresh : 0;
    PSTAMP(3);
    // ---- D. EVICT keys (host offset, id, writeback) + offsets; gaps between kept tensors.
    //      Pass 1 counts kept / evicted / gaps after my first kept record (local), pass 2 writes.
    long long kbase = 0, nkept = 0;                 // this thread's first kept index; total kept
    int nev = 0;
    int pe0_keep = 0;                               // end of the kept record before my first (phase G)
    int last_x = -1;                                // old offset of this thread's last kept record
    {
      long long ck = 0, ce = 0, cg = 0;
      int first_x = -1, last_end = 0;
      FOR_RECS({
        const int k = rec_kind(r, inw);
        if (k != 0) {
          if (rec_evicted(r, k, rule, thresh, j)) {
            ++ce;
          } else {
            if (first_x < 0) first_x = r.x;
            else if (r.x > last_end) ++cg;
            ++ck;
            last_end = r.x + r.y;
            last_x = r.x;
          }
        }
      })
      int pe_all = 0;
      const int pe0 = scanmax(last_end, S.tmp, &pe_all);   // end of the kept record before my first
      pe0_keep = pe0;
      if (first_x >= 0 && first_x > pe0) ++cg;
      long long tot = 0;
      const long long b = scan64((ck << 42) | (ce << 21) | cg, S.tmp, &tot);
      constexpr long long M21 = (1ll << 21) - 1;
      kbase = b >> 42;
      long long be = (b >> 21) & M21, bg = b & M21;
      nkept = tot >> 42;
      nev = (int)((tot >> 21) & M21);
      const int ng = (int)(tot & M21);
      if (c_ev + nev > out.cap_rec) {
        if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_ev + nev); }
        return;
      }
      const bool ev_smem = nev <= kEvSort;
      const bool gap_smem = ng + 1 <= kGapSmem;
      int32_t* gs_ = gap_smem ? S.gap_s : sc.gap_s;
      int32_t* ge_ = gap_smem ? S.gap_e : sc.gap_e;
      int pe = pe0;
      FOR_RECS({
        const int k = rec_kind(r, inw);
        if (k != 0) {
          if (rec_evicted(r, k, rule, thresh, j)) {
            const int t = r.z & kRecIdMask;
            const uint64_t wb = (k == 3 && (r.z & kRecDirty)) ? 1 : 0;
            const uint64_t key = ((uint64_t)(a.t_host[t] / AL) << 21) | ((uint64_t)t << 1) | wb;
            if (ev_smem) { S.ev_key[be] = key; S.ev_off[be] = r.x; }
            else { sc.keys[be] = key; sc.newoff[t] = r.x; }
            ++be;
          } else {
            if (r.x > pe) { gs_[bg] = pe; ge_[bg] = r.x; ++bg; }
            pe = r.x + r.y;
          }
        }
      })
      if (tid == 0) {
        int ngt = ng;
        if (Hu > pe_all) { gs_[ngt] = pe_all; ge_[ngt] = Hu; ++ngt; }
        s_ng = ngt;
      }
    }
    PSTAMP(4);
    if (j == pstamp_j && tid == 0) { g_pstamp[60] = nm; g_pstamp[61] = s_ng; g_pstamp[62] = nkept; g_pstamp[63] = regmode; }
    // ---- E. placement order: CARRY by id, ALLOC by id, FETCH by (host offset, id)
    if (tid == 0) s_np = 0;
    __syncthreads();
#pragma unroll
    for (int q = 0; q < kEntCap / PNT; ++q) {
      const int e = tid + q * PNT;
      if (e < n && S.e_cls[e] != C_KEEP && S.e_cls[e] != C_SHARE) {
        const int c = S.e_cls[e], t = S.e_t[e];
        const uint64_t rank = c == C_CARRY ? 0 : (c == C_ALLOC ? 1 : 2);
        const uint64_t mid = c == C_FETCH ? (uint64_t)(S.e_host[e] / AL) : 0;
        const int k = atomicAdd(&s_np, 1);
        S.pkey[k] = (rank << 62) | (mid << 20) | (uint64_t)t;
        S.pidx[k] = e;
      }
    }
    __syncthreads();
    const int np = s_np;
#pragma unroll
    for (int q = 0; q < kEntCap / PNT; ++q) {
      const int i = tid + q * PNT;
      if (i < np) {
        const int r = rank_u64(S.pkey, np, S.pkey[i]);
        S.p_e[r] = S.pidx[i];
        S.p_au[r] = S.e_au[S.pidx[i]];
      }
    }
    __syncthreads();
    PSTAMP(5);
    // first fit (R11): a run of equal aligned sizes fills the gaps in address order (exact: each
    // tensor of the run takes the lowest gap that still holds it, and lower gaps never regain
    // room). Runs are found in parallel; each run is one block-wide pass: capacities of the gaps
    // (from a per-size cursor past the gaps an earlier run of that size filled), their prefix,
    // and every tensor of the run finds its gap by binary search.
    __shared__ int s_nruns, s_cur_sz[8], s_cur_g[8], s_last_g;
    const int ng = s_ng;
    {
      long long cst = 0;
#pragma unroll
      for (int q = 0; q < kEntCap / PNT; ++q) {
        const int p = tid * (kEntCap / PNT) + q;
        if (p < np && (p == 0 || S.p_au[p] != S.p_au[p - 1])) ++cst;
      }
      long long nr = 0;
      long long b = scan64(cst, S.tmp, &nr);
#pragma unroll
      for (int q = 0; q < kEntCap / PNT; ++q) {
        const int p = tid * (kEntCap / PNT) + q;
        if (p < np && (p == 0 || S.p_au[p] != S.p_au[p - 1])) S.run_st[b++] = p;
      }
      if (tid == 0) { s_nruns = (int)nr; S.run_st[nr] = np; s_compact = 0; }
      if (tid < 8) { s_cur_sz[tid] = 0; s_cur_g[tid] = 0; }
      __syncthreads();
    }
    {
      const bool gap_smem = ng <= kGapSmem;
      int32_t* gs_ = gap_smem ? S.gap_s : sc.gap_s;
      const int32_t* ge_ = gap_smem ? S.gap_e : sc.gap_e;
      int32_t* gcum = gap_smem ? S.gcum : reinterpret_cast<int32_t*>(sc.kept);   // scratch of >= 4T ints
      if (ng <= 64) {
        // few gaps: warp 0 alone, two lanes' worth of gaps per lane group, no block barriers;
        // the run's tensors are written by all lanes (binary search over the lanes' prefixes)
        if (tid < 32) {
          const int g_a = lane, g_b = lane + 32;
          int rem_a = g_a < ng ? gs_[g_a] : 0, rem_b = g_b < ng ? gs_[g_b] : 0;   // current gap starts
          const int end_a = g_a < ng ? ge_[g_a] : 0, end_b = g_b < ng ? ge_[g_b] : 0;
          bool fail = false;
          for (int k = 0; k < s_nruns && !fail; ++k) {
            const int i = S.run_st[k], r = S.run_st[k + 1] - i;
            const int asz = S.p_au[i];
            const int cap_a = (end_a - rem_a) / asz, cap_b = (end_b - rem_b) / asz;
            // inclusive prefix over 64 gaps: lanes 0..31 hold gaps 0..31, then 32..63
            int inc_a = cap_a, inc_b = cap_b;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
              const int ya = __shfl_up_sync(0xffffffffu, inc_a, o), yb = __shfl_up_sync(0xffffffffu, inc_b, o);
              if (lane >= o) { inc_a += ya; inc_b += yb; }
            }
            const int tot_a = __shfl_sync(0xffffffffu, inc_a, 31);
            inc_b += tot_a;
            const int tot = __shfl_sync(0xffffffffu, inc_b, 31);
            if (tot < r) { fail = true; break; }
            for (int x0 = 0; x0 < r; x0 += 32) {
              const int x = x0 + lane;
              // first gap whose inclusive prefix exceeds x (search lanes of the a half, then b)
              const bool in_a = x < tot_a;
              int pos = 0;
#pragma unroll
              for (int st2 = 16; st2 >= 1; st2 >>= 1) {
                const int va = __shfl_sync(0xffffffffu, inc_a, pos + st2 - 1);
                const int vb = __shfl_sync(0xffffffffu, inc_b, pos + st2 - 1);
                if ((in_a ? va : vb) <= x) pos += st2;
              }
              // every lane runs every shuffle (a shuffle inside a divergent ternary is undefined)
              const int ia = __shfl_sync(0xffffffffu, inc_a, pos), ib = __shfl_sync(0xffffffffu, inc_b, pos);
              const int ca = __shfl_sync(0xffffffffu, cap_a, pos), cb = __shfl_sync(0xffffffffu, cap_b, pos);
              const int ra = __shfl_sync(0xffffffffu, rem_a, pos), rb = __shfl_sync(0xffffffffu, rem_b, pos);
              const int excl = in_a ? ia - ca : ib - cb;
              const int gs0 = in_a ? ra : rb;
              if (x < r) S.p_off[i + x] = gs0 + (x - excl) * asz;
            }
            const int take_a = max(0, min(cap_a, r - (inc_a - cap_a)));
            const int take_b = max(0, min(cap_b, r - (inc_b - cap_b)));
            rem_a += take_a * asz;
            rem_b += take_b * asz;
          }
          if (lane == 0) s_compact = fail ? 1 : 0;
        }
        __syncthreads();
      } else
      for (int k = 0; k < s_nruns; ++k) {
        const int i = S.run_st[k], r = S.run_st[k + 1] - i;
        const int asz = S.p_au[i];
        int slot = -1, gstart = 0;
        for (int q = 0; q < 8; ++q)
          if (s_cur_sz[q] == asz) { slot = q; gstart = s_cur_g[q]; }
        const int span = ng - gstart;
        const int per_g = (span + PNT - 1) / PNT;
        const int g0 = gstart + min(span, tid * per_g), g1 = gstart + min(span, tid * per_g + per_g);
        long long cap_t = 0;
        for (int g = g0; g < g1; ++g) cap_t += (ge_[g] - gs_[g]) / asz;
        long long tot = 0;
        long long c = scan64(cap_t, S.tmp, &tot);
        for (int g = g0; g < g1; ++g) { c += (ge_[g] - gs_[g]) / asz; gcum[g - gstart] = (int)min(c, (long long)r); }
        if (tid == 0) s_last_g = gstart;
        __syncthreads();
        // tensor x of the run -> the first gap whose inclusive prefix exceeds x
        for (int x = tid; x < r && x < tot; x += PNT) {
          int lo = 0, hi = span - 1;
          while (lo < hi) { const int mid = (lo + hi) >> 1; if (gcum[mid] > x) hi = mid; else lo = mid + 1; }
          const int before = lo > 0 ? gcum[lo - 1] : 0;
          S.p_off[i + x] = gs_[gstart + lo] + (x - before) * asz;
        }
        __syncthreads();
        // consume the gaps' room; remember where the run ended
        for (int g = g0; g < g1; ++g) {
          const int before = g > gstart ? gcum[g - gstart - 1] : 0;
          const int take = gcum[g - gstart] - before;
          if (take > 0) { gs_[g] += take * asz; atomicMax(&s_last_g, g); }
        }
        __syncthreads();
        if (tid == 0) {
          int q = slot;
          if (q < 0) { for (q = 0; q < 8 && s_cur_sz[q] != 0; ++q) {} }
          if (q < 8) { s_cur_sz[q] = asz; s_cur_g[q] = s_last_g; }
          if (tot < r) s_compact = 1;
        }
        __syncthreads();
        if (tot < r) break;
      }
    }
    const int compact = s_compact;
    long long d2d = 0, h2d = 0, d2h = 0;
    int nmove = 0;
    if (compact) {
      // exclusive prefix sums over [kept in offset order | placed in placement order]; MOVE
      // records for the kept tensors whose offset changes (ascending destination)
      long long cu = 0;
      FOR_RECS({ const int k = rec_kind(r, inw); if (k != 0 && !rec_evicted(r, k, rule, thresh, j)) cu += r.y; })
      long long tot = 0;
      long long base = scan64(cu, S.tmp, &tot);
      long long cm = 0;
      {
        long long b2 = base;
        FOR_RECS({
          const int k = rec_kind(r, inw);
          if (k != 0 && !rec_evicted(r, k, rule, thresh, j)) { cm += b2 != r.x; b2 += r.y; }
        })
      }
      long long nmv = 0;
      long long bm = scan64(cm, S.tmp, &nmv);
      if (c_mv + nmv > out.cap_rec) {
        if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_mv + nmv); }
        return;
      }
      FOR_RECS({
        const int k = rec_kind(r, inw);
        if (k != 0 && !rec_evicted(r, k, rule, thresh, j)) {
          const int t = r.z & kRecIdMask;
          const int no = (int)base;
          if (k == 1) S.e_newoff[hash_find(S, t)] = no;
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
          base += r.y;
        }
      })
      nmove = (int)nmv;
      {
        // placed tensors after the kept run: exclusive prefix sums of their aligned sizes
        // (contiguous placements per thread, one block scan)
        constexpr int PP = kEntCap / PNT;
        const int p0 = tid * PP;
        long long ls = 0;
#pragma unroll
        for (int q = 0; q < PP; ++q) if (p0 + q < np) ls += S.p_au[p0 + q];
        long long ptot = 0;
        long long c = tot + scan64(ls, S.tmp, &ptot);
#pragma unroll
        for (int q = 0; q < PP; ++q) if (p0 + q < np) { S.p_off[p0 + q] = (int)c; c += S.p_au[p0 + q]; }
      }
      __syncthreads();
    }
    if (tid == 0) s_nmove = nmove;
    PSTAMP(6);
    // ---- F. records
    if (c_ca + nc > out.cap_rec || c_al + na > out.cap_rec || c_fe + nf > out.cap_rec) {
      if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = 0; }
      return;
    }
    // EVICT, sorted by (host offset, id)
    if (nev <= kEvSort) {
      uint64_t kk[kEvSort / PNT];
      int ofs[kEvSort / PNT], rk[kEvSort / PNT];
#pragma unroll
      for (int q = 0; q < kEvSort / PNT; ++q) {
        const int i = tid + q * PNT;
        rk[q] = -1;
        if (i < nev) {
          kk[q] = S.ev_key[i];
          ofs[q] = S.ev_off[i];
          rk[q] = rank_u64(S.ev_key, nev, kk[q]);
        }
      }
      __syncthreads();
#pragma unroll
      for (int q = 0; q < kEvSort / PNT; ++q)
        if (rk[q] >= 0) { S.ev_key[rk[q]] = kk[q]; S.ev_off[rk[q]] = ofs[q]; }
      __syncthreads();
    } else {
      block_sort_u64(sc.keys, nev);                 // bitonic in global memory (large evictions)
    }
    for (int k = tid; k < nev; k += PNT) {
      const uint64_t key = nev <= kEvSort ? S.ev_key[k] : sc.keys[k];
      const int t = (int)((key >> 1) & kRecIdMask);
      const int wb = (int)(key & 1);
      const int ou = nev <= kEvSort ? S.ev_off[k] : sc.newoff[t];
      dyo_evict_rec r;
      r.t = t;
      r.src = (int64_t)m * a.H + (int64_t)ou * AL;
      r.host_off = (int64_t)(key >> 21) * AL;
      r.bytes = a.t_bytes[t];
      r.writeback = wb;
      out.ev[c_ev + k] = r;
      if (wb) d2h += r.bytes;
      st.loc[t] = -1;
      st.dirty[t] = 0;
    }
    // CARRY / ALLOC / FETCH + placed state (loc, off, dirty); a copy valid in the other half
    // (CARRY source, or overwritten by an ALLOC) stops being valid there (R1): its record is
    // tombstoned and dropped at that half's next rebuild
    for (int p = tid; p < np; p += PNT) {
      const int e = S.p_e[p];
      const int t = S.e_t[e];
      const int c = S.e_cls[e];
      const int64_t dst = (int64_t)m * a.H + (int64_t)S.p_off[p] * AL;
      const int64_t nbytes = S.e_bytes[e];
      if (S.e_loc[e] == 1 - m) atomicOr(&st.rl[1 - m][s_sel[1 - m]][S.e_pos[e]].z, kRecTomb);
      if (c == C_CARRY) {
        dyo_carry_rec r;
        r.t = t;
        r.src = (int64_t)(1 - m) * a.H + (int64_t)S.e_off[e] * AL;
        r.dst = dst;
        r.bytes = nbytes;
        r.late = (S.e_fl[e] & 2) ? 1 : 0;
        out.ca[c_ca + p] = r;
        d2d += nbytes;
      } else if (c == C_ALLOC) {
        dyo_alloc_rec r;
        r.t = t;
        r.dst = dst;
        r.bytes = nbytes;
        out.al[c_al + p - nc] = r;
      } else {
        dyo_fetch_rec r;
        r.t = t;
        r.host_off = S.e_host[e];
        r.dst = dst;
        r.bytes = nbytes;
        out.fe[c_fe + p - nc - na] = r;
        h2d += nbytes;
      }
      S.e_newoff[e] = S.p_off[p];
      st.loc[t] = (int8_t)m;
      st.off[t] = (int64_t)S.p_off[p] * AL;
    }
    __syncthreads();
    // entry records (placement of every W_j tensor); dirty after block j (writes); pw flags
    for (int i = tid; i < s_prev_n; i += PNT) st.pw[S.prev_t[i]] = 0;
    {
      long long s4[4] = {d2d, h2d, d2h, 0};
      sum4(s4, S.tmp4);                             // (its barriers also order the pw clears)
      if (tid == 0) { hd.d2d = s4[0]; hd.h2d = s4[1]; hd.d2h = s4[2]; }
    }
#pragma unroll
    for (int q = 0; q < kEntCap / PNT; ++q) {
      const int e = tid + q * PNT;
      if (e < n) {
        const int t = S.e_t[e];
        dyo_entry_rec r;
        r.t = t;
        r.mode = S.e_mode[e];
        r.needs_fetch = S.e_rd[e];
        r.dst = (int64_t)(S.e_cls[e] == C_SHARE ? 1 - m : m) * a.H + (int64_t)S.e_newoff[e] * AL;
        out.ent[eb + e] = r;
        const int wr = (S.e_mode[e] & 2) ? 1 : 0;
        // dirty: CARRY/KEEP keep theirs, ALLOC/FETCH start clean; block j's writes set it
        const int dirty = wr || ((S.e_cls[e] == C_KEEP || S.e_cls[e] == C_CARRY || S.e_cls[e] == C_SHARE) && (S.e_fl[e] & 4));
        st.dirty[t] = (uint8_t)dirty;
        S.e_fl[e] = (uint8_t)((S.e_fl[e] & ~4) | (dirty ? 4 : 0));
        st.pw[t] = (uint8_t)wr;
        S.prev_t[e] = t;
      }
    }
    PSTAMP(7);
    // ---- G. rebuild the half's list: kept (offset order, updated) merged with the placed
    //      tensors sorted by their new offsets
#pragma unroll
    for (int q = 0; q < kEntCap / PNT; ++q) {
      const int i = tid + q * PNT;
      if (i < np) {
        const int o = S.p_off[i];
        const int r = rank_i32(S.p_off, np, o);
        S.q_off[r] = o;
        S.q_idx[r] = i;
        S.q_cnt[r] = (int)nkept;                   // default: every kept tensor is below
      }
    }
    __syncthreads();
    const int sel_new = 1 - s_sel[m];
    int4* dst = st.rl[m][sel_new];
    {
      auto lower = [&](int o) {                      // placed offsets below o
        int lo = 0, hi = np;
        while (lo < hi) { const int mid = (lo + hi) >> 1; if (S.q_off[mid] < o) lo = mid + 1; else hi = mid; }
        return lo;
      };
      long long q = kbase;                           // global kept index
      int newx0 = 0;                                 // compaction: new offset of my first kept
      if (compact) {
        long long cu = 0;
        FOR_RECS({ const int k = rec_kind(r, inw); if (k != 0 && !rec_evicted(r, k, rule, thresh, j)) cu += r.y; })
        long long tot = 0;
        newx0 = (int)scan64(cu, S.tmp, &tot);
      }
      // merge (one pass, no per-record search): a kept record's slot = its kept index + the placed
      // offsets below it; a placed tensor's slot = its rank + the kept records below it. No placed
      // offset lies inside a kept range, so a thread's pointer into the ascending placed offsets
      // starts below its first kept record (one binary search from the end of the previous kept
      // record, pe0) and advances linearly: the placed tensors it passes get this record's kept
      // index. Placed tensors above the last kept record keep the default nkept; after a
      // compaction every placed tensor lies above every kept one.
      int ptr = compact ? 0 : lower(pe0_keep);
      int newx = newx0;
      FOR_RECS({
        const int k = rec_kind(r, inw);
        if (k != 0 && !rec_evicted(r, k, rule, thresh, j)) {
          int4 w = r;
          const int t = r.z & kRecIdMask;
          if (compact) { w.x = newx; newx += r.y; }
          if (k == 1) {                              // KEEP: this occurrence updates the record
            const int e = hash_find(S, t);
            w.w = S.e_nx[e];
            w.z = (r.z & ~(kRecNxRd | kRecDirty)) | ((S.e_fl[e] & 8) ? kRecNxRd : 0) | ((S.e_fl[e] & 4) ? kRecDirty : 0);
          }
          if (!compact)
            while (ptr < np && S.q_off[ptr] < w.x) { S.q_cnt[ptr] = (int)q; ++ptr; }
          const int lb = compact ? 0 : ptr;
          dst[q + lb] = w;
          st.pos[t] = (int)(q + lb);
          ++q;
        }
      })
    }
    __syncthreads();
#pragma unroll
    for (int qq = 0; qq < kEntCap / PNT; ++qq) {
      const int i = tid + qq * PNT;
      if (i < np) {
        const int p = S.q_idx[i];
        const int e = S.p_e[p];
        const int t = S.e_t[e];
        const uint8_t fl = S.e_fl[e];
        int4 r;
        r.x = S.p_off[p];
        r.y = S.e_au[e];
        r.z = t | ((fl & 1) ? kRecTransient : 0) | ((fl & 8) ? kRecNxRd : 0) | ((fl & 4) ? kRecDirty : 0);
        r.w = S.e_nx[e];
        dst[i + S.q_cnt[i]] = r;
        st.pos[t] = i + S.q_cnt[i];
      }
    }
#pragma unroll
    for (int q = 0; q < kEntCap / PNT; ++q) {
      const int e = tid + q * PNT;
      if (e < n) { const int t = S.e_t[e]; atomicAnd(&inw[t >> 5], ~(1u << (t & 31))); }
    }
    for (int h = tid; h < kHash; h += PNT) S.h_key[h] = -1;
    // ---- header
    if (tid == 0) {
      s_n[m] = (int)nkept + np;
      s_sel[m] = sel_new;
      s_prev_n = n;
      hd.half = m;
      hd.n_ent = n;
      hd.n_evict = nev;
      hd.n_move = s_nmove;
      hd.n_carry = nc;
      hd.n_alloc = na;
      hd.n_fetch = nf;
      // R20: a compaction of a half holding tensors the running block j-1 SHARE'd waits for its end
      hd.flags = (compact && s_prev_share > 0 ? 1 : 0) | (nsh << 1);
      s_prev_share = nsh;
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
  for (int i = tid; i < s_prev_n; i += PNT) st.prev[i] = S.prev_t[i];
  if (tid == 0) {
    st.prev_n[0] = s_prev_n;
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

// ---- fault injection (DYO_FAULT=drop_prefetch:p[:seed], R17 tests and measurement) ------
// Drops every read-first entry of the predictions' tensor sets whose splitmix64 hash of
// (seed, b, k, t) is below lim (workloads.drop_prefetch is the test side's twin), keeping the
// others in order: the plan then misses those tensors and the runtime faults them in.
__device__ __forceinline__ uint64_t drop_hash(uint64_t seed, uint64_t b, uint64_t k, uint64_t t) {
  uint64_t z = seed * 0x9E3779B97F4A7C15ull + (b << 40) + (k << 20) + t;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

__global__ void fault_drop_kernel(ArchDev a, PredDev pd, int b0, int nb, uint64_t lim, int all, uint64_t seed) {
  __shared__ int warp_tmp[32];
  for (int item = blockIdx.x; item < nb * a.K_max; item += gridDim.x) {
    const int b = b0 + item / a.K_max, k = item % a.K_max;
    if (k >= pd.K[b]) continue;
    int2* ent = pd.ent + ((int64_t)b * a.K_max + k) * kEntCap;
    const int n = pd.ent_n[(int64_t)b * a.K_max + k];
    int base = 0;
    for (int i0 = 0; i0 < n; i0 += blockDim.x) {
      const int i = i0 + threadIdx.x;
      int2 e = make_int2(0, 0);
      int keep = 0;
      if (i < n) {
        e = ent[i];
        const bool rd = (e.y >> 2) & 1;
        keep = !(rd && (all || drop_hash(seed, (uint64_t)b, (uint64_t)k, (uint64_t)e.x) < lim));
      }
      int tot = 0;
      const int p = block_scan(keep, warp_tmp, &tot);   // barriers: every read precedes the writes
      if (keep) ent[base + p] = e;
      base += tot;
      __syncthreads();
    }
    if (threadIdx.x == 0) pd.ent_n[(int64_t)b * a.K_max + k] = base;
    __syncthreads();
  }
}

cudaError_t launch_fault_drop(const ArchDev& a, const PredDev& pd, int b0, int nb, double p, uint64_t seed,
                              cudaStream_t s) {
  const int all = p >= 1.0 ? 1 : 0;
  const uint64_t lim = all ? 0 : (uint64_t)(p * 18446744073709551616.0);
  fault_drop_kernel<<<148, 256, 0, s>>>(a, pd, b0, nb, lim, all, seed);
  return cudaGetLastError();
}

// 8-byte words of the record arrays, grid-stride over all six lists
__global__ void plan_export_kernel(PlanOut d, PlanOut h) {
  pdl_enter();
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
  cudaError_t le = launch_pdl(plan_export_kernel, dim3(64), dim3(256), 0, s, d, h);
  if (le != cudaSuccess) return le;
  return cudaGetLastError();
}

cudaError_t launch_plan(const ArchDev& a, const PredDev& pd, int b0, int nb, int policy,
                        PlanState& in, PlanState& work, PlanScratch& sc, PlanOut& out,
                        int max_groups, cudaStream_t s) {
  static uint64_t attr_done = 0;                   // bit d: set on device d
  const uint64_t bit = 1ull << current_device();
  const size_t base = (sizeof(PlanSmem) + 15) / 16 * 16;
  const int inw_smem = a.T <= kInwSmemWords * 32 ? 1 : 0;
  const size_t smem = base + (inw_smem ? (size_t)kInwSmemWords * 4 : 0);
  if (!(attr_done & bit)) {
    cudaError_t e = cudaFuncSetAttribute(plan_kernel<kPlanBig>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                                         (int)(base + (size_t)kInwSmemWords * 4));
    if (e != cudaSuccess) return e;
    e = cudaFuncSetAttribute(plan_kernel<kPlanSmall>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)(base + (size_t)kInwSmemWords * 4));
    if (e != cudaSuccess) return e;
    attr_done |= bit;
  }
  // DYO_PLAN_THREADS=128: the 4-warp planner (measured slower than 512 threads even on the small
  // MoE / AF halves - 0.56 vs 0.47 ms, 3.2 vs 2.7 ms per plan - the per-transition latency is
  // the threads' serial work between barriers, not the barriers; kept as a tested variant)
  static int forced = -1;
  if (forced < 0) { const char* e = getenv("DYO_PLAN_THREADS"); forced = e ? atoi(e) : 0; }
  const bool small = forced == 128 && a.T <= kPlanSmall * 16 * 64;
  if (nb > NT) return cudaErrorInvalidValue;
  cudaError_t le = launch_pdl(plan_prep_kernel, dim3(1), dim3(NT), 0, s, a, pd, b0, nb, sc, out, max_groups);
  if (le != cudaSuccess) return le;
  const int grid = 296;
  if ((le = launch_pdl(bucket_init_kernel, dim3(grid), dim3(256), 0, s, a, sc)) != cudaSuccess) return le;
  if ((le = launch_pdl(bucket_count_kernel, dim3(grid), dim3(256), 0, s, a, pd, sc)) != cudaSuccess) return le;
  if ((le = launch_pdl(bucket_scan_kernel, dim3(1), dim3(NT), 0, s, a, sc)) != cudaSuccess) return le;
  if ((le = launch_pdl(bucket_fill_kernel, dim3(grid), dim3(256), 0, s, a, pd, sc)) != cudaSuccess) return le;
  if ((le = launch_pdl(bucket_sort_kernel, dim3(grid * 2), dim3(256), 0, s, a, pd, sc)) != cudaSuccess) return le;
  if (small)
    le = launch_pdl(plan_kernel<kPlanSmall>, dim3(1), dim3(kPlanSmall), smem, s, a, pd, policy, in, work, sc, out, inw_smem);
  else
    le = launch_pdl(plan_kernel<kPlanBig>, dim3(1), dim3(kPlanBig), smem, s, a, pd, policy, in, work, sc, out, inw_smem);
  if (le != cudaSuccess) return le;
  return cudaGetLastError();
}

}  // namespace dyo
