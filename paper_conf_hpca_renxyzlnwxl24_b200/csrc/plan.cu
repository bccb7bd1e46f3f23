// K2: the double-buffered evict/prefetch planner (§IV-E, §V;
// DESIGN.md R7-R12). One CTA, integer-only, deterministic (every ordering decision is a sort
// on a unique 64-bit key; atomics only count), so it is bit-exact with oracle/plan.py.
//
// Per plan: copy the committed state to a work copy (transactional, R7), clear transient dirty
// bits (R9), one reverse sweep over the groups gives every entry its next occurrence. Then per
// transition j (sequential; parallel inside):
//   classify W_j (KEEP / CARRY / ALLOC / FETCH, R8) -> scan the resident list of half m for
//   eviction candidates (dead, R9, or live with next-use distance) -> RETAIN keeps the longest
//   prefix of candidates sorted by (distance, aligned size, id) that fits H - need (block
//   bitonic sort + scan: the north_star's "prefix sums and top-k over tensor sizes and predicted
//   reuse distance") -> first-fit placement into the gaps by one warp with ballots, or the
//   compacted layout by exclusive scan (R11) -> records + state update.
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdlib>

#include "dyo_device.cuh"
#include "dyo_internal.h"

namespace dyo {

constexpr int kSortCap = 4096;      // shared-memory sort capacity (larger sorts use global scratch)
constexpr uint64_t kInfD = 0xFFFFull;

__device__ unsigned long long g_pstamp[64];
__device__ int g_pstamp_j = -1;
#define PSTAMP(i) do { if (j == pstamp_j && tid == 0) g_pstamp[i] = (unsigned long long)clock64(); } while (0)

enum RStat : int8_t { RS_NONE = 0, RS_KEEP = 1, RS_LIVE = 2, RS_DEAD = 3, RS_EVICT = 4, RS_RETAIN = 5 };

struct PlanSmem {
  int32_t e_t[kEntCap];
  int8_t e_mode[kEntCap];
  int8_t e_rd[kEntCap];
  int8_t e_cls[kEntCap];
  int64_t e_new[kEntCap];
  uint64_t sortbuf[kSortCap];
  int warp_tmp[32];
  long long sum_tmp[32];
};

__device__ __forceinline__ void sort_keys(uint64_t* key, int n) {
  if (n <= 64) {
    // one warp, registers + shuffles (a block bitonic stage costs a barrier + smem round trip)
    if (threadIdx.x < 32) {
      const int lane = threadIdx.x;
      uint64_t x = lane < n ? key[lane] : ~0ull;
      uint64_t z = lane + 32 < n ? key[lane + 32] : ~0ull;
      warp_sort64(x, z, lane);
      if (lane < n) key[lane] = x;
      if (lane + 32 < n) key[lane + 32] = z;
    }
    __syncthreads();
    return;
  }
  int np2 = 1;
  while (np2 < n) np2 <<= 1;
  for (int i = n + threadIdx.x; i < np2; i += blockDim.x) key[i] = ~0ull;
  __syncthreads();
  for (int k = 2; k <= np2; k <<= 1) {
    for (int j = k >> 1; j > 0; j >>= 1) {
      for (int i = threadIdx.x; i < np2; i += blockDim.x) {
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

__global__ void __launch_bounds__(kPlanThreads, 1)
plan_kernel(ArchDev a, PredDev pd, int b0, int nb, int policy, PlanState in, PlanState stg,
            PlanScratch scg, PlanOut out, int max_groups, int smem_state) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PlanSmem& S = *reinterpret_cast<PlanSmem*>(smem_raw);
  const int T = a.T;
  const int64_t H = a.H, AL = a.align;
  int* status = out.status;
  const int tid = threadIdx.x, NT = blockDim.x;

  // Per-tensor working state and constants: in shared memory when they fit (smem_state), so
  // the many dependent per-transition lookups cost ~30 cycles instead of an L2 round trip.
  PlanState st = stg;
  PlanScratch sc = scg;
  const int64_t* t_ab = a.t_abytes;
  const int64_t* t_host = a.t_host;
  const int64_t* t_by = a.t_bytes;
  const int32_t* t_fl = a.t_flags;
  if (smem_state) {
    unsigned char* q = smem_raw + ((sizeof(PlanSmem) + 15) / 16 * 16);
    auto carve = [&](size_t bytes) { unsigned char* r = q; q += (bytes + 15) / 16 * 16; return r; };
    st.off = reinterpret_cast<int64_t*>(carve(8 * (size_t)T));
    sc.gap_s = reinterpret_cast<int64_t*>(carve(8 * (size_t)(T + 1)));
    sc.gap_e = reinterpret_cast<int64_t*>(carve(8 * (size_t)(T + 1)));
    sc.newoff = reinterpret_cast<int64_t*>(carve(8 * (size_t)T));
    int64_t* ab = reinterpret_cast<int64_t*>(carve(8 * (size_t)T));
    int64_t* ho = reinterpret_cast<int64_t*>(carve(8 * (size_t)T));
    int64_t* by = reinterpret_cast<int64_t*>(carve(8 * (size_t)T));
    st.res = reinterpret_cast<int32_t*>(carve(8 * (size_t)T));
    st.prev = reinterpret_cast<int32_t*>(carve(4 * (size_t)T));
    sc.cur_next = reinterpret_cast<int32_t*>(carve(4 * (size_t)T));
    sc.kept = reinterpret_cast<int32_t*>(carve(4 * (size_t)T));
    int32_t* fl = reinterpret_cast<int32_t*>(carve(4 * (size_t)T));
    st.res_n = reinterpret_cast<int32_t*>(carve(16));
    st.prev_n = reinterpret_cast<int32_t*>(carve(16));
    st.G = reinterpret_cast<int64_t*>(carve(16));
    st.loc = reinterpret_cast<int8_t*>(carve(T));
    st.dirty = reinterpret_cast<uint8_t*>(carve(T));
    st.pw = reinterpret_cast<uint8_t*>(carve(T));
    sc.cur_rd = reinterpret_cast<uint8_t*>(carve(T));
    sc.inw = reinterpret_cast<int8_t*>(carve(T));
    sc.rstat = reinterpret_cast<int8_t*>(carve(T));
    for (int t = tid; t < T; t += NT) {
      ab[t] = a.t_abytes[t];
      ho[t] = a.t_host[t];
      by[t] = a.t_bytes[t];
      fl[t] = a.t_flags[t];
    }
    t_ab = ab;
    t_host = ho;
    t_by = by;
    t_fl = fl;
  }

  // ---- 0. decode status, group list ----
  __shared__ int s_Kt, s_fail;
  if (tid == 0) {
    s_fail = 0;
    if (pd.status[0] != 0) {
      status[0] = pd.status[0];
      status[2] = pd.status[1];
      s_fail = 1;
    } else {
      int Kt = 0;
      for (int b = b0; b < b0 + nb; ++b) {
        for (int k = 0; k < pd.K[b]; ++k) {
          if (Kt < max_groups) { sc.grp_b[Kt] = b; sc.grp_k[Kt] = k; }
          ++Kt;
        }
      }
      if (Kt > max_groups) { status[0] = DYO_E_CAPACITY; status[2] = Kt; s_fail = 1; }
      s_Kt = Kt;
    }
  }
  __syncthreads();
  if (s_fail) return;
  const int Kt = s_Kt;

  // ---- 1. work copy of the committed state (transactional), R9 ----
  for (int t = tid; t < T; t += NT) {
    st.loc[t] = in.loc[t];
    st.off[t] = in.off[t];
    st.dirty[t] = (t_fl[t] & 1) ? 0 : in.dirty[t];
    st.pw[t] = in.pw[t];
    st.res[t] = in.res[t];
    st.res[T + t] = in.res[T + t];
    st.prev[t] = in.prev[t];
    sc.inw[t] = 0;
    sc.cur_next[t] = -1;
    sc.cur_rd[t] = 0;
    sc.rstat[t] = RS_NONE;
  }
  if (tid == 0) {
    st.res_n[0] = in.res_n[0];
    st.res_n[1] = in.res_n[1];
    st.prev_n[0] = in.prev_n[0];
    st.G[0] = in.G[0];
  }
  __syncthreads();
  // entry base offsets of the planned groups (prefix over their entry counts)
  if (tid == 0) {
    int64_t c = 0;
    for (int g = 0; g < Kt; ++g) {
      sc.ebase[g] = c;
      out.hdr[g].o_ent = c;
      c += pd.ent_n[sc.grp_b[g] * a.K_max + sc.grp_k[g]];
    }
    if (c > out.cap_ent) { status[0] = DYO_E_CAPACITY; status[2] = (int)c; s_fail = 1; }
  }
  __syncthreads();
  if (s_fail) return;

  // ---- 2. reverse sweep: next occurrence of every entry ----
  for (int g = Kt - 1; g >= 0; --g) {
    const int2* ent = pd.ent + ((int64_t)sc.grp_b[g] * a.K_max + sc.grp_k[g]) * kEntCap;
    const int n = pd.ent_n[sc.grp_b[g] * a.K_max + sc.grp_k[g]];
    const int64_t base = sc.ebase[g];
    for (int e = tid; e < n; e += NT) {
      const int t = ent[e].x;
      sc.nxt[base + e] = sc.cur_next[t];
      sc.nxt_rd[base + e] = sc.cur_rd[t];
    }
    __syncthreads();
    for (int e = tid; e < n; e += NT) {
      const int t = ent[e].x;
      sc.cur_next[t] = g;
      sc.cur_rd[t] = (uint8_t)((ent[e].y >> 2) & 1);
    }
    __syncthreads();
  }

  // running record counters
  __shared__ int64_t c_ev, c_mv, c_ca, c_al, c_fe;
  if (tid == 0) { c_ev = c_mv = c_ca = c_al = c_fe = 0; }
  __syncthreads();

  const int pstamp_j = g_pstamp_j;
  for (int j = 0; j < Kt; ++j) {
    PSTAMP(0);
    const int64_t Gj = st.G[0] + j;
    const int m = (int)(Gj & 1);
    const int2* ent = pd.ent + ((int64_t)sc.grp_b[j] * a.K_max + sc.grp_k[j]) * kEntCap;
    const int n = pd.ent_n[sc.grp_b[j] * a.K_max + sc.grp_k[j]];
    PlanHdr& hd = out.hdr[j];
    __shared__ unsigned long long s_need, s_livebytes, s_h2d, s_d2h, s_d2d;
    __shared__ int s_nlive, s_nev, s_nkept, s_nplaced, s_ng, s_nc, s_na, s_nf, s_compact, s_nmove;
    if (tid == 0) {
      s_need = s_livebytes = s_h2d = s_d2h = s_d2d = 0;
      s_nlive = s_nev = s_nc = s_na = s_nf = 0;
      s_compact = 0;
    }
    __syncthreads();
    // A. load W_j; need
    long long my_need = 0;
    for (int e = tid; e < n; e += NT) {
      const int t = ent[e].x;
      S.e_t[e] = t;
      S.e_mode[e] = (int8_t)(ent[e].y & 3);
      S.e_rd[e] = (int8_t)((ent[e].y >> 2) & 1);
      my_need += t_ab[t];
    }
    {
      const long long tot = block_sum64(my_need, S.sum_tmp);
      if (tid == 0) s_need = (unsigned long long)tot;
    }
    __syncthreads();
    PSTAMP(1);
    // B. feasibility (R7)
    if ((int64_t)s_need > H) {
      if (tid == 0) { status[0] = DYO_E_BUDGET; status[1] = j; status[2] = 0; }
      return;
    }
    PSTAMP(2);
    // C. classify (R8)
    for (int e = tid; e < n; e += NT) {
      const int t = S.e_t[e];
      const int l = st.loc[t];
      int8_t c;
      if (l == m) c = C_KEEP;
      else if (l == 1 - m && S.e_rd[e]) c = C_CARRY;
      else if (S.e_rd[e]) c = C_FETCH;
      else c = C_ALLOC;
      S.e_cls[e] = c;
      sc.inw[t] = 1;
      if (c == C_CARRY) atomicAdd(&s_nc, 1);
      else if (c == C_ALLOC) atomicAdd(&s_na, 1);
      else if (c == C_FETCH) atomicAdd(&s_nf, 1);
    }
    __syncthreads();
    PSTAMP(3);
    // D. candidates of half m: dead (R9) or live with next-use distance
    const int nm = st.res_n[m];
    const int32_t* resm = st.res + (int64_t)m * T;
    const bool big = nm > kSortCap;
    uint64_t* keys = big ? sc.keys : S.sortbuf;
    long long my_live = 0;
    for (int i = tid; i < nm; i += NT) {
      const int t = resm[i];
      if (sc.inw[t]) { sc.rstat[t] = RS_KEEP; continue; }
      const int nx = sc.cur_next[t];
      const bool dead = (nx < 0 && (t_fl[t] & 1)) || (nx >= 0 && !sc.cur_rd[t]);
      if (dead) { sc.rstat[t] = RS_DEAD; continue; }
      sc.rstat[t] = RS_LIVE;
      const uint64_t d = nx < 0 ? kInfD : (uint64_t)(nx - j);
      const int k = atomicAdd(&s_nlive, 1);
      keys[k] = (d << 48) | ((uint64_t)(t_ab[t] / AL) << 20) | (uint64_t)t;
      my_live += t_ab[t];
    }
    {
      const long long tot = block_sum64(my_live, S.sum_tmp);
      if (tid == 0) s_livebytes = (unsigned long long)tot;
    }
    __syncthreads();
    PSTAMP(4);
    // E. retention (R10)
    const int64_t room = H - (int64_t)s_need;
    const int nlive = s_nlive;
    if (policy == 0 || (int64_t)s_livebytes > room) {
      if (policy == 1) {
        sort_keys(keys, nlive);
        if (tid == 0) {
          int64_t used = 0;
          int k = 0;
          for (; k < nlive; ++k) {
            const int64_t ab = (int64_t)((keys[k] >> 20) & ((1ull << 28) - 1)) * AL;
            if (used + ab > room) break;
            used += ab;
            sc.rstat[(int)(keys[k] & 0xFFFFF)] = RS_RETAIN;
          }
          for (; k < nlive; ++k) sc.rstat[(int)(keys[k] & 0xFFFFF)] = RS_EVICT;
        }
      } else {
        for (int k = tid; k < nlive; k += NT) sc.rstat[(int)(keys[k] & 0xFFFFF)] = RS_EVICT;
      }
    } else {
      for (int k = tid; k < nlive; k += NT) sc.rstat[(int)(keys[k] & 0xFFFFF)] = RS_RETAIN;
    }
    __syncthreads();
    PSTAMP(5);
    // F. EVICT records sorted by (host offset, id)
    for (int i = tid; i < nm; i += NT) {
      const int t = resm[i];
      const int8_t r = sc.rstat[t];
      if (r == RS_DEAD || r == RS_EVICT) {
        const int k = atomicAdd(&s_nev, 1);
        keys[k] = ((uint64_t)(t_host[t] / AL) << 20) | (uint64_t)t;
      }
    }
    __syncthreads();
    const int nev = s_nev;
    if (c_ev + nev > out.cap_rec) {
      if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_ev + nev); }
      return;
    }
    sort_keys(keys, nev);
    long long my_d2h = 0;
    for (int k = tid; k < nev; k += NT) {
      const int t = (int)(keys[k] & 0xFFFFF);
      const bool wb = sc.rstat[t] == RS_EVICT && st.dirty[t];
      dyo_evict_rec r;
      r.t = t;
      r.src = (int64_t)m * H + st.off[t];
      r.host_off = t_host[t];
      r.bytes = t_by[t];
      r.writeback = wb ? 1 : 0;
      out.ev[c_ev + k] = r;
      if (wb) my_d2h += t_by[t];
    }
    {
      const long long tot = block_sum64(my_d2h, S.sum_tmp);
      if (tid == 0) s_d2h = (unsigned long long)tot;
    }
    __syncthreads();
    PSTAMP(6);
    // G. kept list in ascending old offset (order-preserving compaction of the resident list)
    {
      int total = 0, base = 0;
      for (int i0 = 0; i0 < nm; i0 += NT) {
        const int i = i0 + tid;
        int f = 0;
        if (i < nm) { const int8_t r = sc.rstat[resm[i]]; f = (r == RS_KEEP || r == RS_RETAIN); }
        const int p = block_scan(f, S.warp_tmp, &total);
        if (f) sc.kept[base + p] = resm[i];
        base += total;
        __syncthreads();
      }
      if (tid == 0) s_nkept = base;
      __syncthreads();
    }
    const int nkept = s_nkept;
    PSTAMP(7);
    // H. gaps of half m between kept tensors
    {
      int total = 0, base = 0;
      for (int i0 = 0; i0 <= nkept; i0 += NT) {
        const int i = i0 + tid;
        int f = 0;
        int64_t gs = 0, ge = 0;
        if (i <= nkept) {
          gs = i == 0 ? 0 : st.off[sc.kept[i - 1]] + t_ab[sc.kept[i - 1]];
          ge = i == nkept ? H : st.off[sc.kept[i]];
          f = ge > gs;
        }
        const int p = block_scan(f, S.warp_tmp, &total);
        if (f) { sc.gap_s[base + p] = gs; sc.gap_e[base + p] = ge; }
        base += total;
        __syncthreads();
      }
      if (tid == 0) s_ng = base;
      __syncthreads();
    }
    PSTAMP(8);
    // I. placement order: CARRY by id, ALLOC by id, FETCH by (host offset, id)
    __shared__ uint64_t pkey[kEntCap];
    {
      if (tid == 0) s_nplaced = 0;
      __syncthreads();
      for (int e = tid; e < n; e += NT) {
        const int c = S.e_cls[e];
        if (c == C_KEEP) continue;
        const int t = S.e_t[e];
        const uint64_t rank = c == C_CARRY ? 0 : (c == C_ALLOC ? 1 : 2);
        const uint64_t mid = c == C_FETCH ? (uint64_t)(t_host[t] / AL) : 0;
        const int k = atomicAdd(&s_nplaced, 1);
        pkey[k] = (rank << 62) | (mid << 20) | (uint64_t)t;
      }
      __syncthreads();
      sort_keys(pkey, s_nplaced);
    }
    const int np = s_nplaced;
    PSTAMP(9);
    // J. first fit by warp 0 (R11). <= 32 gaps and placed tensors: gaps and sizes live in
    //    registers (lane g owns gap g, lane p holds placed tensor p), one ballot per placement
    if (tid < 32) {
      const int lane = tid;
      const int ng = s_ng;
      bool fail = false;
      if (ng <= 32 && np <= 32) {
        int64_t gs = lane < ng ? sc.gap_s[lane] : 0, ge = lane < ng ? sc.gap_e[lane] : 0;
        const int my_t = lane < np ? (int)(pkey[lane] & 0xFFFFF) : 0;
        const int64_t my_a = lane < np ? t_ab[my_t] : 0;
        for (int p = 0; p < np; ++p) {
          const int64_t need_t = __shfl_sync(0xffffffffu, my_a, p);
          const unsigned bal = __ballot_sync(0xffffffffu, lane < ng && ge - gs >= need_t);
          if (!bal) { fail = true; break; }
          const int found = __ffs(bal) - 1;
          const int64_t off = __shfl_sync(0xffffffffu, gs, found);
          if (lane == found) gs += need_t;
          if (lane == p) sc.newoff[my_t] = off;
        }
      } else {
        for (int p = 0; p < np && !fail; ++p) {
          const int t = (int)(pkey[p] & 0xFFFFF);
          const int64_t need_t = t_ab[t];
          int found = -1;
          for (int g0 = 0; g0 < ng; g0 += 32) {
            const int g = g0 + lane;
            const bool fits = g < ng && (sc.gap_e[g] - sc.gap_s[g]) >= need_t;
            const unsigned bal = __ballot_sync(0xffffffffu, fits);
            if (bal) { found = g0 + __ffs(bal) - 1; break; }
          }
          if (found < 0) { fail = true; break; }
          if (lane == 0) {
            sc.newoff[t] = sc.gap_s[found];
            sc.gap_s[found] += need_t;
          }
          __syncwarp();
        }
      }
      if (lane == 0) s_compact = fail ? 1 : 0;
    }
    __syncthreads();
    // compaction fallback: exclusive prefix sums over [kept | placed]
    if (s_compact) {
      if (tid == 0) {
        int64_t c = 0;
        for (int i = 0; i < nkept; ++i) { const int t = sc.kept[i]; sc.newoff[t] = c; c += t_ab[t]; }
        for (int p = 0; p < np; ++p) { const int t = (int)(pkey[p] & 0xFFFFF); sc.newoff[t] = c; c += t_ab[t]; }
      }
    } else {
      for (int i = tid; i < nkept; i += NT) sc.newoff[sc.kept[i]] = st.off[sc.kept[i]];
    }
    __syncthreads();
    PSTAMP(11);
    // K. records
    if (c_ca + s_nc > out.cap_rec || c_al + s_na > out.cap_rec || c_fe + s_nf > out.cap_rec ||
        c_mv + nkept > out.cap_rec) {
      if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_mv + nkept); }
      return;
    }
    // MOVE (compaction only): kept whose offset changed, in kept order
    long long my_d2d = 0, my_h2d = 0;
    {
      int total = 0, base = 0;
      if (s_compact) {
        for (int i0 = 0; i0 < nkept; i0 += NT) {
          const int i = i0 + tid;
          int f = 0, t = -1;
          if (i < nkept) { t = sc.kept[i]; f = sc.newoff[t] != st.off[t]; }
          const int p = block_scan(f, S.warp_tmp, &total);
          if (f) {
            dyo_move_rec r;
            r.t = t;
            r.src = (int64_t)m * H + st.off[t];
            r.dst = (int64_t)m * H + sc.newoff[t];
            r.bytes = t_by[t];
            out.mv[c_mv + base + p] = r;
            my_d2d += t_by[t];
          }
          base += total;
          __syncthreads();
        }
      }
      if (tid == 0) s_nmove = base;
    }
    const int nc = s_nc, na = s_na, nf = s_nf;
    for (int p = tid; p < np; p += NT) {
      const int t = (int)(pkey[p] & 0xFFFFF);
      const int64_t dst = (int64_t)m * H + sc.newoff[t];
      if (p < nc) {
        dyo_carry_rec r;
        r.t = t;
        r.src = (int64_t)(1 - m) * H + st.off[t];
        r.dst = dst;
        r.bytes = t_by[t];
        r.late = st.pw[t] ? 1 : 0;
        out.ca[c_ca + p] = r;
        my_d2d += t_by[t];
      } else if (p < nc + na) {
        dyo_alloc_rec r;
        r.t = t;
        r.dst = dst;
        r.bytes = t_by[t];
        out.al[c_al + p - nc] = r;
      } else {
        dyo_fetch_rec r;
        r.t = t;
        r.host_off = t_host[t];
        r.dst = dst;
        r.bytes = t_by[t];
        out.fe[c_fe + p - nc - na] = r;
        my_h2d += t_by[t];
      }
    }
    const int64_t ebase_j = sc.ebase[j];
    for (int e = tid; e < n; e += NT) {
      const int t = S.e_t[e];
      dyo_entry_rec r;
      r.t = t;
      r.mode = S.e_mode[e];
      r.needs_fetch = S.e_rd[e];
      r.dst = (int64_t)m * H + sc.newoff[t];
      out.ent[ebase_j + e] = r;
    }
    {
      const long long t1 = block_sum64(my_d2d, S.sum_tmp);
      const long long t2 = block_sum64(my_h2d, S.sum_tmp);
      if (tid == 0) { s_d2d = (unsigned long long)t1; s_h2d = (unsigned long long)t2; }
    }
    __syncthreads();
    PSTAMP(12);
    // L. state update
    for (int i = tid; i < nm; i += NT) {
      const int t = resm[i];
      const int8_t r = sc.rstat[t];
      if (r == RS_DEAD || r == RS_EVICT) { st.loc[t] = -1; st.dirty[t] = 0; }
    }
    for (int i = tid; i < nkept; i += NT) st.off[sc.kept[i]] = sc.newoff[sc.kept[i]];
    for (int p = tid; p < np; p += NT) {
      const int t = (int)(pkey[p] & 0xFFFFF);
      st.loc[t] = (int8_t)m;
      st.off[t] = sc.newoff[t];
      if (p >= nc) st.dirty[t] = 0;   // ALLOC, FETCH
    }
    __syncthreads();
    for (int e = tid; e < n; e += NT) {
      if (S.e_mode[e] & 2) st.dirty[S.e_t[e]] = 1;   // block j writes
    }
    PSTAMP(13);
    // previous-group written flags, next occurrences, inW
    const int pn = st.prev_n[0];
    for (int i = tid; i < pn; i += NT) st.pw[st.prev[i]] = 0;
    __syncthreads();
    for (int e = tid; e < n; e += NT) {
      const int t = S.e_t[e];
      st.pw[t] = (S.e_mode[e] & 2) ? 1 : 0;
      st.prev[e] = t;
      sc.cur_next[t] = sc.nxt[ebase_j + e];
      sc.cur_rd[t] = sc.nxt_rd[ebase_j + e];
      sc.inw[t] = 0;
    }
    for (int i = tid; i < nm; i += NT) sc.rstat[resm[i]] = RS_NONE;
    if (tid == 0) st.prev_n[0] = n;
    __syncthreads();
    PSTAMP(14);
    // resident lists: half m = kept + placed sorted by offset; half 1-m drops what left it
    {
      // the kept tensors are already in ascending offset (first fit leaves them in place,
      // compaction preserves their order), so only the placed ones are sorted (|W_j| keys) and
      // the two runs are merged: every element's slot = its rank in its own run + the number of
      // smaller keys in the other run (binary search; offsets of one half are unique)
      const int nnew = nkept + np;
      int32_t* resw = st.res + (int64_t)m * T;
      uint64_t* pk = S.sortbuf;                       // placed keys (np <= kEntCap <= kSortCap)
      int64_t* kk = sc.gap_s;                         // kept offsets (the gaps are consumed)
      for (int k = tid; k < np; k += NT) {
        const int t = (int)(pkey[k] & 0xFFFFF);
        pk[k] = ((uint64_t)(st.off[t] / AL) << 20) | (uint64_t)t;
      }
      for (int i = tid; i < nkept; i += NT) kk[i] = st.off[sc.kept[i]];
      __syncthreads();
      sort_keys(pk, np);
      for (int i = tid; i < nkept; i += NT) {
        const uint64_t key = (uint64_t)(kk[i] / AL) << 20;
        int lo = 0, hi = np;                          // placed keys below this kept offset
        while (lo < hi) { const int mid = (lo + hi) >> 1; if (pk[mid] < key) lo = mid + 1; else hi = mid; }
        resw[i + lo] = sc.kept[i];
      }
      for (int k = tid; k < np; k += NT) {
        const int64_t o = (int64_t)((pk[k] >> 20) * (uint64_t)AL);
        int lo = 0, hi = nkept;                       // kept offsets below this placed offset
        while (lo < hi) { const int mid = (lo + hi) >> 1; if (kk[mid] < o) lo = mid + 1; else hi = mid; }
        resw[k + lo] = (int)(pk[k] & 0xFFFFF);
      }
      if (tid == 0) st.res_n[m] = nnew;
      __syncthreads();
      const int no = st.res_n[1 - m];
      int32_t* reso = st.res + (int64_t)(1 - m) * T;
      int total = 0, base = 0;
      for (int i0 = 0; i0 < no; i0 += NT) {
        const int i = i0 + tid;
        int f = 0, t = -1;
        if (i < no) { t = reso[i]; f = st.loc[t] == 1 - m; }
        const int p = block_scan(f, S.warp_tmp, &total);
        // in-place compaction is safe: p <= i and the scan completed before any write
        if (f) sc.kept[base + p] = t;
        base += total;
        __syncthreads();
      }
      for (int i = tid; i < base; i += NT) reso[i] = sc.kept[i];
      if (tid == 0) st.res_n[1 - m] = base;
    }
    PSTAMP(15);
    // M. header
    if (tid == 0) {
      hd.half = m;
      hd.n_ent = n;
      hd.n_evict = nev;
      hd.n_move = s_nmove;
      hd.n_carry = nc;
      hd.n_alloc = na;
      hd.n_fetch = nf;
      hd.need = (int64_t)s_need;
      hd.h2d = (int64_t)s_h2d;
      hd.d2h = (int64_t)s_d2h;
      hd.d2d = (int64_t)s_d2d;
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
  }
  if (tid == 0) st.G[0] += Kt;
  if (smem_state) {
    __syncthreads();
    for (int t = tid; t < T; t += NT) {
      stg.loc[t] = st.loc[t];
      stg.off[t] = st.off[t];
      stg.dirty[t] = st.dirty[t];
      stg.pw[t] = st.pw[t];
      stg.res[t] = st.res[t];
      stg.res[T + t] = st.res[T + t];
      stg.prev[t] = st.prev[t];
    }
    if (tid == 0) {
      stg.res_n[0] = st.res_n[0];
      stg.res_n[1] = st.res_n[1];
      stg.prev_n[0] = st.prev_n[0];
      stg.G[0] = st.G[0];
    }
  }
  if (tid == 0) {
    out.counts[0] = Kt;
    out.counts[1] = (int)c_ev;
    out.counts[2] = (int)c_mv;
    out.counts[3] = (int)c_ca;
    out.counts[4] = (int)c_al;
    out.counts[5] = (int)c_fe;
    status[0] = 0;
  }
}

size_t plan_state_smem_bytes(int T) {
  auto r16 = [](size_t b) { return (b + 15) / 16 * 16; };
  const size_t t = (size_t)T;
  return r16(8 * t) + 2 * r16(8 * (t + 1)) + 4 * r16(8 * t) + r16(8 * t) + 4 * r16(4 * t) + 3 * 16 + 6 * r16(t);
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
  static bool attr = false;
  constexpr int kMaxDyn = 227 * 1024 - 12 * 1024;      // leave room for the static shared arrays
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(plan_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, kMaxDyn);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  const size_t base = (sizeof(PlanSmem) + 15) / 16 * 16;
  const size_t need = base + plan_state_smem_bytes(a.T);
  const int smem_state = (need <= (size_t)kMaxDyn && !getenv("DYO_PLAN_GLOBAL_STATE")) ? 1 : 0;
  const size_t smem = smem_state ? need : sizeof(PlanSmem);
  plan_kernel<<<1, kPlanThreads, smem, s>>>(a, pd, b0, nb, policy, in, work, sc, out, max_groups, smem_state);
  return cudaGetLastError();
}

}  // namespace dyo
