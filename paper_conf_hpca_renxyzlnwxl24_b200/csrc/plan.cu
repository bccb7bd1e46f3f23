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

#include "dyo_internal.h"

namespace dyo {

constexpr int kSortCap = 4096;      // shared-memory sort capacity (larger sorts use global scratch)
constexpr uint64_t kInfD = 0xFFFFull;

enum RStat : int8_t { RS_NONE = 0, RS_KEEP = 1, RS_LIVE = 2, RS_DEAD = 3, RS_EVICT = 4, RS_RETAIN = 5 };

struct PlanSmem {
  int32_t e_t[kEntCap];
  int8_t e_mode[kEntCap];
  int8_t e_rd[kEntCap];
  int8_t e_cls[kEntCap];
  int64_t e_new[kEntCap];
  uint64_t sortbuf[kSortCap];
  int warp_tmp[32];
  int i_tmp[16];
  unsigned long long u_tmp[8];
};

__device__ __forceinline__ void sort_keys(uint64_t* key, int n) {
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

// Block-wide exclusive scan of one int per thread; returns the prefix, *total gets the sum.
__device__ __forceinline__ int block_scan(int v, int* warp_tmp, int* total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nw = blockDim.x >> 5;
  int x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    const int y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_tmp[w] = x;
  __syncthreads();
  if (w == 0) {
    int s = lane < nw ? warp_tmp[lane] : 0;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const int y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < nw) warp_tmp[lane] = s;
  }
  __syncthreads();
  const int base = w > 0 ? warp_tmp[w - 1] : 0;
  const int tot = warp_tmp[nw - 1];
  __syncthreads();
  if (total) *total = tot;
  return base + x - v;
}

__global__ void __launch_bounds__(kPlanThreads, 1)
plan_kernel(ArchDev a, PredDev pd, int b0, int nb, int policy, PlanState in, PlanState st,
            PlanScratch sc, PlanOut out, int max_groups) {
  extern __shared__ __align__(16) unsigned char smem_raw[];
  PlanSmem& S = *reinterpret_cast<PlanSmem*>(smem_raw);
  const int T = a.T;
  const int64_t H = a.H, AL = a.align;
  int* status = out.status;
  const int tid = threadIdx.x, NT = blockDim.x;

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
    st.dirty[t] = (a.t_flags[t] & 1) ? 0 : in.dirty[t];
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

  for (int j = 0; j < Kt; ++j) {
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
    for (int e = tid; e < n; e += NT) {
      const int t = ent[e].x;
      S.e_t[e] = t;
      S.e_mode[e] = (int8_t)(ent[e].y & 3);
      S.e_rd[e] = (int8_t)((ent[e].y >> 2) & 1);
      atomicAdd(&s_need, (unsigned long long)a.t_abytes[t]);
    }
    __syncthreads();
    // B. feasibility (R7)
    if ((int64_t)s_need > H) {
      if (tid == 0) { status[0] = DYO_E_BUDGET; status[1] = j; status[2] = 0; }
      return;
    }
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
    // D. candidates of half m: dead (R9) or live with next-use distance
    const int nm = st.res_n[m];
    const int32_t* resm = st.res + (int64_t)m * T;
    const bool big = nm > kSortCap;
    uint64_t* keys = big ? sc.keys : S.sortbuf;
    for (int i = tid; i < nm; i += NT) {
      const int t = resm[i];
      if (sc.inw[t]) { sc.rstat[t] = RS_KEEP; continue; }
      const int nx = sc.cur_next[t];
      const bool dead = (nx < 0 && (a.t_flags[t] & 1)) || (nx >= 0 && !sc.cur_rd[t]);
      if (dead) { sc.rstat[t] = RS_DEAD; continue; }
      sc.rstat[t] = RS_LIVE;
      const uint64_t d = nx < 0 ? kInfD : (uint64_t)(nx - j);
      const int k = atomicAdd(&s_nlive, 1);
      keys[k] = (d << 48) | ((uint64_t)(a.t_abytes[t] / AL) << 20) | (uint64_t)t;
      atomicAdd(&s_livebytes, (unsigned long long)a.t_abytes[t]);
    }
    __syncthreads();
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
    // F. EVICT records sorted by (host offset, id)
    for (int i = tid; i < nm; i += NT) {
      const int t = resm[i];
      const int8_t r = sc.rstat[t];
      if (r == RS_DEAD || r == RS_EVICT) {
        const int k = atomicAdd(&s_nev, 1);
        keys[k] = ((uint64_t)(a.t_host[t] / AL) << 20) | (uint64_t)t;
      }
    }
    __syncthreads();
    const int nev = s_nev;
    if (c_ev + nev > out.cap_rec) {
      if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_ev + nev); }
      return;
    }
    sort_keys(keys, nev);
    for (int k = tid; k < nev; k += NT) {
      const int t = (int)(keys[k] & 0xFFFFF);
      const bool wb = sc.rstat[t] == RS_EVICT && st.dirty[t];
      dyo_evict_rec r;
      r.t = t;
      r.src = (int64_t)m * H + st.off[t];
      r.host_off = a.t_host[t];
      r.bytes = a.t_bytes[t];
      r.writeback = wb ? 1 : 0;
      out.ev[c_ev + k] = r;
      if (wb) atomicAdd(&s_d2h, (unsigned long long)a.t_bytes[t]);
    }
    __syncthreads();
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
    // H. gaps of half m between kept tensors
    {
      int total = 0, base = 0;
      for (int i0 = 0; i0 <= nkept; i0 += NT) {
        const int i = i0 + tid;
        int f = 0;
        int64_t gs = 0, ge = 0;
        if (i <= nkept) {
          gs = i == 0 ? 0 : st.off[sc.kept[i - 1]] + a.t_abytes[sc.kept[i - 1]];
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
        const uint64_t mid = c == C_FETCH ? (uint64_t)(a.t_host[t] / AL) : 0;
        const int k = atomicAdd(&s_nplaced, 1);
        pkey[k] = (rank << 62) | (mid << 20) | (uint64_t)t;
      }
      __syncthreads();
      sort_keys(pkey, s_nplaced);
    }
    const int np = s_nplaced;
    // J. first fit by warp 0 (R11)
    if (tid < 32) {
      const int lane = tid;
      const int ng = s_ng;
      bool fail = false;
      for (int p = 0; p < np && !fail; ++p) {
        const int t = (int)(pkey[p] & 0xFFFFF);
        const int64_t need_t = a.t_abytes[t];
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
      if (lane == 0) s_compact = fail ? 1 : 0;
    }
    __syncthreads();
    // compaction fallback: exclusive prefix sums over [kept | placed]
    if (s_compact) {
      if (tid == 0) {
        int64_t c = 0;
        for (int i = 0; i < nkept; ++i) { const int t = sc.kept[i]; sc.newoff[t] = c; c += a.t_abytes[t]; }
        for (int p = 0; p < np; ++p) { const int t = (int)(pkey[p] & 0xFFFFF); sc.newoff[t] = c; c += a.t_abytes[t]; }
      }
    } else {
      for (int i = tid; i < nkept; i += NT) sc.newoff[sc.kept[i]] = st.off[sc.kept[i]];
    }
    __syncthreads();
    // K. records
    if (c_ca + s_nc > out.cap_rec || c_al + s_na > out.cap_rec || c_fe + s_nf > out.cap_rec ||
        c_mv + nkept > out.cap_rec) {
      if (tid == 0) { status[0] = DYO_E_CAPACITY; status[1] = j; status[2] = (int)(c_mv + nkept); }
      return;
    }
    // MOVE (compaction only): kept whose offset changed, in kept order
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
            r.bytes = a.t_bytes[t];
            out.mv[c_mv + base + p] = r;
            atomicAdd(&s_d2d, (unsigned long long)a.t_bytes[t]);
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
        r.bytes = a.t_bytes[t];
        r.late = st.pw[t] ? 1 : 0;
        out.ca[c_ca + p] = r;
        atomicAdd(&s_d2d, (unsigned long long)a.t_bytes[t]);
      } else if (p < nc + na) {
        dyo_alloc_rec r;
        r.t = t;
        r.dst = dst;
        r.bytes = a.t_bytes[t];
        out.al[c_al + p - nc] = r;
      } else {
        dyo_fetch_rec r;
        r.t = t;
        r.host_off = a.t_host[t];
        r.dst = dst;
        r.bytes = a.t_bytes[t];
        out.fe[c_fe + p - nc - na] = r;
        atomicAdd(&s_h2d, (unsigned long long)a.t_bytes[t]);
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
    __syncthreads();
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
    // resident lists: half m = kept + placed sorted by offset; half 1-m drops what left it
    {
      const int nnew = nkept + np;
      uint64_t* rk = nnew > kSortCap ? sc.keys : S.sortbuf;
      for (int i = tid; i < nnew; i += NT) {
        const int t = i < nkept ? sc.kept[i] : (int)(pkey[i - nkept] & 0xFFFFF);
        rk[i] = ((uint64_t)(st.off[t] / AL) << 20) | (uint64_t)t;
      }
      __syncthreads();
      sort_keys(rk, nnew);
      int32_t* resw = st.res + (int64_t)m * T;
      for (int i = tid; i < nnew; i += NT) resw[i] = (int)(rk[i] & 0xFFFFF);
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
  if (tid == 0) {
    st.G[0] += Kt;
    out.counts[0] = Kt;
    out.counts[1] = (int)c_ev;
    out.counts[2] = (int)c_mv;
    out.counts[3] = (int)c_ca;
    out.counts[4] = (int)c_al;
    out.counts[5] = (int)c_fe;
    status[0] = 0;
  }
}

cudaError_t launch_plan(const ArchDev& a, const PredDev& pd, int b0, int nb, int policy,
                        PlanState& in, PlanState& work, PlanScratch& sc, PlanOut& out,
                        int max_groups, cudaStream_t s) {
  static bool attr = false;
  const size_t smem = sizeof(PlanSmem);
  if (!attr) {
    cudaError_t e = cudaFuncSetAttribute(plan_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    if (e != cudaSuccess) return e;
    attr = true;
  }
  plan_kernel<<<1, kPlanThreads, smem, s>>>(a, pd, b0, nb, policy, in, work, sc, out, max_groups);
  return cudaGetLastError();
}

}  // namespace dyo
