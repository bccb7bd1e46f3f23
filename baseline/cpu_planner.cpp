// Compiled single-core CPU planner - the honest baseline for K2 ("report the plan
// against a compiled single-core CPU planner, timed by the bench on the box's host").
// NOT part of the product path: the bench times it beside the GPU planner; tests check it is
// bit-exact with oracle/plan.py (the same readings R7-R12, R9 as of round 2). Plain C ABI.
//
// Per transition: classify W_j (KEEP/CARRY/ALLOC/FETCH) from the residency, scan half m's
// resident list (kept sorted by offset) for dead / live candidates, RETAIN's prefix cut by a
// sort of the live keys, EVICT sorted by (host offset, id), first fit into the gaps between the
// kept tensors (or the compaction prefix sums), records and state. Next uses come from one
// reverse sweep over the plan's entries.
#include <algorithm>
#include <cstdint>
#include <cstring>
#include <tuple>
#include <vector>

namespace {

struct State {
  std::vector<int8_t> loc;
  std::vector<int64_t> off;
  std::vector<uint8_t> dirty;
  std::vector<int32_t> prev_t;     // W_{j-1} tensors
  std::vector<int32_t> prev_m;     // their modes
  int64_t G = 0;
  std::vector<int32_t> res[2];     // residents of each half, ascending offset
};

}  // namespace

extern "C" {

// counts[6] out: K, evict, move, carry, alloc, fetch records. Record arrays are caller-owned
// with capacity cap each (5, 4, 5, 3, 4 int64 per record as in include/dyo.h). hdr: per
// transition {half, n_evict, n_move, n_carry, n_alloc, n_fetch, h2d, d2h, d2d, need} (10 int64).
// Returns 0, -3 (budget), -6 (capacity).
void* cpu_plan_create(int32_t T) {
  State* s = new State();
  s->loc.assign(T, -1);
  s->off.assign(T, 0);
  s->dirty.assign(T, 0);
  return s;
}

void cpu_plan_destroy(void* p) { delete static_cast<State*>(p); }

int32_t cpu_plan(void* sp, int32_t T, const int64_t* bytes, const int64_t* host_off, const int32_t* transient,
                 int64_t budget, int64_t align, int32_t policy, int32_t K, const int32_t* ent_ptr /*K+1*/,
                 const int32_t* ent_t, const int32_t* ent_mode, const int32_t* ent_rd, int64_t cap, int64_t* hdr,
                 int64_t* ev, int64_t* mv, int64_t* ca, int64_t* al, int64_t* fe, int64_t* counts) {
  State st = *static_cast<State*>(sp);          // transactional: committed on success only
  const int64_t H = budget / 2 / align * align;
  std::vector<int64_t> a(T);
  for (int t = 0; t < T; ++t) a[t] = (bytes[t] + align - 1) / align * align;
  for (int t = 0; t < T; ++t)
    if (transient[t]) st.dirty[t] = 0;           // R9
  // next occurrence of every entry and the first occurrence of every tensor (reverse sweep)
  const int E = ent_ptr[K];
  std::vector<int32_t> nxt(E), nxt_rd(E), cur(T, -1), cur_rd(T, 0);
  for (int j = K - 1; j >= 0; --j) {
    for (int e = ent_ptr[j]; e < ent_ptr[j + 1]; ++e) {
      nxt[e] = cur[ent_t[e]];
      nxt_rd[e] = cur_rd[ent_t[e]];
    }
    for (int e = ent_ptr[j]; e < ent_ptr[j + 1]; ++e) {
      cur[ent_t[e]] = j;
      cur_rd[ent_t[e]] = ent_rd[e];
    }
  }
  // next use of every tensor from transition j on: starts at its first occurrence
  std::vector<int32_t> nx = cur, nxr = cur_rd;
  std::vector<uint8_t> inw(T, 0), pw(T, 0);
  for (size_t i = 0; i < st.prev_t.size(); ++i)
    if (st.prev_m[i] & 2) pw[st.prev_t[i]] = 1;
  int64_t c_ev = 0, c_mv = 0, c_ca = 0, c_al = 0, c_fe = 0;
  std::vector<int32_t> keep, carry, alloc, fetch, kept;
  std::vector<std::tuple<int64_t, int64_t, int32_t>> live;
  std::vector<int32_t> evicted;
  std::vector<int64_t> newoff(T);
  std::vector<uint8_t> is_dead(T, 0), retained(T, 0);
  for (int j = 0; j < K; ++j) {
    const int m = (int)((st.G + j) & 1);
    const int e0 = ent_ptr[j], e1 = ent_ptr[j + 1];
    int64_t need = 0;
    keep.clear(); carry.clear(); alloc.clear(); fetch.clear();
    for (int e = e0; e < e1; ++e) {
      const int t = ent_t[e];
      inw[t] = 1;
      // R20 (policy bit 2): valid in the other half and held by the next group -> stays there
      const bool share = (policy & 2) && st.loc[t] == 1 - m && nxt[e] == j + 1;
      if (!share) need += a[t];
      if (st.loc[t] == m) keep.push_back(t);
      else if (share) continue;
      else if (st.loc[t] == 1 - m && ent_rd[e]) carry.push_back(t);
      else if (ent_rd[e]) fetch.push_back(t);
      else alloc.push_back(t);
    }
    if (need > H) return -3;
    // candidates of half m
    live.clear();
    evicted.clear();
    std::vector<int32_t> cands;
    for (int t : st.res[m])
      if (st.loc[t] == m && !inw[t]) cands.push_back(t);
    int64_t room = H - need;
    for (int t : cands) {
      const bool dead = transient[t] && (nx[t] < 0 || !nxr[t]);
      is_dead[t] = dead;
      if (!dead) live.emplace_back(nx[t] < 0 ? (int64_t)1 << 62 : (int64_t)(nx[t] - j), a[t], t);
    }
    std::vector<int32_t> ret;
    if (policy & 1) {
      std::sort(live.begin(), live.end());
      int64_t used = 0;
      for (auto& x : live) {
        if (used + std::get<1>(x) > room) break;
        used += std::get<1>(x);
        ret.push_back(std::get<2>(x));
        retained[std::get<2>(x)] = 1;
      }
    }
    for (int t : cands)
      if (is_dead[t] || !retained[t]) evicted.push_back(t);
    std::sort(evicted.begin(), evicted.end(), [&](int x, int y) {
      return host_off[x] != host_off[y] ? host_off[x] < host_off[y] : x < y; });
    if (c_ev + (int64_t)evicted.size() > cap) return -6;
    int64_t d2h = 0, h2d = 0, d2d = 0;
    for (int t : evicted) {
      int64_t* r = ev + 5 * c_ev++;
      const bool wb = st.dirty[t] && !is_dead[t];
      r[0] = t; r[1] = (int64_t)m * H + st.off[t]; r[2] = host_off[t]; r[3] = bytes[t]; r[4] = wb;
      if (wb) d2h += bytes[t];
    }
    // kept (KEEP + retained), ascending old offset; placed: CARRY by id, ALLOC by id, FETCH by (host, id)
    kept.clear();
    for (int t : st.res[m])
      if (st.loc[t] == m && (inw[t] || retained[t])) kept.push_back(t);
    std::sort(carry.begin(), carry.end());
    std::sort(alloc.begin(), alloc.end());
    std::sort(fetch.begin(), fetch.end(), [&](int x, int y) {
      return host_off[x] != host_off[y] ? host_off[x] < host_off[y] : x < y; });
    std::vector<int32_t> placed;
    placed.insert(placed.end(), carry.begin(), carry.end());
    placed.insert(placed.end(), alloc.begin(), alloc.end());
    placed.insert(placed.end(), fetch.begin(), fetch.end());
    // first fit (R11)
    std::vector<std::pair<int64_t, int64_t>> gaps;
    int64_t cu = 0;
    for (int t : kept) {
      if (st.off[t] > cu) gaps.push_back({cu, st.off[t]});
      cu = st.off[t] + a[t];
    }
    if (H > cu) gaps.push_back({cu, H});
    bool ok = true;
    for (int t : placed) {
      bool got = false;
      for (auto& g : gaps)
        if (g.second - g.first >= a[t]) { newoff[t] = g.first; g.first += a[t]; got = true; break; }
      if (!got) { ok = false; break; }
    }
    for (int t : kept) newoff[t] = st.off[t];
    if (!ok) {
      int64_t c = 0;
      for (int t : kept) { newoff[t] = c; c += a[t]; }
      for (int t : placed) { newoff[t] = c; c += a[t]; }
    }
    if (c_mv + (int64_t)kept.size() > cap || c_ca + (int64_t)carry.size() > cap || c_al + (int64_t)alloc.size() > cap ||
        c_fe + (int64_t)fetch.size() > cap)
      return -6;
    int64_t n_mv = 0;
    for (int t : kept)
      if (newoff[t] != st.off[t]) {
        int64_t* r = mv + 4 * c_mv++;
        r[0] = t; r[1] = (int64_t)m * H + st.off[t]; r[2] = (int64_t)m * H + newoff[t]; r[3] = bytes[t];
        d2d += bytes[t];
        ++n_mv;
      }
    for (int t : carry) {
      int64_t* r = ca + 5 * c_ca++;
      r[0] = t; r[1] = (int64_t)(1 - m) * H + st.off[t]; r[2] = (int64_t)m * H + newoff[t]; r[3] = bytes[t];
      r[4] = pw[t];
      d2d += bytes[t];
    }
    for (int t : alloc) {
      int64_t* r = al + 3 * c_al++;
      r[0] = t; r[1] = (int64_t)m * H + newoff[t]; r[2] = bytes[t];
    }
    for (int t : fetch) {
      int64_t* r = fe + 4 * c_fe++;
      r[0] = t; r[1] = host_off[t]; r[2] = (int64_t)m * H + newoff[t]; r[3] = bytes[t];
      h2d += bytes[t];
    }
    int64_t* hd = hdr + 10 * j;
    hd[0] = m; hd[1] = (int64_t)evicted.size(); hd[2] = n_mv; hd[3] = (int64_t)carry.size();
    hd[4] = (int64_t)alloc.size(); hd[5] = (int64_t)fetch.size(); hd[6] = h2d; hd[7] = d2h; hd[8] = d2d; hd[9] = need;
    // state
    for (int t : evicted) { st.loc[t] = -1; st.dirty[t] = 0; }
    std::vector<int32_t> order = kept;
    order.insert(order.end(), placed.begin(), placed.end());
    for (int t : order) { st.loc[t] = (int8_t)m; st.off[t] = newoff[t]; }
    for (int t : fetch) st.dirty[t] = 0;
    for (int t : alloc) st.dirty[t] = 0;
    for (int e = e0; e < e1; ++e)
      if (ent_mode[e] & 2) st.dirty[ent_t[e]] = 1;
    // resident lists: half m rebuilt by offset; half 1-m drops what left it
    std::sort(order.begin(), order.end(), [&](int x, int y) { return st.off[x] < st.off[y]; });
    st.res[m] = order;
    std::vector<int32_t> other;
    for (int t : st.res[1 - m])
      if (st.loc[t] == 1 - m) other.push_back(t);
    st.res[1 - m].swap(other);
    // W_j's next uses, previous-group written flags, membership
    for (int t : st.prev_t) pw[t] = 0;
    st.prev_t.clear();
    st.prev_m.clear();
    for (int e = e0; e < e1; ++e) {
      const int t = ent_t[e];
      nx[t] = nxt[e];
      nxr[t] = nxt_rd[e];
      inw[t] = 0;
      pw[t] = (ent_mode[e] & 2) ? 1 : 0;
      st.prev_t.push_back(t);
      st.prev_m.push_back(ent_mode[e]);
    }
    for (int t : ret) retained[t] = 0;
    for (int t : cands) is_dead[t] = 0;
  }
  st.G += K;
  counts[0] = K; counts[1] = c_ev; counts[2] = c_mv; counts[3] = c_ca; counts[4] = c_al; counts[5] = c_fe;
  *static_cast<State*>(sp) = std::move(st);
  return 0;
}

}  // extern "C"
