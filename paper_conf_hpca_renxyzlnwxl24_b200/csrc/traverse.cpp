// A3 traversal decode (§IV-B; R4): map the predicted execution-
// block vectors back onto the program when the pilot has no branch head.
//
// "we traverse the control flow graph ... to find a path whose operators, grouped by the
// predicted numbers of operators, match the predicted block vectors" (L145); "if no path
// matches, we choose the path whose number of operators is closest" (L147).
//
// Runs on the host, like the paper's mapping (it needs the logits D2H: dyo_pilot_predict syncs
// once in this mode). Reading R4 fixes the order: paths are visited in lexicographic order of
// the sites' choices (preorder; lower branch index / lower trip count first); the first exact
// match wins; otherwise the path with the smallest |L - sum n_0|, first in that order.
//
//   exact match: depth-first over the top-level pieces in site order, rows streamed into the
//                current group's running block vector; a branch is cut as soon as a partial sum
//                exceeds the predicted vector (all signature elements are >= 0, so running sums
//                only grow) or a completed group differs. Failed states
//                (piece, group, partial vector, choices of tie targets still referenced) are
//                memoised, so the search is polynomial on programs whose sites repeat.
//   fallback:    L = static + sum over free sites f_s(c_s) (a tied site adds to its target's
//                f), so the reachable lengths are a subset-sum over free sites: suffix bitsets,
//                then the lexicographically first choice vector reaching the best distance.
#include <algorithm>
#include <array>
#include <cstdlib>
#include <cstdint>
#include <cstring>
#include <string>
#include <unordered_set>
#include <vector>

#include "dyo_internal.h"

namespace dyo {

namespace {

struct Key {
  std::vector<int64_t> v;
  bool operator==(const Key& o) const { return v == o.v; }
};
struct KeyHash {
  size_t operator()(const Key& k) const {
    uint64_t h = 1469598103934665603ull;
    for (int64_t x : k.v) {
      h ^= (uint64_t)x;
      h *= 1099511628211ull;
    }
    return (size_t)h;
  }
};

struct Dfs {
  const TravArch& A;
  std::vector<std::array<int64_t, 10>> pred;   // non-empty predicted slots, slot order
  int nk = 0;
  std::vector<int32_t> ch;                     // choice per site
  std::vector<std::vector<int>> live;          // per piece: tie targets decided before it and used at/after it
  std::unordered_set<Key, KeyHash> failed;
  size_t memo_cap = 4u << 20;
  int64_t steps = 0, step_cap = (int64_t)1 << 31;
  bool overflow = false;
  // streaming state
  int g = 0;
  int64_t acc[10];

  explicit Dfs(const TravArch& a) : A(a) {}

  // feed one row (op index, or -1 for a control row); false = this prefix cannot match
  bool row(int op) {
    if (g >= nk) return false;
    acc[0] += 1;
    if (op >= 0) {
      const int32_t* s = &A.sig[(size_t)op * 9];
      for (int e = 0; e < 9; ++e) acc[1 + e] += s[e];
    }
    const auto& p = pred[g];
    for (int e = 0; e < 10; ++e)
      if (std::min<int64_t>(acc[e], kSat) > p[e]) return false;
    if (acc[0] == p[0]) {
      for (int e = 0; e < 10; ++e)
        if (std::min<int64_t>(acc[e], kSat) != p[e]) return false;
      ++g;
      std::memset(acc, 0, sizeof acc);
    }
    return true;
  }

  int n_choices(int p) const {
    const int k = A.piece_kind[p];
    if (k == 0) return 1;
    const int s = A.piece_a[p];
    return A.site_tie[s] >= 0 ? 1 : A.site_nch[s];
  }

  // rows of piece p under choice c; false as soon as the prefix fails
  bool feed(int p, int c) {
    const int k = A.piece_kind[p];
    if (k == 0) {
      for (int q = 0; q < A.piece_b[p]; ++q)
        if (!row(A.piece_a[p] + q)) return false;
      return true;
    }
    const int s = A.piece_a[p];
    if (k == 1) {
      if (!row(-1)) return false;
      const int arm = A.site_arm_ptr[s] + c;
      for (int q = 0; q < A.arm_n[arm]; ++q)
        if (!row(A.arm_first[arm] + q)) return false;
      return true;
    }
    const int n = A.site_lo[s] + c;
    for (int it = 0; it < n; ++it) {
      if (!row(-1)) return false;
      for (int q = 0; q < A.piece_c[p]; ++q)
        if (!row(A.piece_b[p] + q)) return false;
      if (++steps > step_cap) { overflow = true; return false; }
    }
    return row(-1);
  }

  Key key(int p) const {
    Key k;
    k.v.reserve(12 + live[p].size());
    k.v.push_back(p);
    k.v.push_back(g);
    for (int e = 0; e < 10; ++e) k.v.push_back(acc[e]);
    for (int t : live[p]) k.v.push_back(ch[t]);
    return k;
  }

  bool search(int p) {
    if (overflow) return false;
    const int np = (int)A.piece_kind.size();
    if (p == np) {
      if (g != nk) return false;
      for (int e = 0; e < 10; ++e)
        if (acc[e]) return false;
      return true;
    }
    Key k = key(p);
    if (failed.count(k)) return false;
    const int kind = A.piece_kind[p];
    const int s = kind == 0 ? -1 : A.piece_a[p];
    const int nc = n_choices(p);
    const int g0 = g;
    int64_t acc0[10];
    std::memcpy(acc0, acc, sizeof acc);
    for (int c = 0; c < nc; ++c) {
      int cc = c;
      if (s >= 0) {
        cc = A.site_tie[s] >= 0 ? ch[A.site_tie[s]] : c;
        ch[s] = cc;
      }
      ++steps;
      if (feed(p, cc) && search(p + 1)) return true;
      if (overflow) return false;
      g = g0;
      std::memcpy(acc, acc0, sizeof acc);
    }
    if (failed.size() < memo_cap) failed.insert(std::move(k));
    return false;
  }
};

int64_t piece_len(const TravArch& A, int p, int c) {
  const int k = A.piece_kind[p];
  if (k == 0) return A.piece_b[p];
  const int s = A.piece_a[p];
  if (k == 1) return 1 + A.arm_n[A.site_arm_ptr[s] + c];
  return (int64_t)(A.site_lo[s] + c) * (1 + A.piece_c[p]) + 1;
}

}  // namespace

dyo_status traverse_decode(const TravArch& A, const int32_t* slots, int K_max, int32_t* choices, int* matched,
                           std::string& err) {
  const int n_sites = (int)A.site_kind.size();
  const int np = (int)A.piece_kind.size();
  Dfs d(A);
  int64_t total = 0;
  for (int k = 0; k < K_max; ++k) {
    if (slots[k * 10] == 0) continue;
    std::array<int64_t, 10> v;
    for (int e = 0; e < 10; ++e) v[e] = slots[k * 10 + e];
    d.pred.push_back(v);
    total += v[0];
  }
  d.nk = (int)d.pred.size();
  d.ch.assign(n_sites, 0);
  // tie targets still referenced at or after each piece (memo key component)
  std::vector<int> piece_site(np, -1), last_use(n_sites, -1);
  for (int p = 0; p < np; ++p)
    if (A.piece_kind[p] != 0) piece_site[p] = A.piece_a[p];
  for (int p = 0; p < np; ++p) {
    const int s = piece_site[p];
    if (s >= 0 && A.site_tie[s] >= 0) last_use[A.site_tie[s]] = p;
  }
  std::vector<int> site_piece(n_sites, -1);
  for (int p = 0; p < np; ++p)
    if (piece_site[p] >= 0) site_piece[piece_site[p]] = p;
  std::vector<int> targets;
  for (int t = 0; t < n_sites; ++t)
    if (last_use[t] >= 0 && site_piece[t] >= 0) targets.push_back(t);
  d.live.assign(np + 1, {});
  for (int t : targets)
    for (int p = site_piece[t] + 1; p <= last_use[t]; ++p) d.live[p].push_back(t);
  std::memset(d.acc, 0, sizeof d.acc);
  d.g = 0;
  if (d.search(0)) {
    for (int s = 0; s < n_sites; ++s) choices[s] = d.ch[s];
    *matched = 1;
    return DYO_OK;
  }
  if (d.overflow) {
    err = "traversal: search exceeded its step budget";
    return DYO_E_CAPACITY;
  }
  // ---- fallback: closest operator count, first in lexicographic order ----
  *matched = 0;
  int64_t stat = 0;
  std::vector<int> free_sites;
  for (int s = 0; s < n_sites; ++s)
    if (A.site_tie[s] < 0) free_sites.push_back(s);
  const int nf = (int)free_sites.size();
  std::vector<int> fidx(n_sites, -1);
  for (int i = 0; i < nf; ++i) fidx[free_sites[i]] = i;
  std::vector<std::vector<int64_t>> f(nf);
  for (int i = 0; i < nf; ++i) f[i].assign(A.site_nch[free_sites[i]], 0);
  for (int p = 0; p < np; ++p) {
    const int s = piece_site[p];
    if (s < 0) { stat += piece_len(A, p, 0); continue; }
    const int root = A.site_tie[s] >= 0 ? A.site_tie[s] : s;
    const int i = fidx[root];
    for (int c = 0; c < (int)f[i].size(); ++c) f[i][c] += piece_len(A, p, c);
  }
  int64_t maxL = 0;
  for (int i = 0; i < nf; ++i) maxL += *std::max_element(f[i].begin(), f[i].end());
  const int64_t W = maxL + 1;
  if ((double)(nf + 1) * (double)W > (double)(1ll << 31)) {
    err = "traversal fallback: reachable-length table too large";
    return DYO_E_CAPACITY;
  }
  // R[i] = lengths reachable by free sites i..nf-1 (byte per length: simple and small here)
  std::vector<std::vector<uint8_t>> R(nf + 1, std::vector<uint8_t>(W, 0));
  R[nf][0] = 1;
  for (int i = nf - 1; i >= 0; --i)
    for (int64_t v = 0; v < W; ++v)
      if (R[i + 1][v])
        for (int64_t fl : f[i])
          if (v + fl < W) R[i][v + fl] = 1;
  int64_t dmin = INT64_MAX;
  for (int64_t v = 0; v < W; ++v)
    if (R[0][v]) dmin = std::min<int64_t>(dmin, std::llabs(stat + v - total));
  int64_t pre = stat;
  std::vector<int32_t> ch(n_sites, 0);
  for (int i = 0; i < nf; ++i) {
    int pick = -1;
    for (int c = 0; c < (int)f[i].size() && pick < 0; ++c) {
      const int64_t base = pre + f[i][c];
      for (int64_t tgt : {total - dmin, total + dmin}) {
        const int64_t v = tgt - base;
        if (v >= 0 && v < W && R[i + 1][v]) { pick = c; break; }
      }
    }
    if (pick < 0) { err = "traversal fallback: internal inconsistency"; return DYO_E_INVAL; }
    ch[free_sites[i]] = pick;
    pre += f[i][pick];
  }
  for (int s = 0; s < n_sites; ++s) choices[s] = A.site_tie[s] >= 0 ? ch[A.site_tie[s]] : ch[s];
  return DYO_OK;
}

}  // namespace dyo
