// A3 decode of nested control flow (§IV-B; reading R16): a site
// inside a top-level loop body or If arm executes once per iteration / arm execution, each time
// with its own choice, and has no branch-head logit. With the top-level choices fixed (branch
// head), the path is a flat sequence of rows and choice points (one per nested execution). The
// paper's mapping "enumerates and traverses each possible branch" whenever a control flow is
// met (L145): executions in order, lower branch first; the first path whose cut at the
// predicted cumulative counts gives exactly the predicted vectors wins; otherwise the path with
// the closest operator count (L147), first in the same order.
//
//   exact:    depth-first over the choice points; rows stream into the current group's running
//             vector and a prefix is abandoned as soon as a partial sum exceeds the prediction
//             (all elements >= 0) or a finished group differs; failed states (choice point,
//             group, running vector) are memoised.
//   fallback: lengths = static rows + the chosen arms' lengths: suffix reachability over the
//             choice points, then the lexicographically first choice sequence at the best
//             distance.
// Runs on the host like the paper's mapping; dyo_pilot_predict hands the resolved paths to the
// decode kernels.
#include <algorithm>
#include <array>
#include <cstdint>
#include <cstdlib>
#include <cstring>
#include <string>
#include <unordered_set>
#include <vector>

#include "dyo_internal.h"

namespace dyo {

namespace {

struct Atom {
  int type;        // 0 row, 1 choice
  int op;          // row: operator or -1
  int it;          // iteration index (R13) of the row / of the choice's arms
  int arm0, narm;  // choice: arms [arm0, arm0 + narm) of the arm table
};
struct Arm { int first_op, n_ops; };

struct Flat {
  std::vector<Atom> at;
  std::vector<Arm> arms;
};

struct StateKey {
  int pos, g;
  std::array<int64_t, 10> acc;
  bool operator==(const StateKey& o) const { return pos == o.pos && g == o.g && acc == o.acc; }
};
struct StateHash {
  size_t operator()(const StateKey& k) const {
    uint64_t h = 1469598103934665603ull ^ (uint64_t)k.pos * 0x9E3779B97F4A7C15ull ^ (uint64_t)k.g;
    for (int64_t x : k.acc) { h ^= (uint64_t)x; h *= 1099511628211ull; }
    return (size_t)h;
  }
};

// Operators of an arm / body node range, contiguous in preorder (an arm of a nested If holds
// operators only: checked at load).
void flatten_range(const NestArch& N, int first, int last, int it, Flat& F) {
  for (int q = first; q < last;) {
    const int k = N.kind[q];
    if (k == 0) {
      F.at.push_back({0, N.a[q], it, 0, 0});
      ++q;
    } else if (k == 1) {                       // nested If: control row, then a choice point
      F.at.push_back({0, -1, it, 0, 0});
      Atom c{1, -1, it, (int)F.arms.size(), N.a[q]};
      int r = q + 1;
      for (int br = 0; br < N.a[q]; ++br) {
        const int n = N.span[r];
        F.arms.push_back({n > 0 ? N.a[r + 1] : 0, n});   // BRANCH node r, its ops r+1 .. r+n
        r += 1 + n;
      }
      F.at.push_back(c);
      q += 1 + N.span[q];
    } else {
      ++q;                                     // BRANCH markers are consumed by their If
    }
  }
}

Flat flatten(const NestArch& N, const int32_t* ch) {
  Flat F;
  const int n = (int)N.kind.size();
  for (int q = 0; q < n;) {
    const int k = N.kind[q];
    if (k == 0) {
      F.at.push_back({0, N.a[q], 0, 0, 0});
      ++q;
      continue;
    }
    const int s = N.site_of[q];
    const int c = N.site_tie[s] >= 0 ? ch[N.site_tie[s]] : ch[s];
    if (k == 1) {
      F.at.push_back({0, -1, 0, 0, 0});
      int r = q + 1;
      for (int br = 0; br < c; ++br) r += 1 + N.span[r];
      flatten_range(N, r + 1, r + 1 + N.span[r], 0, F);
    } else {
      const int trips = N.site_lo[s] + c;
      const bool rev = N.flags[q] & 1;
      for (int i = 0; i < trips; ++i) {
        F.at.push_back({0, -1, 0, 0, 0});
        flatten_range(N, q + 1, q + 1 + N.span[q], rev ? trips - 1 - i : i, F);
      }
      F.at.push_back({0, -1, 0, 0, 0});
    }
    q += 1 + N.span[q];
  }
  return F;
}

struct Search {
  const NestArch& N;
  const Flat& F;
  std::vector<std::array<int64_t, 10>> pred;
  int g = 0;
  std::array<int64_t, 10> acc{};
  std::vector<int32_t> rows_op, rows_it, nested;
  std::unordered_set<StateKey, StateHash> failed;
  size_t memo_cap = 4u << 20;

  Search(const NestArch& n, const Flat& f) : N(n), F(f) {}

  bool row(int op, int it) {
    if (g >= (int)pred.size()) return false;
    acc[0] += 1;
    if (op >= 0) {
      const int32_t* s = &N.sig[(size_t)op * 9];
      for (int e = 0; e < 9; ++e) acc[1 + e] += s[e];
    }
    const auto& p = pred[g];
    for (int e = 0; e < 10; ++e)
      if (std::min<int64_t>(acc[e], kSat) > p[e]) return false;
    if (acc[0] == p[0]) {
      for (int e = 0; e < 10; ++e)
        if (std::min<int64_t>(acc[e], kSat) != p[e]) return false;
      ++g;
      acc.fill(0);
    }
    rows_op.push_back(op);
    rows_it.push_back(it);
    return true;
  }

  bool go(int pos) {
    const int n = (int)F.at.size();
    while (pos < n && F.at[pos].type == 0) {
      if (!row(F.at[pos].op, F.at[pos].it)) return false;
      ++pos;
    }
    if (pos == n) {
      if (g != (int)pred.size()) return false;
      for (int64_t x : acc)
        if (x) return false;
      return true;
    }
    StateKey key{pos, g, acc};
    if (failed.count(key)) return false;
    const Atom& c = F.at[pos];
    const int g0 = g;
    const auto acc0 = acc;
    const size_t r0 = rows_op.size(), n0 = nested.size();
    for (int a = 0; a < c.narm; ++a) {
      nested.push_back(a);
      const Arm& arm = F.arms[c.arm0 + a];
      bool ok = true;
      for (int q = 0; q < arm.n_ops && ok; ++q) ok = row(arm.first_op + q, c.it);
      if (ok && go(pos + 1)) return true;
      g = g0;
      acc = acc0;
      rows_op.resize(r0);
      rows_it.resize(r0);
      nested.resize(n0);
    }
    if (failed.size() < memo_cap) failed.insert(key);
    return false;
  }
};

}  // namespace

dyo_status nested_decode(const NestArch& N, const int32_t* slots, int K_max, const int32_t* top_choices,
                         std::vector<int32_t>& path_op, std::vector<int32_t>& path_it, std::vector<int32_t>& nested,
                         int* matched, std::string& err) {
  const Flat F = flatten(N, top_choices);
  Search S(N, F);
  int64_t total = 0;
  for (int k = 0; k < K_max; ++k) {
    if (slots[k * 10] == 0) continue;
    std::array<int64_t, 10> v;
    for (int e = 0; e < 10; ++e) v[e] = slots[k * 10 + e];
    S.pred.push_back(v);
    total += v[0];
  }
  if (S.go(0)) {
    path_op = S.rows_op;
    path_it = S.rows_it;
    nested = S.nested;
    *matched = 1;
    return DYO_OK;
  }
  // ---- fallback: closest operator count, first in lexicographic order ----
  *matched = 0;
  std::vector<int> cp;                         // choice points in order
  int64_t stat = 0;
  for (int i = 0; i < (int)F.at.size(); ++i) {
    if (F.at[i].type == 1) cp.push_back(i);
    else ++stat;
  }
  const int m = (int)cp.size();
  int64_t maxL = 0;
  for (int i : cp) {
    int64_t mx = 0;
    for (int a = 0; a < F.at[i].narm; ++a) mx = std::max<int64_t>(mx, F.arms[F.at[i].arm0 + a].n_ops);
    maxL += mx;
  }
  const int64_t W = maxL + 1;
  if ((double)(m + 1) * (double)W > (double)(1ll << 31)) {
    err = "nested decode fallback: reachable-length table too large";
    return DYO_E_CAPACITY;
  }
  std::vector<std::vector<uint8_t>> R(m + 1, std::vector<uint8_t>(W, 0));
  R[m][0] = 1;
  for (int i = m - 1; i >= 0; --i) {
    const Atom& c = F.at[cp[i]];
    for (int64_t v = 0; v < W; ++v)
      if (R[i + 1][v])
        for (int a = 0; a < c.narm; ++a) {
          const int64_t l = F.arms[c.arm0 + a].n_ops;
          if (v + l < W) R[i][v + l] = 1;
        }
  }
  int64_t dmin = INT64_MAX;
  for (int64_t v = 0; v < W; ++v)
    if (R[0][v]) dmin = std::min<int64_t>(dmin, std::llabs(stat + v - total));
  int64_t pre = stat;
  nested.clear();
  for (int i = 0; i < m; ++i) {
    const Atom& c = F.at[cp[i]];
    int pick = -1;
    for (int a = 0; a < c.narm && pick < 0; ++a) {
      const int64_t base = pre + F.arms[c.arm0 + a].n_ops;
      for (int64_t tgt : {total - dmin, total + dmin}) {
        const int64_t v = tgt - base;
        if (v >= 0 && v < W && R[i + 1][v]) { pick = a; break; }
      }
    }
    if (pick < 0) { err = "nested decode fallback: internal inconsistency"; return DYO_E_INVAL; }
    nested.push_back(pick);
    pre += F.arms[c.arm0 + pick].n_ops;
  }
  path_op.clear();
  path_it.clear();
  int ci = 0;
  for (const Atom& a : F.at) {
    if (a.type == 0) {
      path_op.push_back(a.op);
      path_it.push_back(a.it);
    } else {
      const Arm& arm = F.arms[a.arm0 + nested[ci++]];
      for (int q = 0; q < arm.n_ops; ++q) {
        path_op.push_back(arm.first_op + q);
        path_it.push_back(a.it);
      }
    }
  }
  return DYO_OK;
}

dyo_status trace_path(const NestArch& N, const int32_t* choices, const int32_t* nested, int n_nested,
                      std::vector<int32_t>& path_op, std::vector<int32_t>& path_it, std::string& err) {
  const Flat F = flatten(N, choices);
  path_op.clear();
  path_it.clear();
  int ci = 0;
  for (const Atom& a : F.at) {
    if (a.type == 0) {
      path_op.push_back(a.op);
      path_it.push_back(a.it);
      continue;
    }
    if (ci >= n_nested) { err = "trace: fewer nested choices than nested executions"; return DYO_E_INVAL; }
    const int c = nested[ci++];
    if (c < 0 || c >= a.narm) { err = "trace: nested choice out of range"; return DYO_E_INVAL; }
    const Arm& arm = F.arms[a.arm0 + c];
    for (int q = 0; q < arm.n_ops; ++q) {
      path_op.push_back(arm.first_op + q);
      path_it.push_back(a.it);
    }
  }
  if (ci != n_nested) { err = "trace: more nested choices than nested executions"; return DYO_E_INVAL; }
  return DYO_OK;
}

}  // namespace dyo
