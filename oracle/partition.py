"""Partition of an execution trace into execution blocks - the pilot's training labels
(§IV-D: Sentinel-style labels that "maximize the overlap between tensor
migration and training computation without violating the GPU memory capacity"; §V L203-L205 the
partition simulator; §VI-G L275 the three heuristics it is compared with). DESIGN.md reading R18.

Oracle - test infrastructure only (see oracle/__init__.py).

Trace: the rows of a resolved path (Op or None for a control row) with per-row compute times
(integer ns). A partition cuts the rows into K non-empty consecutive blocks. For block j = rows
[s, e):
  need(s, e)  = aligned bytes of the block's tensor set W_j (R8)            (capacity: <= H, R7)
  fetch(s, e) = bytes of the tensors the block reads first (R8 needs_fetch) (migrated for it)
  comp(s, e)  = sum of the rows' compute times (ns)
Block j's migration overlaps block j-1's compute (P:L176 double buffer): its exposed time is
max(0, xfer(fetch_j) - comp_{j-1}) with xfer(b) = ceil(b * 1000 / bw) ns for a link of bw bytes
per microsecond; block 0's migration has nothing to hide behind and is left out (the same for
every partition). The overlap partition minimises the total exposed time subject to need <= H
for every block; ties go to the lexicographically smallest vector of cut positions. Everything is
integer, so the result is exact. The heuristics (L275) cut at even operator counts, even compute
time and even tensor bytes.
"""
from __future__ import annotations

import math

from workloads import R
from . import decode as D

INF = float("inf")


def block_tables(rows, times, tensors, align):
    """need/fetch/comp of every block [s, e), 0 <= s < e <= L (plain nested loops)."""
    L = len(rows)
    a = [(t.nbytes + align - 1) // align * align for t in tensors]
    need = [[0] * (L + 1) for _ in range(L + 1)]
    fetch = [[0] * (L + 1) for _ in range(L + 1)]
    comp = [[0] * (L + 1) for _ in range(L + 1)]
    for s in range(L):
        for e in range(s + 1, L + 1):
            W = D.tensor_sets(rows, [(s, e)])[0]
            need[s][e] = sum(a[t] for t, _, _ in W)
            fetch[s][e] = sum(tensors[t].nbytes for t, _, rd in W if rd)
            comp[s][e] = sum(times[s:e])
    return need, fetch, comp


def xfer(nbytes, bw):
    """Transfer time (ns, rounded up) of nbytes over bw bytes per microsecond."""
    return -(-nbytes * 1000 // bw)


def exposed(cuts, fetch, comp, bw):
    """Total exposed migration time (ns) of the partition given by its cut positions
    [0 = c_0 < c_1 < ... < c_K = L]: sum over blocks j >= 1 of max(0, xfer(fetch_j) - comp_{j-1})."""
    tot = 0
    for j in range(1, len(cuts) - 1):
        tot += max(0, xfer(fetch[cuts[j]][cuts[j + 1]], bw) - comp[cuts[j - 1]][cuts[j]])
    return tot


def feasible(cuts, need, H):
    return all(need[cuts[j]][cuts[j + 1]] <= H for j in range(len(cuts) - 1))


def overlap_partition(L, K, need, fetch, comp, H, bw):
    """The overlap-maximising partition (R18): among the cut vectors 0 = c_0 < ... < c_K = L with
    need(c_j, c_{j+1}) <= H for every block, the minimum total exposed time; among the
    minimisers, the lexicographically smallest cut vector. Written as a suffix recurrence over
    (block j = [s, e)):
      f[K-1][s][L] = 0                                          (the last block ends at L)
      f[j][s][e]   = min over e' > e with need(e, e') <= H of
                     max(0, xfer(fetch(e, e')) - comp(s, e)) + f[j+1][e][e']
    OPT = min over c_1 with need(0, c_1) <= H of f[0][0][c_1]; the cuts are then chosen front to
    back, each the smallest that still reaches the optimum (exact integer equality). Returns
    (cuts, exposed) or (None, inf) if no feasible partition."""
    f = [[[INF] * (L + 1) for _ in range(L + 1)] for _ in range(K)]
    for s in range(L):
        if need[s][L] <= H:
            f[K - 1][s][L] = 0
    for j in range(K - 2, -1, -1):
        for s in range(L):
            for e in range(s + 1, L):
                best = INF
                for e2 in range(e + 1, L + 1):
                    if need[e][e2] <= H and f[j + 1][e][e2] < INF:
                        best = min(best, max(0, xfer(fetch[e][e2], bw) - comp[s][e]) + f[j + 1][e][e2])
                f[j][s][e] = best
    opt = min((f[0][0][c] for c in range(1, L + 1) if need[0][c] <= H), default=INF)
    if opt == INF:
        return None, INF
    cuts = [0, next(c for c in range(1, L + 1) if need[0][c] <= H and f[0][0][c] == opt)]
    rem = opt
    for j in range(1, K):
        s, e = cuts[-2], cuts[-1]
        for e2 in range(e + 1, L + 1):
            if need[e][e2] <= H and f[j][e][e2] < INF:
                step = max(0, xfer(fetch[e][e2], bw) - comp[s][e])
                if step + f[j][e][e2] == rem:
                    cuts.append(e2)
                    rem -= step
                    break
    return cuts, opt


def even_partition(weights, K):
    """Cut j (j = 1..K-1) after the longest prefix whose integer weight W(p) satisfies
    W(p) * K <= total * j, clamped to [c_{j-1} + 1, L - (K - j)] so every block is non-empty: the
    L275 heuristics with weights = 1 per operator row (even operators; control rows weigh 0),
    compute time (even time), or the bytes of the tensors a row accesses (even size)."""
    L = len(weights)
    tot = sum(weights)
    pref = [0]
    for w in weights:
        pref.append(pref[-1] + w)
    cuts = [0]
    for j in range(1, K):
        p = max(i for i in range(L + 1) if pref[i] * K <= tot * j)
        cuts.append(max(cuts[-1] + 1, min(p, L - (K - j))))
    cuts.append(L)
    return cuts


def heuristic_weights(rows, times, tensors, kind):
    if kind == "ops":
        return [0 if r is None else 1 for r in rows]
    if kind == "time":
        return list(times)
    if kind == "size":
        return [0 if r is None else sum(tensors[t].nbytes for t, _ in r.acc) for r in rows]
    raise ValueError(kind)


def labels(rows, cuts, K_max):
    """The pilot-training label (L164: the pilot output format, L143): the block vectors of the
    blocks, then zero slots up to K_max."""
    from . import afm as A
    out = [A.block10(rows[cuts[j]:cuts[j + 1]]) for j in range(len(cuts) - 1)]
    return out + [(0,) * 10] * (K_max - len(out))
