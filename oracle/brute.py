"""Brute-force optimal retention on tiny instances (north_star "brute-force optimal eviction
on tiny budgets"; DESIGN.md §5 plan pins).

Oracle — test infrastructure only (see oracle/__init__.py).

two_half_opt: enumerate every retention subset of the live candidates at every transition
              of the two-half model (oracle/plan.transition with an explicit choice) and
              minimise total H2D + D2H bytes.
pool_belady / pool_opt: POOL mode — one arena of capacity C tensors (uniform sizes, read-only
              tensors), protected set W_{j-1} u W_j; Belady's farthest-next-use rule as the
              prefix cut of plan.prefix_cut versus exhaustive search of every retained set.
"""
from __future__ import annotations

import copy
from itertools import combinations

from .plan import transition, BudgetError, prefix_cut, INF


def _subsets(live, room):
    items = [(a, t) for _, a, t in live]
    out = []
    for r in range(len(items) + 1):
        for comb in combinations(items, r):
            if sum(a for a, _ in comb) <= room:
                out.append([t for _, t in comb])
    return out


def two_half_opt(state, wl, Ws, start=0):
    """Minimum total (H2D + D2H) bytes over all retention choices; returns (bytes, choices)."""
    if start == len(Ws):
        return 0, []
    best = None
    probe = copy.deepcopy(state)
    options = []

    def grab(live, room):
        options.extend(_subsets(live, room))
        return []
    try:
        transition(probe, wl, Ws, start, 0, choose=grab)
    except BudgetError:
        return None, None
    for keep in options:
        st = copy.deepcopy(state)
        tr = transition(st, wl, Ws, start, 0, choose=lambda live, room, k=keep: k)
        rest, ch = two_half_opt(st, wl, Ws, start + 1)
        if rest is None:
            continue
        cost = tr.h2d + tr.d2h + rest
        if best is None or cost < best[0]:
            best = (cost, [keep] + ch)
    return best if best else (None, None)


def _pool_next(Ws, t, j):
    for jj in range(j + 1, len(Ws)):
        if t in Ws[jj]:
            return jj - j
    return INF


def pool_run(C, Ws, chooser):
    """POOL mode: returns number of fetches. Ws: list of sets of tensor ids."""
    S = set()
    fetches = 0
    prev = set()
    for j, Wj in enumerate(Ws):
        prot = set(Wj) | prev
        if len(prot) > C:
            raise BudgetError("pool infeasible")
        fetches += len(set(Wj) - S)
        cands = [(_pool_next(Ws, t, j), 1, t) for t in sorted(S - prot)]
        keep = chooser(cands, C - len(prot), j)
        S = prot | set(keep)
        prev = set(Wj)
    return fetches


def pool_belady(C, Ws):
    return pool_run(C, Ws, lambda cands, room, j: prefix_cut(cands, room))


def pool_opt(C, Ws):
    """Exhaustive search over every retained subset at every step."""
    def rec(j, S, prev):
        if j == len(Ws):
            return 0
        Wj = set(Ws[j])
        prot = Wj | prev
        f = len(Wj - S)
        cands = sorted(S - prot)
        room = C - len(prot)
        best = None
        for r in range(min(room, len(cands)) + 1):
            for comb in combinations(cands, r):
                v = rec(j + 1, prot | set(comb), Wj)
                if best is None or v < best:
                    best = v
        return f + best
    return rec(0, set(), set())
