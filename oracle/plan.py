"""Double-buffered evict/prefetch plan (§IV-E, §V;
DESIGN.md readings R7-R12). Integer-only.

Oracle — test infrastructure only (see oracle/__init__.py).

Model: the device budget B is split into two equal halves H = floor(B/2/ALIGN)*ALIGN.
Block j (global counter G+j) runs from half m = (G+j) mod 2 while transition j+1 prepares the
other half; so transition j re-lays-out half m, which block j-1 does not touch (R7).
Transition j, in order:
  1. infeasible if the aligned bytes of W_j exceed H (R7)
  2. classify W_j: in half m -> KEEP; valid in half 1-m and read first -> CARRY (D2D; `late`
     if block j-1 writes it, R8); not valid and read first -> FETCH; written first -> ALLOC
  3. other valid tensors of half m are eviction candidates: dead ones (R9) are freed; the
     live ones are evicted all (PAPER policy, "evict unused tensors") or, under RETAIN,
     sorted by (next-use distance, aligned size, id) and the longest prefix fitting in
     H - need(W_j) is kept (Belady as a prefix cut, north_star "top-k over sizes and reuse
     distance"); an evicted live dirty tensor is written back (R10)
  4. half m layout (R11): kept tensors stay in place; CARRY (by id), ALLOC (by id), FETCH (by
     host offset) go first-fit into the free gaps; only if a tensor finds no gap is the half
     compacted: exclusive prefix sums over [kept by old offset | CARRY | ALLOC | FETCH]
  5. operation order (P:L180 evict first, then prefetch): EVICT writebacks, MOVE (compaction,
     ascending destination), CARRY, FETCH; then block j marks its written tensors dirty.

Policy bit SHARE (reading R20): a tensor of W_j valid in half 1-m that the next group
W_{j+1} also holds stays where it is (SHARE, no copy, no space in half m): block j reads it in
the other half, and transition j+1 finds it in its own half (KEEP). While block j runs, transition
j+1 must not move it, so a compaction of a half holding tensors of the running block waits for
that block's end (the transition is `late_all`: its MOVE / CARRY / FETCH run after block j-1).
Without SHARE every W_j tensor is in half m when block j starts (R1: ping-pong by D2D).
"""
from __future__ import annotations

from dataclasses import dataclass, field
import copy

from workloads import R, W

HOST = -1
INF = 1 << 62
PAPER, RETAIN = 0, 1
SHARE = 2          # policy bit (R20); policy & 1 selects RETAIN


class BudgetError(Exception):
    pass


@dataclass
class State:
    loc: list
    off: list
    dirty: list
    prev: list = field(default_factory=list)   # W entries of the last executed group
    G: int = 0                                  # global block counter


def initial_state(n_tensors):
    """Every tensor starts in CPU memory (P:L197 'initially allocates all tensors on CPU')."""
    return State([HOST] * n_tensors, [0] * n_tensors, [False] * n_tensors, [], 0)


@dataclass
class Transition:
    j: int
    half: int
    need: int
    evict: list      # (t, src_abs, host_off, nbytes, writeback)
    move: list       # (t, old_abs, new_abs, nbytes)
    carry: list      # (t, src_abs, dst_abs, nbytes, late)
    alloc: list      # (t, dst_abs, nbytes)
    fetch: list      # (t, host_off, dst_abs, nbytes)
    share: list = field(default_factory=list)   # (t, abs) of the W_j tensors left in half 1-m (R20)
    late_all: bool = False                      # R20: MOVE / CARRY / FETCH wait for block j-1's end
    h2d: int = 0
    d2h: int = 0
    d2d: int = 0


def half_size(budget, align):
    return budget // 2 // align * align


def aligned(nbytes, align):
    return (nbytes + align - 1) // align * align


def tensor_table(wl):
    """(aligned sizes, byte sizes, host offsets) of every tensor, cached on the workload."""
    key = (wl.align, len(wl.tensors))
    cached = getattr(wl, "_oracle_tensor_table", None)
    if cached is None or cached[0] != key:
        a = [aligned(t.nbytes, wl.align) for t in wl.tensors]
        cached = (key, (a, [t.nbytes for t in wl.tensors], [t.host_off for t in wl.tensors]))
        wl._oracle_tensor_table = cached
    return cached[1]


def occurrences(Ws):
    """occ[t] = [(j, entry), ...] in ascending j: every group whose tensor set holds t."""
    occ = {}
    for jj, Wj in enumerate(Ws):
        for e in Wj:
            occ.setdefault(e[0], []).append((jj, e))
    return occ


def next_use(Ws, t, j, occ=None):
    """(distance to the first group j' > j whose tensor set holds t, that entry) or (INF, None).
    occ (from occurrences(Ws)) only indexes the same search."""
    if occ is None:
        occ = occurrences(Ws)
    for jj, e in occ.get(t, ()):
        if jj > j:
            return jj - j, e
    return INF, None


def prefix_cut(cands, room):
    """cands: list of (distance, aligned_size, tensor_id). Sort ascending and keep the longest
    prefix whose cumulative aligned size fits in `room` (no skip-and-continue)."""
    kept, used = [], 0
    for d, a, t in sorted(cands):
        if used + a > room:
            break
        kept.append(t)
        used += a
    return kept


def first_fit(kept, placed, off, a, H):
    """Reading R11: kept tensors stay in place; each placed tensor (in the given order) takes
    the start of the lowest-addressed free gap of [0, H) that can hold its aligned size.
    Returns {tensor: offset} or None when some tensor finds no gap."""
    gaps, cur = [], 0
    for t in kept:                      # kept is in ascending offset
        if off[t] > cur:
            gaps.append([cur, off[t]])
        cur = off[t] + a[t]
    if H > cur:
        gaps.append([cur, H])
    new_off = {t: off[t] for t in kept}
    for t in placed:
        for g in gaps:
            if g[1] - g[0] >= a[t]:
                new_off[t] = g[0]
                g[0] += a[t]
                break
        else:
            return None
    return new_off


def transition(state, wl, Ws, j, policy, choose=None, occ=None):
    """Plan transition j in place on `state`. `choose(live, room)` overrides the retention
    choice (brute force); default is the policy's. occ: occurrences(Ws), to share the index."""
    if occ is None:
        occ = occurrences(Ws)
    T = len(wl.tensors)
    H = half_size(wl.budget, wl.align)
    a, nb, host_off = tensor_table(wl)
    m = (state.G + j) % 2
    Wj = Ws[j]
    in_w = {t for t, _, _ in Wj}
    prev_written = {t for t, mode, _ in state.prev if mode & W}
    share_on = bool(policy & SHARE)
    nxt = {t for t, _, _ in Ws[j + 1]} if share_on and j + 1 < len(Ws) else set()
    # R20: tensors of the running block j-1 in half m (left there by SHARE at transition j-1)
    pinned = {t for t, _, _ in state.prev if state.loc[t] == m}

    keep, carry, alloc, fetch, share = [], [], [], [], []
    for t, mode, rd in Wj:
        if state.loc[t] == m:
            keep.append(t)
        elif state.loc[t] == 1 - m and t in nxt:
            share.append(t)
        elif state.loc[t] == 1 - m and rd:
            carry.append(t)
        elif rd:
            fetch.append(t)
        else:
            alloc.append(t)
    shared = set(share)
    need = sum(a[t] for t, _, _ in Wj if t not in shared)
    if need > H:
        raise BudgetError(f"transition {j}: W_j needs {need} B > H = {H} B")

    # eviction candidates: other valid tensors of half m
    cands = [t for t in range(T) if state.loc[t] == m and t not in in_w]
    live, dead = [], []
    for t in cands:
        d, e = next_use(Ws, t, j, occ)
        # R9: only a transient tensor can be dead (no later access, or its next access writes it
        # first); a persistent tensor is never dropped on a predicted overwrite (R17: under a
        # mis-prediction the overwrite may not happen)
        is_dead = wl.tensors[t].transient and (e is None or not e[2])
        if is_dead:
            dead.append(t)
        else:
            live.append((d, a[t], t))
    room = H - need
    if choose is not None:
        retained = list(choose(live, room))
    elif policy & RETAIN:                  # bit 0 (bit 1 is SHARE, R20)
        retained = prefix_cut(live, room)
    else:
        retained = []
    assert sum(a[t] for t in retained) <= room
    rset = set(retained)
    evicted = dead + [t for _, _, t in live if t not in rset]

    evict = sorted(((t, m * H + state.off[t], host_off[t], nb[t],
                     bool(state.dirty[t]) and t not in dead) for t in evicted),
                   key=lambda r: (r[2], r[0]))

    kept_all = sorted(keep + retained, key=lambda t: state.off[t])
    placed = sorted(carry) + sorted(alloc) + sorted(fetch, key=lambda t: (host_off[t], t))
    new_off = first_fit(kept_all, placed, state.off, a, H)
    late_all = False
    if new_off is None:                   # fragmentation: compact (R11 fallback)
        late_all = bool(pinned)           # R20: it moves tensors block j-1 is using: after its end
        new_off, cur = {}, 0
        for t in kept_all + placed:
            new_off[t] = cur
            cur += a[t]
        assert cur <= H
    order = kept_all + placed

    move = [(t, m * H + state.off[t], m * H + new_off[t], nb[t])
            for t in kept_all if new_off[t] != state.off[t]]
    carry_l = [(t, (1 - m) * H + state.off[t], m * H + new_off[t], nb[t], t in prev_written)
               for t in sorted(carry)]
    alloc_l = [(t, m * H + new_off[t], nb[t]) for t in sorted(alloc)]
    fetch_l = [(t, host_off[t], m * H + new_off[t], nb[t])
               for t in sorted(fetch, key=lambda t: (host_off[t], t))]

    tr = Transition(j, m, need, evict, move, carry_l, alloc_l, fetch_l,
                    [(t, (1 - m) * H + state.off[t]) for t in share], late_all)
    tr.h2d = sum(r[3] for r in fetch_l)
    tr.d2h = sum(r[3] for r in evict if r[4])
    tr.d2d = sum(r[3] for r in move) + sum(r[3] for r in carry_l)

    # state update
    for t in evicted:
        state.loc[t] = HOST
        state.dirty[t] = False
    for t in order:
        state.loc[t] = m
        state.off[t] = new_off[t]
    for t in fetch + alloc:
        state.dirty[t] = False
    for t, mode, _ in Wj:          # block j runs: written tensors become dirty
        if mode & W:
            state.dirty[t] = True
    state.prev = list(Wj)
    return tr


def plan(state, wl, Ws, policy=None):
    """Plan all transitions of one step's prediction. Transactional: on BudgetError the
    caller's state is unchanged. Returns (transitions, new_state)."""
    policy = wl.policy if policy is None else policy
    st = copy.deepcopy(state)
    for t, ten in enumerate(wl.tensors):      # R9: a transient tensor's contents end with the step
        if ten.transient:
            st.dirty[t] = False
    occ = occurrences(Ws)
    trs = [transition(st, wl, Ws, j, policy, occ=occ) for j in range(len(Ws))]
    st.G += len(Ws)
    return trs, st
