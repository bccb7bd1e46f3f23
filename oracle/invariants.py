"""Plan invariants I1-I7 (DESIGN.md §4 table, north_star).

Oracle — test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

from .plan import HOST, half_size, aligned, transition
from .migrate import VersionSim


def check_layout(state, wl):
    """I1: in each half, resident tensors occupy disjoint aligned ranges inside [0, H)."""
    H = half_size(wl.budget, wl.align)
    for half in (0, 1):
        iv = sorted((state.off[t], state.off[t] + aligned(wl.tensors[t].nbytes, wl.align), t)
                    for t in range(len(wl.tensors)) if state.loc[t] == half)
        end = 0
        for s, e, t in iv:
            assert s >= end, f"I1 overlap at tensor {t} in half {half}"
            end = e
        assert end <= H, f"I1: half {half} uses {end} > H={H}"


def run_checked(state, wl, Ws, policy, vs=None):
    """Plan a step transition by transition and assert I1-I5 on the way; returns
    (transitions, final_state)."""
    import copy
    st = copy.deepcopy(state)
    H = half_size(wl.budget, wl.align)
    vs = VersionSim(wl) if vs is None else vs
    vs.new_step()
    for t, ten in enumerate(wl.tensors):      # as plan(): transient contents end with the step
        if ten.transient:
            st.dirty[t] = False
    trs = []
    for j in range(len(Ws)):
        prev_set = {t for t, _, _ in st.prev}
        tr = transition(st, wl, Ws, j, policy)
        # I3: nothing block j-1 uses is evicted or compacted at transition j
        assert not prev_set & {r[0] for r in tr.evict}, "I3 evict"
        assert tr.late_all or not prev_set & {r[0] for r in tr.move}, "I3 move"   # R20: late_all waits
        check_layout(st, wl)
        shared = {t for t, _ in tr.share}
        for t, _, _ in Ws[j]:                       # I2: W_j resident in half m (or SHARE'd, R20)
            assert st.loc[t] == tr.half or (t in shared and st.loc[t] == 1 - tr.half), \
                f"I2: tensor {t} not in half {tr.half}"
        vs.apply(tr)
        bad = vs.run_block(Ws[j], tr.half, st, H)   # I4/I5 via versions read by block j
        assert not bad, f"stale read of tensors {bad} at block {j}"
        trs.append(tr)
    st.G += len(Ws)
    return trs, st, vs


def host_current(state, wl, vs):
    """I5 at a step boundary: every non-resident non-transient tensor's host home holds its
    latest version."""
    for t, ten in enumerate(wl.tensors):
        if state.loc[t] == HOST and not ten.transient:
            assert vs.host_ver[t] == vs.ver[t], f"I5: host home of {t} is stale"
