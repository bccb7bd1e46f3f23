"""Oracle pins for the mis-prediction record + exact-match memo (reading
R15): closed-form mis-prediction counts over repeated samples, the memo-resolved prediction equal
to the textbook resolution of the actual control flow, FIFO capacity, most-recent-wins, and the
validity rule for reported choices."""
import numpy as np
import pytest

import workloads as WL
from oracle import afm as A, decode as D, encode as E, memo as M, pilot as P

pytestmark = pytest.mark.filterwarnings("ignore")


def _logits(wl, s):
    x = E.encode(wl, wl.samples[s], wl.hist_ids, ())
    return P.forward(wl.pilot, x, wl.nn_type)


@pytest.fixture(scope="module")
def tiny():
    wl = WL.make("tiny", n_samples=16)
    ys = [_logits(wl, s) for s in range(len(wl.samples))]
    preds = [D.decode(wl, y) for y in ys]
    acts = [WL.actual_choices(wl, s) for s in range(len(wl.samples))]
    return wl, ys, preds, acts


def test_correct_prediction_is_not_recorded(tiny):
    wl, ys, preds, acts = tiny
    m = M.Memo()
    assert m.report(preds[0], preds[0].choices) is False
    assert m.mispredictions == 0 and not m.table


def test_hit_resolves_the_actual_control_flow(tiny):
    wl, ys, preds, acts = tiny
    bad = [s for s in range(len(ys)) if list(acts[s]) != list(preds[s].choices)]
    assert bad, "the seeded tiny stream must contain mis-predictions"
    m = M.Memo()
    for s in bad:
        assert m.report(preds[s], acts[s], sample=s)
    for s in bad:
        got, hit = M.decode_with_memo(wl, ys[s], m)
        assert hit
        # the path is the actual control flow's resolution (A.resolve = the R2 rows), found
        # independently among the enumerated paths of the program
        # (samples sharing an output share the most recent report's actual choices)
        want = m.lookup(preds[s])
        paths = {tuple(c): list(p) for c, p in D.enumerate_paths(wl.program)}
        assert list(got.path) == list(paths[tuple(want)])
        assert got.choices == list(want)
        # cut at the PREDICTED counts (R4) and tensor sets of the actual rows
        counts = [v[0] for v in preds[s].slots if v[0] != 0]
        assert got.groups == D.cut(len(got.path), counts)
        assert got.W == D.tensor_sets(got.path, got.groups)
        assert got.blocks == [A.block10(got.path[a:b]) for a, b in got.groups]


def test_closed_form_counts_over_repeats(tiny):
    """D distinct samples, each repeated r times: without the memo every repeat of a
    mis-predicted sample is mis-predicted again (r*m); with it only the first is (m), when the
    mis-predicted samples' outputs are pairwise distinct (P:L280 'avoid repeated mis-prediction')."""
    wl, ys, preds, acts = tiny
    keys = {}
    for s in range(len(ys)):
        keys.setdefault(M.key_of(preds[s]), []).append(s)
    distinct = [v[0] for v in keys.values() if all(list(acts[t]) == list(acts[v[0]]) for t in v)]
    r = 3
    m_bad = sum(1 for s in distinct if list(acts[s]) != list(preds[s].choices))
    without = M.Memo()
    with_m = M.Memo()
    for _ in range(r):
        for s in distinct:
            without.report(preds[s], acts[s])
            got, hit = M.decode_with_memo(wl, ys[s], with_m)
            with_m.report(got, acts[s])
            without.table.clear()
            without.order.clear()
    assert without.mispredictions == r * m_bad
    assert with_m.mispredictions == m_bad


def test_fifo_capacity_and_most_recent_wins(tiny):
    wl, ys, preds, acts = tiny
    bad = [s for s in range(len(ys)) if list(acts[s]) != list(preds[s].choices)
           and M.key_of(preds[s]) != M.key_of(preds[0])]
    a, b = bad[0], next(s for s in bad if M.key_of(preds[s]) != M.key_of(preds[bad[0]]))
    m = M.Memo(capacity=1)
    m.report(preds[a], acts[a])
    m.report(preds[b], acts[b])
    assert m.lookup(preds[a]) is None and m.lookup(preds[b]) == tuple(acts[b])
    # same output reported twice with different actual choices: the later one is kept
    alt = [(c + 1) % A.n_choices(site) if site.tie < 0 else None for c, site in zip(acts[b], A.sites(wl.program))]
    sl = A.sites(wl.program)
    for i, site in enumerate(sl):
        if site.tie >= 0:
            alt[i] = alt[site.tie]
    m2 = M.Memo()
    m2.report(preds[b], acts[b])
    m2.report(preds[b], alt)
    assert m2.lookup(preds[b]) == tuple(alt) and len(m2.table) == 1


def test_valid_choices_rule():
    wl = WL.make("moe", n_samples=2)
    c = WL.actual_choices(wl, 1)
    assert M.valid_choices(wl.program, c)
    sl = A.sites(wl.program)
    tied = next(i for i, s in enumerate(sl) if s.tie >= 0)
    bad = list(c)
    bad[tied] = (bad[tied] + 1) % A.n_choices(sl[tied])
    assert not M.valid_choices(wl.program, bad)
    assert not M.valid_choices(wl.program, c[:-1])
