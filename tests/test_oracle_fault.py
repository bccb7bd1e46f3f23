"""Pins for oracle/fault.py (reading R17: on-demand fetch of mis-predicted tensors, P:L184,
P:L197) and the DYO_FAULT drop injection of workloads."""
import numpy as np

import workloads as WL
from workloads import R, W, RW
from oracle import fault as F, encode as E, pilot as P, decode as D, afm as A


def test_classify_hand_cases():
    planned = [(1, R, True), (2, W, False), (4, R, True), (5, RW, True)]
    actual = [(1, R, True), (2, RW, True), (3, R, True), (4, RW, True), (5, RW, True), (6, W, False)]
    assert F.classify(planned, actual) == [
        (1, R, "slot"),        # fetched as planned
        (2, RW, "fault"),      # planned write-first (ALLOC, no bytes fetched), read first here
        (3, R, "fault"),       # not planned
        (4, RW, "fault"),      # planned read-only: a write the plan does not know about
        (5, RW, "slot"),
        (6, W, "fault")]       # not planned, written first: a fault-area slot, nothing copied in


def test_no_misprediction_no_fault():
    """Actual control flow = the predicted one: the actual blocks are the predicted ones and
    every access is served from its planned slot."""
    wl = WL.make("moe", n_samples=4)
    for s in range(4):
        x = E.encode(wl, wl.samples[s], wl.hist_ids, ())
        pred = D.decode(wl, P.forward(wl.pilot, x, wl.nn_type))
        counts = [v[0] for v in pred.slots if v[0]]
        act, groups = F.actual_sets(wl, pred.choices, counts)
        assert act == pred.W and groups == pred.groups
        assert all(k == "slot" for Wj, Aj in zip(pred.W, act) for _, _, k in F.classify(Wj, Aj))


def test_mispredicted_expert_faults_exactly_the_actual_expert():
    """MoE: with the actual routing of one layer changed, the faults are the tensors the actual
    block touches that the predicted one does not (the other expert's weights), nothing else."""
    wl = WL.make("moe", n_samples=4)
    x = E.encode(wl, wl.samples[0], wl.hist_ids, ())
    pred = D.decode(wl, P.forward(wl.pilot, x, wl.nn_type))
    counts = [v[0] for v in pred.slots if v[0]]
    act_choices = list(pred.choices)
    sl = A.sites(wl.program)
    first = next(i for i, s in enumerate(sl) if s.tie < 0)
    act_choices[first] = (act_choices[first] + 1) % A.n_choices(sl[first])
    for i, s in enumerate(sl):                   # tied sites replay (R6)
        if s.tie >= 0:
            act_choices[i] = act_choices[s.tie]
    act, _ = F.actual_sets(wl, act_choices, counts)
    n_fault = 0
    for Wj, Aj in zip(pred.W, act):
        planned = {t for t, _, _ in Wj}
        for t, m, k in F.classify(Wj, Aj):
            assert (k == "fault") == (t not in planned or any(t == u and (not rd and m & R) for u, _, rd in Wj))
            n_fault += k == "fault"
    assert n_fault > 0


def test_drop_prefetch_injection():
    wl = WL.make("tiny", n_samples=4)
    x = E.encode(wl, wl.samples[0], wl.hist_ids, ())
    pred = D.decode(wl, P.forward(wl.pilot, x, wl.nn_type))
    assert WL.drop_prefetch(pred.W, 0.0, 1, 0) == pred.W
    allw = WL.drop_prefetch(pred.W, 1.0, 1, 0)
    assert all(not rd for Wj in allw for _, _, rd in Wj)
    half = WL.drop_prefetch(pred.W, 0.5, 7, 0)
    kept = sum(len(Wj) for Wj in half)
    assert 0 < kept < sum(len(Wj) for Wj in pred.W)
    # the dropped entries are exactly the faults of the undropped (actual) blocks
    for Wj, Hj in zip(pred.W, half):
        dropped = {t for t, _, _ in Wj} - {t for t, _, _ in Hj}
        assert {t for t, _, k in F.classify(Hj, Wj) if k == "fault"} == dropped
    # splitmix64 reference values (fixed by the definition)
    # (seed 1 -> the mix of the golden gamma = the first output of splitmix64 seeded with 0)
    assert WL.drop_hash(1, 0, 0, 0) == 0xE220A8397B1DCDAF
