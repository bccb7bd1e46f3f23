"""Pins for oracle/plan.py: hand-derived plans, brute-force optimality, invariants I1-I7."""
import copy
import random

import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import plan as PL, brute as BR, invariants as INV, run as OR
from workloads import Workload, PilotSpec, Tensor, R, W, RW
import workloads as WL
from helpers import load


def _wl(tensors, budget, policy=1):
    return Workload("hand", 0, [], [Tensor(b, h, tr) for b, h, tr in tensors], 1, 1, 0, 8, budget, 256,
                    policy, PilotSpec(16, 8, [], [], 0, {}), np.zeros((1, 1), np.int64), np.zeros(0, np.int32), 0)


@pytest.mark.parametrize("case", load("plan_hand.json")["cases"], ids=lambda c: c["name"])
def test_hand_plans(case):
    g = load("plan_hand.json")
    wl = _wl(g["tensors"], case["budget"], case["policy"])
    Ws = [[(t, m, f) for t, m, f in Wj] for Wj in g["W"]]
    trs, st_ = PL.plan(PL.initial_state(4), wl, Ws)
    for tr, want in zip(trs, case["transitions"]):
        assert tr.half == want["half"]
        for k in ("evict", "move", "carry", "alloc", "fetch"):
            assert [list(r) for r in getattr(tr, k)] == want[k], (tr.j, k)
    assert sum(t.h2d for t in trs) == case["h2d"]
    assert sum(t.d2h for t in trs) == case["d2h"]
    assert sum(t.d2d for t in trs) == case["d2d"]


def test_budget_error_is_transactional():
    wl = _wl([[1024, 0, False]], 1024)
    st0 = PL.initial_state(1)
    with pytest.raises(PL.BudgetError):
        PL.plan(st0, wl, [[(0, R, True)]])
    assert st0.loc == [PL.HOST]


def test_writeback_of_dirty_live_tensor():
    # t0 written in block 0, unused in block 1..2, read in block 3: with no room it is evicted
    # with writeback; t1 (transient) dies -> freed without writeback
    wl = _wl([[512, 0, False], [512, 512, True], [512, 1024, False]], 2048)
    Ws = [[(0, W, False), (1, W, False)], [(1, R, True)], [(2, R, True), (1, W, False)], [(0, R, True)]]
    trs, _ = PL.plan(PL.initial_state(3), wl, Ws, policy=0)
    ev = trs[2].evict
    assert [(r[0], r[4]) for r in ev] == [(0, True)]
    assert trs[2].d2h == 512


def test_prefix_cut_is_a_prefix():
    cands = [(3, 256, 7), (1, 512, 2), (1, 256, 9), (2, 256, 1)]
    assert PL.prefix_cut(cands, 768) == [9, 2]       # (1,256,9), (1,512,2) then (2,...) does not fit
    assert PL.prefix_cut(cands, 700) == [9]          # no skip-and-continue past (1,512,2)


def _random_trace(rng, T=7, K=5, budget=4096):
    sizes = [int(rng.integers(1, 4)) * 256 for _ in range(T)]
    offs = np.cumsum([0] + sizes[:-1]).tolist()
    tens = [(sizes[i], offs[i], bool(rng.random() < 0.3)) for i in range(T)]
    Ws = []
    for _ in range(K):
        ids = sorted(rng.choice(T, size=int(rng.integers(1, 3)), replace=False).tolist())
        Ws.append([(t, int(rng.choice([R, W, RW])), None) for t in ids])
    Ws = [[(t, m, bool(m & R)) for t, m, _ in Wj] for Wj in Ws]
    return tens, Ws, budget


@settings(max_examples=60, deadline=None)
@given(st.integers(0, 10 ** 6))
def test_bruteforce_two_half(seed):
    rng = np.random.default_rng(seed)
    tens, Ws, budget = _random_trace(rng, T=6, K=4, budget=int(rng.choice([2048, 3072, 4096])))
    wl = _wl(tens, budget)
    try:
        trs_r, _ = PL.plan(PL.initial_state(len(tens)), wl, Ws, policy=1)
        trs_p, _ = PL.plan(PL.initial_state(len(tens)), wl, Ws, policy=0)
    except PL.BudgetError:
        return
    opt, _ = BR.two_half_opt(PL.initial_state(len(tens)), wl, Ws)
    cost_r = sum(t.h2d + t.d2h for t in trs_r)
    assert opt <= cost_r
    assert sum(t.h2d for t in trs_r) <= sum(t.h2d for t in trs_p)          # I6


@settings(max_examples=80, deadline=None)
@given(st.integers(0, 10 ** 6))
def test_pool_mode_belady_is_optimal(seed):
    rng = random.Random(seed)
    T = rng.randint(3, 7)
    K = rng.randint(2, 7)
    C = rng.randint(2, 5)
    Ws = [set(rng.sample(range(T), rng.randint(1, 2))) for _ in range(K)]
    try:
        b = BR.pool_belady(C, Ws)
    except PL.BudgetError:
        return
    assert b == BR.pool_opt(C, Ws)


@pytest.mark.parametrize("name,steps", [("tiny", 6), ("moe", 3), ("af", 1)])
@pytest.mark.parametrize("policy", [0, 1])
def test_invariants_on_configs(name, steps, policy):
    wl = WL.make(name)
    st_ = PL.initial_state(len(wl.tensors))
    table = ()
    vs = None
    from oracle import encode as E, pilot as P, decode as D
    for s in range(steps):
        x = E.encode(wl, wl.samples[s], wl.hist_ids, table)
        pred = D.decode(wl, P.forward(wl.pilot, x, wl.nn_type))
        trs, st_, vs = INV.run_checked(st_, wl, pred.W, policy, vs)
        table = pred.blocks
        INV.host_current(st_, wl, vs)


def test_I7_cold_misses_only():
    wl = WL.make("tiny")
    wl.budget = 2 * sum(PL.aligned(t.nbytes, wl.align) for t in wl.tensors) + 4096
    res = OR.run(wl, 5)
    fetched = {}
    for r in res:
        for tr in r.transitions:
            for f in tr.fetch:
                if not wl.tensors[f[0]].transient:
                    fetched[f[0]] = fetched.get(f[0], 0) + 1
    assert fetched and max(fetched.values()) == 1


@settings(max_examples=40, deadline=None)
@given(st.integers(0, 10 ** 6))
def test_invariants_random(seed):
    rng = np.random.default_rng(seed)
    tens, Ws, budget = _random_trace(rng, T=9, K=7, budget=int(rng.choice([2048, 3072, 8192])))
    wl = _wl(tens, budget)
    st_ = PL.initial_state(len(tens))
    for policy in (0, 1):
        try:
            INV.run_checked(st_, wl, Ws, policy)
        except PL.BudgetError:
            pass
