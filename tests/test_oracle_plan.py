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
@pytest.mark.parametrize("policy", [0, 1, 2, 3])
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
    for policy in (0, 1, 2, 3):
        try:
            INV.run_checked(st_, wl, Ws, policy)
        except PL.BudgetError:
            pass


@pytest.mark.parametrize("K", [2, 3, 6, 7])
@pytest.mark.parametrize("policy", [0, 1])
def test_share_running_state_closed_form(K, policy):
    """R20 closed form: a running state t0 read and written by every block (the AlphaFold MSA/pair
    state) ping-pongs by K-1 late carries without SHARE; with SHARE it never moves except a final
    carry when it sits in the wrong half at the plan's last transition (K even), and every block
    still reads the latest version (run_checked: I1-I5 on versions)."""
    tens = [[512, 0, False]] + [[256, 512 + 256 * k, True] for k in range(K)]
    wl = _wl(tens, 4096, policy)
    Ws = [[(0, RW, True), (1 + k, W, False)] for k in range(K)]
    trs, _, _ = INV.run_checked(PL.initial_state(K + 1), wl, Ws, policy)
    carries = [(tr.j, r[0], r[4]) for tr in trs for r in tr.carry]
    assert carries == [(j, 0, True) for j in range(1, K)]
    trs, _, _ = INV.run_checked(PL.initial_state(K + 1), wl, Ws, policy | PL.SHARE)
    carries = [(tr.j, r[0], r[4]) for tr in trs for r in tr.carry]
    assert carries == ([(K - 1, 0, True)] if K % 2 == 0 else [])
    assert [tr.j for tr in trs if tr.share] == [j for j in range(1, K - 1) if j % 2 == 1]
    assert sum(tr.d2d for tr in trs) == (512 if K % 2 == 0 else 0)


def test_share_needs_the_next_group_and_frees_half_m():
    """R20 eligibility: only a tensor the next group also holds stays in the other half (a tensor
    used by j-1 and j only is carried as in R1), and a SHARE'd tensor takes no room in half m."""
    wl = _wl([[512, 0, False], [512, 512, False], [512, 1024, True]], 2048, 1)   # H = 1024
    Ws = [[(0, R, True), (1, R, True)], [(0, R, True), (1, R, True)], [(0, R, True), (2, W, False)]]
    trs, _, _ = INV.run_checked(PL.initial_state(3), wl, Ws, 1 | PL.SHARE)
    assert trs[1].share == [(0, 0)] and [r[0] for r in trs[1].carry] == [1]
    assert trs[1].need == 512
    # without SHARE block 1 needs both in half 1 (1024 = H): fits, both carried
    trs, _, _ = INV.run_checked(PL.initial_state(3), wl, Ws, 1)
    assert [r[0] for r in trs[1].carry] == [0, 1] and trs[1].need == 1024


def _share_late_checked(seed):
    """R20: a transition compacts a half holding tensors of the running block j-1 only as a late
    transition (after block j-1 ends); otherwise no MOVE touches W_{j-1} (I3, run_checked)."""
    rng = np.random.default_rng(seed)
    tens, Ws, budget = _random_trace(rng, T=9, K=8, budget=int(rng.choice([1536, 2048, 3072])))
    wl = _wl(tens, budget)
    try:
        trs, _, _ = INV.run_checked(PL.initial_state(len(tens)), wl, Ws, 1 | PL.SHARE)
    except PL.BudgetError:
        return []
    for j, tr in enumerate(trs):
        pinned = {t for t, _ in (trs[j - 1].share if j else [])}
        if tr.late_all:
            assert pinned
        if pinned & {r[0] for r in tr.move}:
            assert tr.late_all
    return trs


@pytest.mark.parametrize("seed", [204, 505, 710, 1227])     # seeds whose plans compact under SHARE'd tensors
def test_share_late_all_cases(seed):
    assert any(tr.late_all for tr in _share_late_checked(seed))


@settings(max_examples=60, deadline=None)
@given(st.integers(0, 10 ** 6))
def test_share_late_all_random(seed):
    _share_late_checked(seed)
