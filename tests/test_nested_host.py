"""libdyo's host nested-site decode (reading R16; nested.cpp via dyo_nested_check, no GPU)
against the oracle, plus the load-time checks of nested programs (dyo_arch_check)."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import workloads as WL
from workloads import Op, If, Loop, R
from oracle import afm as A, decode as D
from helpers import load, build_program
from test_oracle_nested import nested_programs


@pytest.fixture(scope="module")
def dyo():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_hpca_renxyzlnwxl24_b200 import dyo as mod
    return mod


def _wl(prog, K_max=4):
    return WL.Workload("t", WL.CNN, prog, [WL.Tensor(256, 256 * i, False) for i in range(64)], 2, 0, 0, K_max,
                       1 << 30, 256, 1, None, np.zeros((1, 0), np.int64), np.zeros(0, np.int32), 0)


def _slots(blocks, K_max):
    s = np.zeros((K_max, 10), np.int32)
    for i, v in enumerate(blocks):
        s[i] = v
    return s


def _path_ops(prog, rows):
    """Operator indices (preorder numbering) of a row list; bind() may copy strided operators,
    so rows are matched by their (unique) names."""
    by_name = {o.name: i for i, o in enumerate(_all_ops(prog))}
    return [-1 if r is None else by_name[r.name] for r in rows]


def _all_ops(prog):
    out = []

    def rec(items):
        for it in items:
            if isinstance(it, Op):
                out.append(it)
            elif isinstance(it, If):
                for br in it.branches:
                    rec(br)
            else:
                rec(it.body)
    rec(prog)
    return out


def test_golden_tree_cnn_exact_and_fallback(dyo):
    g = load("tree_cnn_loop.json")
    prog = build_program(g["program"], g["ops"])
    wl = _wl(prog)
    for case in ("three_blocks", "one_block", "fallback"):
        blocks = [tuple(v) for v in g[case]["block10"]]
        top = g["resolved"]["top_choices"] if case == "three_blocks" else g[case]["top_choices"]
        want_nest, want_rows, want_ok = D.nested_traversal(prog, top, blocks)
        st_, nest, path, m, err = dyo.nested_check(wl, _slots(blocks, 4), top)
        assert st_ == 0, err
        assert nest == want_nest and m == int(want_ok) and path == _path_ops(prog, want_rows), case


@settings(max_examples=80, deadline=None)
@given(nested_programs(), st.data())
def test_random_nested_programs_match_oracle(dyo, prog, data):
    for i, o in enumerate(_all_ops(prog)):
        o.name = f"o{i}"
    wl = _wl(prog)
    tops = list(D.top_choice_vectors(prog))
    ch = data.draw(st.sampled_from(tops))
    res = list(D._all_resolutions(D._atoms(prog, ch, 0)))
    nest, rows = data.draw(st.sampled_from(res))
    L = len(rows)
    k = data.draw(st.integers(1, min(4, L)))
    cuts = sorted(data.draw(st.sets(st.integers(1, L - 1), min_size=k - 1, max_size=k - 1))) if L > 1 else []
    bounds = [0] + cuts + [L]
    blocks = [A.block10(rows[bounds[i]:bounds[i + 1]]) for i in range(len(bounds) - 1)]
    if data.draw(st.booleans()):                       # perturb: exercise the fallback
        blocks = [tuple(v[:1]) + tuple(x + 1 for x in v[1:]) for v in blocks]
    want_nest, want_rows, want_ok = D.nested_traversal(prog, ch, blocks)
    st_, got_nest, path, m, err = dyo.nested_check(wl, _slots(blocks, 4), ch)
    assert st_ == 0, err
    assert got_nest == want_nest and m == int(want_ok)
    assert path == _path_ops(prog, want_rows)


def test_tree_workload_arch_and_one_sample(dyo):
    wl = WL.make("tree", n_samples=4, batch=4)
    st_, summ, _, _, err = dyo.arch_check(wl)
    assert st_ == 0, err
    # L_max: embed + 127 nodes x (loop test + If row + the internal arm's 2 ops) + exit + loss
    #        + 127 backward iterations x 2 + exit + optimizer
    assert summ["L_max"] == 1 + 127 * 4 + 1 + 1 + 127 * 2 + 1 + 1
    assert summ["n_branch_logits"] == 113 and summ["n_sites"] == 3
    from oracle import encode as E, pilot as P
    for s in range(2):
        x = E.encode(wl, wl.samples[s], wl.hist_ids, ())
        y = P.forward(wl.pilot, x, wl.nn_type)
        pred = D.decode(wl, y, b=s)
        assert pred.matched
        st_, nest, path, m, err = dyo.nested_check(wl, np.array(pred.slots, np.int32), pred.choices)
        assert st_ == 0 and m == 1 and nest == pred.nested and len(path) == len(pred.path), err


@pytest.mark.parametrize("prog,status", [
    ([Loop([Loop([Op((0,) * 6, (), (), "a")], 1, 2)], 1, 2)], -7),              # nested loop
    ([Loop([If([[If([[], []])], []])], 1, 2)], -7),                              # If inside a nested arm
    ([If([[], []]), Loop([If([[], []], tie=0)], 1, 2)], -1),                    # nested site replays
])
def test_nested_shapes_rejected(dyo, prog, status):
    st_, _, _, _, err = dyo.arch_check(_wl(prog))
    assert st_ == status, err


def test_nested_needs_branch_head(dyo):
    wl = _wl([Loop([If([[], []])], 1, 2)])
    st_, _, _, _, err = dyo.arch_check(wl, branch_head=False)
    assert st_ == -7, err
