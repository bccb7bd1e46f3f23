"""Pins for oracle/decode.py: rounding, argmax ties, cut rule, traversal."""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

from oracle import afm as A, decode as D
from workloads import Op, If, Loop, R, W
from helpers import load, build_program


def test_block_head_rounding_half_even_and_clamp():
    y = np.zeros(20)
    y[0] = 2.5 / 16        # -> 2 (half to even)
    y[1] = 3.5 / 16        # -> 4
    y[2] = -1.0            # clamps to 0
    y[7] = 1.5 / 1024      # dim elements use 2^10 -> 2
    y[10] = 0.0            # slot 1 empty
    near = []
    slots = D.decode_block_head(y, 2, near)
    assert slots[0][:3] == (2, 4, 0) and slots[0][7] == 2
    assert slots[1][0] == 0
    assert len(near) == 3  # 2.5, 3.5 and 1.5 are exact ties -> logged


def test_branch_argmax_lowest_index_on_ties():
    prog = [If([[], [], []]), Loop([], 2, 4), If([[], []], tie=0)]
    y = np.zeros(10 * 1 + 3 + 3)
    y[10:13] = [1.0, 3.0, 3.0]
    y[13:16] = [0.5, 0.1, 0.7]
    near = []
    ch = D.decode_branch_head(y, prog, 1, near)
    assert ch == [1, 2, 1]          # tie at 3.0 -> index 1; loop -> index 2 (trip 4); tied site copies site 0
    assert ("site", 0) in near


@pytest.mark.parametrize("L,counts,want", [
    (6, [2, 2, 2], [(0, 2), (2, 4), (4, 6)]),
    (5, [2, 2, 2], [(0, 2), (2, 4), (4, 5)]),        # truncated at the end
    (3, [2, 2, 2], [(0, 2), (2, 3)]),                # groups past the end dropped
    (9, [2, 2, 2], [(0, 2), (2, 4), (4, 9)]),        # last group absorbs the remainder
    (4, [], [(0, 4)]),                               # no non-empty slot -> one group
    (0, [3], []),
])
def test_cut(L, counts, want):
    assert D.cut(L, counts) == want


def _golden_prog():
    g = load("tree_cnn_node.json")
    return g, build_program(g["program"], g["ops"])


def test_traversal_exact_match_fig5():
    g, prog = _golden_prog()
    blocks = [tuple(v) for v in g["three_blocks"]["block10"]]
    choices, rows, ok = D.traversal(prog, blocks)
    assert ok and choices == [1] and len(rows) == 6


def test_traversal_other_branch_and_fallback():
    g, prog = _golden_prog()
    b = [tuple(v) for v in g["three_blocks"]["block10"]]
    ch, rows, ok = D.traversal(prog, [b[0], b[1], (1,) + (0,) * 9])
    assert ok and ch == [0]
    # counts sum to 7: no path matches; closest in operator count is the 6-row path
    ch, rows, ok = D.traversal(prog, [b[0], b[1], (3,) + (0,) * 9])
    assert not ok and ch == [1]


def test_enumeration_order_and_count():
    wl = __import__("workloads").make("tiny")
    paths = list(D.enumerate_paths(wl.program))
    assert len(paths) == 12
    assert [p[0] for p in paths][:4] == [[0, 0, 0], [0, 0, 1], [0, 0, 2], [0, 1, 0]]
    lens = [len(r) for _, r in paths]
    assert min(lens) >= 30 and max(lens) <= 50
    for ch, rows in paths:
        assert rows == A.resolve(wl.program, ch)


def test_tensor_sets_order_modes():
    o1 = Op((0,) * 6, (), ((3, W), (5, R)))
    o2 = Op((0,) * 6, (), ((1, R), (3, R), (5, W)))
    Ws = D.tensor_sets([o1, None, o2], [(0, 3)])
    assert Ws == [[(3, W | R, False), (5, R | W, True), (1, R, True)]]


# --- round trip (T5, "12,000 cases ... all find an exact match") -------------------

@st.composite
def small_program(draw):
    def op():
        return Op(tuple(draw(st.lists(st.integers(0, 3), min_size=6, max_size=6))),
                  (tuple(draw(st.lists(st.integers(1, 9), min_size=1, max_size=3))),), ())
    items = []
    for _ in range(draw(st.integers(1, 4))):
        kind = draw(st.integers(0, 2))
        if kind == 0:
            items.append(op())
        elif kind == 1:
            items.append(If([[op() for _ in range(draw(st.integers(0, 3)))] for _ in range(draw(st.integers(2, 3)))]))
        else:
            lo = draw(st.integers(0, 2))
            items.append(Loop([op() for _ in range(draw(st.integers(1, 2)))], lo, lo + draw(st.integers(0, 2))))
    return items


@settings(max_examples=150, deadline=None)
@given(small_program(), st.data())
def test_traversal_round_trip(prog, data):
    paths = list(D.enumerate_paths(prog))
    ch, rows = paths[data.draw(st.integers(0, len(paths) - 1))]
    L = len(rows)
    if L == 0:
        return
    cuts = sorted(set(data.draw(st.lists(st.integers(1, max(1, L - 1)), max_size=4))) | {L})
    counts, prev = [], 0
    for c in cuts:
        counts.append(c - prev)
        prev = c
    blocks = [A.block10(rows[s:e]) for s, e in D.cut(L, counts)]
    ch2, rows2, ok = D.traversal(prog, blocks)
    assert ok
    # same block vectors; same path unless another path has identical vectors (documented ambiguity)
    assert [A.block10(rows2[s:e]) for s, e in D.cut(len(rows2), counts)] == blocks
    first = next(c for c, r in paths if len(r) == L and
                 [A.block10(r[s:e]) for s, e in D.cut(L, counts)] == blocks)
    assert ch2 == first
