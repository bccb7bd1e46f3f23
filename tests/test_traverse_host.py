"""Host-side traversal decode of libdyo (R4) against the oracle, on CPU.

dyo_traverse_check runs the same search dyo_pilot_predict runs when the arch has no branch
head; the oracle (oracle/decode.traversal) enumerates every path in lexicographic order. Both
must pick the same choices and agree on exact match vs the closest-count fallback.
"""
import numpy as np
import pytest
from hypothesis import given, settings, strategies as st

import workloads as WL
from workloads import Op, If, Loop, R, W
from oracle import afm as A, decode as D, pilot as OP, encode as E


@pytest.fixture(scope="module")
def dyo():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_hpca_renxyzlnwxl24_b200 import dyo as m
    return m


def _wl(program, K_max, tensors=4):
    ts = [WL.Tensor(1 << 20, i << 20, False) for i in range(tensors)]
    return WL.Workload("t", WL.LSTM, program, ts, 2, 1, 0, K_max, 1 << 30, 256, 1, None,
                       np.zeros((1, 1), np.int64), np.zeros(0, np.int32), 0)


def _slots(blocks, K_max):
    s = np.zeros((K_max, 10), np.int32)
    for k, v in enumerate(blocks[:K_max]):
        s[k] = v
    return s


@st.composite
def flat_program(draw):
    """Top-level sites with flat arms / bodies (the shape the library decodes), ties included:
    a later If may replay an earlier free If of the same arity (reading R6)."""
    def op():
        return Op(tuple(draw(st.lists(st.integers(0, 2), min_size=6, max_size=6))),
                  (tuple(draw(st.lists(st.integers(1, 5), min_size=1, max_size=3))),),
                  ((draw(st.integers(0, 3)), R),))
    items, free_ifs, n_sites = [], [], 0
    for _ in range(draw(st.integers(1, 5))):
        kind = draw(st.integers(0, 3))
        if kind == 0:
            items.append(op())
        elif kind == 1 or (kind == 3 and not free_ifs):
            nb = draw(st.integers(2, 3))
            items.append(If([[op() for _ in range(draw(st.integers(0, 3)))] for _ in range(nb)]))
            free_ifs.append((n_sites, nb))
            n_sites += 1
        elif kind == 2:
            lo = draw(st.integers(0, 2))
            items.append(Loop([op() for _ in range(draw(st.integers(1, 2)))], lo, lo + draw(st.integers(0, 3))))
            n_sites += 1
        else:
            tgt, nb = free_ifs[draw(st.integers(0, len(free_ifs) - 1))]
            items.append(If([[op() for _ in range(draw(st.integers(0, 2)))] for _ in range(nb)], tie=tgt))
            n_sites += 1
    return items


@settings(max_examples=200, deadline=None)
@given(flat_program(), st.data())
def test_traversal_matches_oracle_on_cut_paths(dyo, prog, data):
    """Blocks cut from a real path: both find an exact match, and the same (first) one."""
    paths = list(D.enumerate_paths(prog))
    ch, rows = paths[data.draw(st.integers(0, len(paths) - 1))]
    L = len(rows)
    if L == 0:
        return
    cuts = sorted(set(data.draw(st.lists(st.integers(1, max(1, L - 1)), max_size=5))) | {L})
    counts, prev = [], 0
    for c in cuts:
        counts.append(c - prev)
        prev = c
    blocks = [A.block10(rows[s:e]) for s, e in D.cut(L, counts)]
    K_max = 8
    if len(blocks) > K_max:
        return
    ch_o, _, ok_o = D.traversal(prog, blocks)
    st_, ch_l, ok_l, err = dyo.traverse_check(_wl(prog, K_max), _slots(blocks, K_max))
    assert st_ == 0, err
    assert ok_o and ok_l == 1
    assert ch_l == ch_o


@settings(max_examples=200, deadline=None)
@given(flat_program(), st.data())
def test_traversal_matches_oracle_on_arbitrary_blocks(dyo, prog, data):
    """Arbitrary (mostly unmatched) block vectors: same exact-match / fallback decision and the
    same choices (the fallback picks the first path closest in operator count)."""
    K_max = 4
    nk = data.draw(st.integers(0, K_max))
    blocks = []
    for _ in range(nk):
        n0 = data.draw(st.integers(1, 8))
        blocks.append((n0,) + tuple(data.draw(st.lists(st.integers(0, 12), min_size=9, max_size=9))))
    ch_o, _, ok_o = D.traversal(prog, blocks)
    st_, ch_l, ok_l, err = dyo.traverse_check(_wl(prog, K_max), _slots(blocks, K_max))
    assert st_ == 0, err
    assert bool(ok_l) == ok_o
    assert ch_l == ch_o


def test_traversal_tiny_pilot_logits(dyo):
    """The tiny config without a branch head: block head decoded from the oracle's fp64 logits
    (R4), then the library's traversal and the oracle's decode pick the same path."""
    wl = WL.make("tiny", branch_head=False)
    for s in range(4):
        x = E.encode(wl, wl.samples[s])
        y = OP.forward(wl.pilot, x, wl.nn_type)
        pred = D.decode(wl, y, branch_head=False)
        slots = np.array(pred.slots, np.int32)
        st_, ch_l, ok_l, err = dyo.traverse_check(wl, slots)
        assert st_ == 0, err
        assert ch_l == pred.choices and bool(ok_l) == pred.matched


def test_traversal_rejects_nested_sites(dyo):
    prog = [If([[Loop([Op((1,) * 6, ((2,),), ())], 1, 2)], []])]
    st_, *_ = dyo.traverse_check(_wl(prog, 2), np.zeros((2, 10), np.int32))
    assert st_ == -7
