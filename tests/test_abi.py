"""CPU-side checks of the C-ABI library: it loads, exports every symbol include/dyo.h declares,
and its host-side arch parse (signatures, AFM segment table, sites, path bound) matches the
oracle. No compute calls (no GPU here)."""
import re
import os

import numpy as np
import pytest

import workloads as WL
from oracle import afm as A, encode as E, decode as D


@pytest.fixture(scope="module")
def dyo():
    import __graft_entry__
    __graft_entry__.build()
    from paper_conf_hpca_renxyzlnwxl24_b200 import dyo as m
    return m


def test_exports_match_header(dyo):
    hdr = open(os.path.join(os.path.dirname(__file__), "..", "include", "dyo.h")).read()
    declared = set(re.findall(r"\b(dyo_[a-z_]+)\s*\(", hdr)) - {"dyo_status"}
    L = dyo.lib()
    for name in declared:
        assert hasattr(L, name), name
    assert declared == set(dyo.EXPORTS)


@pytest.mark.parametrize("name", ["tiny", "moe", "af", "lstm"])
def test_arch_parse_matches_oracle(dyo, name):
    wl = WL.make(name)
    st, summ, seg, sig, err = dyo.arch_check(wl)
    assert st == 0, err
    assert summ["F"] == wl.pilot.F == E.feature_width(wl.S_max, wl.D_s, wl.h)
    assert [tuple(r) for r in seg.tolist()] == E.static_segment_table(wl)
    ops = [r for c, r in A.afm_rows(wl.program) if not c]
    assert [tuple(r) for r in sig.tolist()] == ops
    sites = A.sites(wl.program)
    assert summ["n_sites"] == len(sites)
    assert summ["n_branch_logits"] == WL.n_branch_logits(wl.program)
    assert summ["host_pool_bytes"] == max(t.host_off + (t.nbytes + 255) // 256 * 256 for t in wl.tensors)


def test_path_bound_is_the_longest_path(dyo):
    wl = WL.make("tiny")
    st, summ, *_ = dyo.arch_check(wl)
    assert summ["L_max"] == max(len(r) for _, r in D.enumerate_paths(wl.program))


def test_arch_validation_errors(dyo):
    wl = WL.make("tiny")
    wl.tensors[3].host_off += 8            # not ALIGN-aligned
    st, *_, err = dyo.arch_check(wl)
    assert st == -1 and "host_off" in err
    wl = WL.make("tiny")
    op = wl.program[0]
    wl.program[0] = WL.Op(op.idioms, op.inputs, ((5, 1), (2, 1)))   # descending tensor ids
    st, *_ = dyo.arch_check(wl)
    assert st == -1
    wl = WL.make("tiny")
    wl.program.append(WL.If([[WL.Loop([wl.program[0]], 1, 2)], []]))   # nested site
    st, *_ = dyo.arch_check(wl)
    assert st == -7
    st, summ, *_ = dyo.arch_check(WL.make("tiny"), branch_head=False)   # traversal decode: no branch head
    assert st == 0 and summ["n_branch_logits"] == 0


def test_strided_access_validation(dyo):
    """R13: strides only inside loops; named ids stay in [0, T) and ascending at every k."""
    from workloads import R, W
    T = 8
    ts = [WL.Tensor(256, 256 * i, False) for i in range(T)]

    def wl_of(prog):
        return WL.Workload("s", WL.LSTM, prog, ts, 1, 1, 0, 2, 1 << 30, 256, 1, None,
                           np.zeros((1, 1), np.int64), np.zeros(0, np.int32), 0)
    ok = [WL.Loop([WL.Op((0,) * 6, (), ((0, R), (1, W, 1)))], 1, 7)]     # ids 1..7 at k <= 6
    assert dyo.arch_check(wl_of(ok))[0] == 0
    too_far = [WL.Loop([WL.Op((0,) * 6, (), ((0, R), (1, W, 1)))], 1, 8)]
    assert dyo.arch_check(wl_of(too_far))[0] == -1
    crossing = [WL.Loop([WL.Op((0,) * 6, (), ((0, R, 2), (3, W)))], 1, 4)]   # 0,2,4 passes 3
    assert dyo.arch_check(wl_of(crossing))[0] == -1
    outside = [WL.Op((0,) * 6, (), ((0, R, 1),))]
    assert dyo.arch_check(wl_of(outside))[0] == -1
