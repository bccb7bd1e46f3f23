"""Pins for oracle/afm.py: Fig. 3 signature, Fig. 4 AFM, block vector, resolved path."""
import pytest

from oracle import afm as A
from workloads import Op, If, Loop
from helpers import load, build_program


def test_fig3_signature():
    g = load("fig3_matmul.json")
    for c in g["cases"]:
        op = Op(tuple(c["idioms"]), tuple(tuple(s) for s in c["inputs"]), ())
        assert A.signature(op) == tuple(c["signature"])


def test_tree_cnn_afm_and_segments():
    g = load("tree_cnn_node.json")
    prog = build_program(g["program"], g["ops"])
    assert A.afm(prog) == [tuple(r) for r in g["afm"]]
    rows = A.afm_rows(prog)
    assert [c for c, _ in rows] == [False] * 4 + [True, False]   # control row at its position
    segs = A.segments(rows)
    assert [A.block10_of_sig_rows(s) for s in segs] == [tuple(v) for v in g["segments_block10"]]


def test_resolved_paths_and_blocks():
    g = load("tree_cnn_node.json")
    ops = g["ops"]
    prog = build_program(g["program"], ops)
    name = lambda rows: ["Z" if r is None else r.name for r in rows]
    assert name(A.resolve(prog, [1])) == g["path_branch1"]
    assert name(A.resolve(prog, [0])) == g["path_branch0"]
    path = A.resolve(prog, [1])
    tb = g["three_blocks"]
    cuts, c = [], 0
    for n in tb["counts"]:
        cuts.append(path[c:c + n])
        c += n
    assert [A.block10(b) for b in cuts] == [tuple(v) for v in tb["block10"]]
    le = g["loop_example"]
    lp = build_program(le["program"], ops)
    assert name(A.resolve(lp, [le["trip_index"]])) == le["path"]


def test_block_vector_storage_is_tens_of_bytes():
    # T8 / P:L149: one block vector = 10 x int32 = 40 bytes
    import numpy as np
    assert np.zeros(10, np.int32).nbytes == 40


def test_all_zero_signature_op_is_not_a_control_row():
    prog = [Op((0,) * 6, (), ()), If([[Op((0,) * 6, (), ())]])]
    rows = A.afm_rows(prog)
    assert [c for c, _ in rows] == [False, True, False]
    assert len(A.segments(rows)) == 2


def test_saturation():
    op = Op((1 << 30, 0, 0, 0, 0, 0), ((1 << 25,), (5,)), ())
    s = A.signature(op)
    assert s[0] == A.SAT and s[6] == A.SAT
    assert A.block10([op] * 3)[1] == A.SAT


def test_loop_rows_count():
    body = [Op((0, 0, 0, 0, 1, 0), ((2,),), ())] * 4
    prog = [Loop(body, 1, 3)]
    for idx, n in enumerate((1, 2, 3)):
        rows = A.resolve(prog, [idx])
        assert len(rows) == 4 * n + n + 1
        assert sum(r is None for r in rows) == n + 1


def test_strided_accesses_forward_reverse_and_per_sample():
    """Reading R13, written out by hand: an access (t, m, stride_k, stride_b) names tensor
    t + stride_k * k + stride_b * b; a reversed loop counts k down from n - 1."""
    from workloads import R, W
    from oracle import decode as D
    fwd = Op((0, 0, 0, 1, 1, 0), ((2,),), ((0, R), (10, R, 1, 100), (20, W, 1)), "f")
    bwd = Op((0, 0, 0, 1, 1, 0), ((2,),), ((0, R), (20, R, 1)), "g")
    prog = [Loop([fwd], 1, 4), Loop([bwd], 1, 4, tie=0, rev=True)]
    rows = A.resolve(prog, [2], b=1)                     # trip 3, sample 1 of the batch
    accs = [r.acc for r in rows if r is not None]
    assert accs == [((0, R), (20, W), (110, R)),          # k = 0: x[1,0] = 10 + 100
                    ((0, R), (21, W), (111, R)),
                    ((0, R), (22, W), (112, R)),
                    ((0, R), (22, R)),                    # reversed: k = 2, 1, 0
                    ((0, R), (21, R)),
                    ((0, R), (20, R))]
    assert [r is None for r in rows] == [True, False] * 3 + [True] + [True, False] * 3 + [True]
    # the same binding through path enumeration, and W_j in first-access order (R8)
    for ch, rr in D.enumerate_paths(prog, b=1):
        if ch == [2, 2]:
            assert rr == rows
    Ws = D.tensor_sets(rows, [(0, 4), (4, len(rows))])
    assert Ws[0] == [(0, R, True), (20, W, False), (110, R, True), (21, W, False), (111, R, True)]
    assert [t for t, _, _ in Ws[1]] == [0, 22, 112, 21, 20]      # ascending within an operator


def test_strided_access_outside_loop_is_rejected():
    from workloads import R
    with pytest.raises(ValueError):
        A.resolve([Op((0,) * 6, (), ((3, R, 1),))], [])
