"""Pins for oracle/partition.py (reading R18: Sentinel-style overlap partition, P:L164-L170,
L203-L205; the L275 heuristics)."""
import itertools

from hypothesis import given, settings, strategies as st

import workloads as WL
from workloads import Op, R, W, RW
from oracle import partition as PT, afm as A


def _trace(rows_spec, sizes):
    """rows_spec: list of (inputs elements, accesses) or None (control row)."""
    rows = []
    for i, r in enumerate(rows_spec):
        if r is None:
            rows.append(None)
        else:
            n, acc = r
            rows.append(Op((0, 0, 0, 0, 1, 0), ((n,),), tuple(sorted(acc)), f"r{i}"))
    tensors = [WL.Tensor(b, 0, False) for b in sizes]
    times = [WL.op_time_ns(r) for r in rows]
    return rows, times, tensors


def test_hand_example():
    # four rows; tensors: 0 (1000 B, read), 1 (5000 B, read), 2 (64 B, written)
    rows, times, tens = _trace([(640, [(0, R)]), (64, [(2, W)]), (64, [(1, R)]), (6400, [(1, R), (2, R)])],
                               [1000, 5000, 64])
    assert times == [11, 2, 2, 101]
    need, fetch, comp = PT.block_tables(rows, times, tens, 64)
    # block [2, 4) reads 1 and 2 first: fetch 5064 B; [1, 2) writes 2 first: fetch 0
    assert fetch[2][4] == 5064 and fetch[1][2] == 0 and need[1][4] == 5056 + 64     # aligned to 64 B
    assert comp[0][2] == 13
    bw = 1000                                 # bytes per microsecond = 1 GB/s: 1 ns per byte
    # cuts [0,1,2,4]: block 1 ([1,2)) fetches 0; block 2 ([2,4)) fetches 5064 -> 5064 ns - comp(1,2)=2
    assert PT.exposed([0, 1, 2, 4], fetch, comp, bw) == 5062
    # cuts [0,1,3,4]: block 1 [1,3) reads 1 first (5000 ns) - comp(0,1) = 11; block 2 [3,4) reads
    # 1 and 2 first (5064 ns) - comp(1,3) = 4
    assert PT.exposed([0, 1, 3, 4], fetch, comp, bw) == 4989 + 5060
    # cuts [0,2,3,4]: 5000 - 13 and 5064 - 2
    assert PT.exposed([0, 2, 3, 4], fetch, comp, bw) == 4987 + 5062
    cuts, ex = PT.overlap_partition(4, 3, need, fetch, comp, 1 << 30, bw)
    assert cuts == [0, 1, 2, 4] and ex == 5062


def test_infinite_bandwidth_gives_the_first_feasible_cuts():
    rows, times, tens = _trace([(64, [(0, R)])] * 6, [100])
    need, fetch, comp = PT.block_tables(rows, times, tens, 64)
    cuts, ex = PT.overlap_partition(6, 3, need, fetch, comp, 1 << 30, 10 ** 18)
    assert ex == 0 and cuts == [0, 1, 2, 6]


def test_capacity_is_respected_or_infeasible():
    rows, times, tens = _trace([(64, [(0, R)]), (64, [(1, R)]), (64, [(2, R)])], [1000, 1000, 1000])
    need, fetch, comp = PT.block_tables(rows, times, tens, 256)
    cuts, ex = PT.overlap_partition(3, 2, need, fetch, comp, 1024, 1000)
    assert cuts is None                       # two blocks cannot hold three 1 KiB tensors in 1 KiB each
    cuts, ex = PT.overlap_partition(3, 3, need, fetch, comp, 1024, 1000)
    assert cuts == [0, 1, 2, 3]


@st.composite
def traces(draw):
    L = draw(st.integers(3, 8))
    T = draw(st.integers(1, 5))
    spec = []
    for _ in range(L):
        if draw(st.booleans()) and spec:
            spec.append(None)
        else:
            ts = draw(st.sets(st.integers(0, T - 1), min_size=1, max_size=min(3, T)))
            spec.append((draw(st.integers(1, 4000)), [(t, draw(st.sampled_from([R, W, RW]))) for t in ts]))
    sizes = [draw(st.integers(1, 5000)) for _ in range(T)]
    return spec, sizes


@settings(max_examples=120, deadline=None)
@given(traces(), st.data())
def test_overlap_partition_equals_brute_force(tr, data):
    rows, times, tens = _trace(*tr)
    L = len(rows)
    K = data.draw(st.integers(1, L))
    H = data.draw(st.integers(256, 20000))
    bw = data.draw(st.integers(1, 100000))
    need, fetch, comp = PT.block_tables(rows, times, tens, 256)
    best = None
    for inner in itertools.combinations(range(1, L), K - 1):
        c = [0, *inner, L]
        if not PT.feasible(c, need, H):
            continue
        cand = (PT.exposed(c, fetch, comp, bw), c)
        if best is None or cand < best:
            best = cand
    cuts, ex = PT.overlap_partition(L, K, need, fetch, comp, H, bw)
    if best is None:
        assert cuts is None
    else:
        assert (ex, cuts) == best


def test_even_partitions():
    assert PT.even_partition([1, 1, 1, 1, 1, 1], 3) == [0, 2, 4, 6]
    assert PT.even_partition([1, 0, 1, 0, 1, 0], 3) == [0, 2, 4, 6]
    assert PT.even_partition([10, 1, 1, 1, 1, 1, 1], 2) == [0, 1, 7]       # no prefix within 8: clamp to 1
    assert PT.even_partition([0, 0, 0, 9], 3) == [0, 2, 3, 4]             # p = 3 for both cuts, clamped


def test_labels_are_the_blocks_vectors():
    rows, times, tens = _trace([(64, [(0, R)]), None, (128, [(1, W)])], [100, 100])
    lab = PT.labels(rows, [0, 1, 3], 4)
    assert lab[0] == A.block10(rows[0:1]) and lab[1] == A.block10(rows[1:3]) and lab[2] == (0,) * 10
