"""Pins for oracle/migrate.py: bytes follow versions through evict/move/carry/fetch."""
import numpy as np
import pytest

from oracle import migrate as M, plan as PL, run as OR, encode as E, pilot as P, decode as D
import workloads as WL


def _new_step(wl, st_):
    for t, ten in enumerate(wl.tensors):      # as plan.plan(): R9 at the step boundary
        if ten.transient:
            st_.dirty[t] = False


def _tiny_kib(seed=0):
    wl = WL.make("tiny", seed=seed)
    # scale sizes MiB -> KiB (input construction) so the byte model fits in memory quickly
    off = 0
    for t in wl.tensors:
        t.nbytes //= 1024
        t.host_off = off
        off += PL.aligned(t.nbytes, wl.align)
    wl.budget //= 1024
    return wl


@pytest.mark.parametrize("seed", [0, 1, 2])
@pytest.mark.parametrize("policy", [0, 1])
def test_bytesim_reads_latest_versions(seed, policy):
    wl = _tiny_kib(seed)
    bs = M.ByteSim(wl)
    st_ = PL.initial_state(len(wl.tensors))
    table = ()
    for s in range(4):
        x = E.encode(wl, wl.samples[s], wl.hist_ids, table)
        pred = D.decode(wl, P.forward(wl.pilot, x, wl.nn_type))
        _new_step(wl, st_)
        for j in range(len(pred.W)):
            tr = PL.transition(st_, wl, pred.W, j, policy)
            bs.apply(tr)
            assert bs.run_block(pred.W[j], tr.half, st_) == []
        st_.G += len(pred.W)
        table = pred.blocks
        bs.new_step()
    # I5: host homes of non-resident, non-transient tensors hold the latest version
    for t, ten in enumerate(wl.tensors):
        if st_.loc[t] == PL.HOST and not ten.transient:
            assert np.array_equal(bs.host[ten.host_off: ten.host_off + ten.nbytes],
                                  M.content_bytes(t, bs.ver[t], ten.nbytes))


def test_dropping_a_writeback_is_detected():
    """Mutation check: the byte model catches a plan that forgets a dirty writeback.
    Hand trace: t0 (non-transient) written by block 0, evicted dirty at transition 2, read by
    block 3 (same trace as test_oracle_plan.test_writeback_of_dirty_live_tensor)."""
    from workloads import Workload, PilotSpec, Tensor, R, W
    wl = Workload("hand", 0, [], [Tensor(512, 0, False), Tensor(512, 512, True), Tensor(512, 1024, False)],
                  1, 1, 0, 8, 2048, 256, 0, PilotSpec(16, 8, [], [], 0, {}), np.zeros((1, 1), np.int64),
                  np.zeros(0, np.int32), 0)
    Ws = [[(0, W, False), (1, W, False)], [(1, R, True)], [(2, R, True), (1, W, False)], [(0, R, True)]]
    for mutate in (False, True):
        bs = M.ByteSim(wl)
        st_ = PL.initial_state(3)
        bad = []
        for j in range(4):
            tr = PL.transition(st_, wl, Ws, j, 0)
            if mutate:
                tr.evict = [(t, a, b, n, False) for t, a, b, n, wb in tr.evict]
            bs.apply(tr)
            bad += bs.run_block(Ws[j], tr.half, st_)
        assert bad == ([0] if mutate else [])


def test_content_generator_numpy_torch_agree():
    import torch
    a = WL.content_words_np(17, 3, 4096, start=100)
    b = WL.content_words_torch(17, 3, 4096, "cpu", start=100).numpy().view(np.uint32)
    assert np.array_equal(a, b)
