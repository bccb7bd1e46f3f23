"""GPU migration parity: bytes moved by dyo_migrate (DMA / pack / zero-copy / D2D kernels)
against the oracle's plan and version model, with emulated compute between transitions."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

import workloads as WL
from oracle import plan as PL, migrate as M
from gpu_harness import make_ctx, oracle_step, hist_for, tr_lists, gpu_lists, F_NO_ZEROCOPY, F_NO_PACK


@pytest.fixture(scope="module", autouse=True)
def _cuda():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    import __graft_entry__
    __graft_entry__.build()


class _Dev:
    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "|u1", "data": (ptr, False), "version": 3}


def _arena(d):
    base, H = d.arena()
    return torch.as_tensor(_Dev(base, 2 * H), device="cuda"), H


def _words(t, v, nb):
    return WL.content_words_torch(t, v, nb // 4, "cuda")


def _check_dev(arena, dst, t, v, nb):
    got = arena[dst: dst + nb].view(torch.int32)
    return bool(torch.equal(got, _words(t, v, nb)))


def _fill_pool_gpu(pool, wl):
    """Initial host homes from the shared counter-based generator, generated on the device (the
    torch twin of content_bytes, tested equal) and copied into the pinned pool: full-size pools
    (MoE 48 GiB) are too large to generate with numpy in a test."""
    for t, ten in enumerate(wl.tensors):
        torch.from_numpy(pool[ten.host_off: ten.host_off + ten.nbytes]).copy_(
            _words(t, 0, ten.nbytes).view(torch.uint8))


def _host_home_ok_gpu(pool, t, v, nb, off):
    return bool(torch.equal(torch.from_numpy(pool[off: off + nb]).cuda().view(torch.int32), _words(t, v, nb)))


def run_bytes(wl, steps, policy=None, flags=0, dma_min=0, staging=0, B=1, gpu_fill=False):
    for t in wl.tensors:
        assert t.nbytes % 4 == 0
    d = make_ctx(wl, flags=flags, policy=policy, dma_min_bytes=dma_min, staging_bytes=staging, max_batch=B)
    pool = d.host_pool_array()
    if gpu_fill:
        _fill_pool_gpu(pool, wl)
    else:
        for t, ten in enumerate(wl.tensors):
            pool[ten.host_off: ten.host_off + ten.nbytes] = M.content_bytes(t, 0, ten.nbytes)
    arena, H = _arena(d)
    stream = torch.cuda.current_stream()
    st = PL.initial_state(len(wl.tensors))
    table = ()
    ver = [0] * len(wl.tensors)
    mech = {"dma": 0, "zc": 0, "packed": 0}
    for s in range(steps):
        ids = [(s * B + i) % len(wl.samples) for i in range(B)]
        r = oracle_step(wl, ids, st, table, policy)
        assert r["err"] is None
        d.predict(wl.samples[ids].copy(), hist_for(wl, B), B, stream=stream.cuda_stream)
        K = d.plan(stream=stream.cuda_stream)
        assert K == len(r["trs"])
        fresh = set()
        Ws = [Wj for p in r["preds"] for Wj in p.W]
        for j, tr in enumerate(r["trs"]):
            assert gpu_lists(d, j) == tr_lists(tr)
            d.migrate(j, stream.cuda_stream)
            ent = d.plan_records(j, "entries")
            for (t, mode, rd, dst) in ent.tolist():
                nb = wl.tensors[t].nbytes
                if rd and (not wl.tensors[t].transient or t in fresh):
                    assert _check_dev(arena, dst, t, ver[t], nb), f"step {s} block {j}: tensor {t} stale"
            for (t, mode, rd, dst) in ent.tolist():
                if mode & 2:
                    ver[t] += 1
                    fresh.add(t)
                    nb = wl.tensors[t].nbytes
                    arena[dst: dst + nb].view(torch.int32).copy_(_words(t, ver[t], nb))
        st = r["state"]
        table = r["table"]
        torch.cuda.synchronize()
        c = d.counters(reset=True)
        mech["dma"] += c["h2d_dma"] + c["d2h_dma"]
        mech["zc"] += c["h2d_zc"] + c["d2h_zc"]
        mech["packed"] += c["d2h_packed"]
        # every resident non-transient tensor holds its latest bytes on the device (I2 + moves)
        for t, ten in enumerate(wl.tensors):
            if st.loc[t] != PL.HOST and not ten.transient:
                assert _check_dev(arena, st.loc[t] * H + st.off[t], t, ver[t], ten.nbytes), f"resident {t}"
    # I5: host homes of non-resident non-transient tensors hold their latest bytes
    n_home = 0
    for t, ten in enumerate(wl.tensors):
        if st.loc[t] == PL.HOST and not ten.transient:
            if gpu_fill:
                assert _host_home_ok_gpu(pool, t, ver[t], ten.nbytes, ten.host_off), f"host home of {t}"
            else:
                assert np.array_equal(pool[ten.host_off: ten.host_off + ten.nbytes],
                                      M.content_bytes(t, ver[t], ten.nbytes)), f"host home of {t}"
            n_home += 1
    mech["homes_checked"] = n_home
    mech["written_back_versions"] = sum(1 for t, ten in enumerate(wl.tensors) if not ten.transient and ver[t] > 0)
    d.close()
    return mech


@pytest.mark.parametrize("policy", [0, 1])
def test_tiny_fullsize_default_mechanisms(policy):
    wl = WL.make("tiny", n_samples=16)
    m = run_bytes(wl, 4, policy)
    assert m["dma"] > 0


def test_tiny_all_zero_copy():
    wl = WL.make("tiny", n_samples=16)
    m = run_bytes(wl, 3, 1, dma_min=1 << 40)
    assert m["dma"] == 0 and m["zc"] > 0


@pytest.mark.parametrize("flags", [0, F_NO_PACK, F_NO_ZEROCOPY])
def test_tiny_tight_budget_writebacks(flags):
    wl = WL.make("tiny", seed=2, n_samples=16)
    wl.budget = 384 << 20
    run_bytes(wl, 6, 0, flags=flags)


def test_moe_scaled_tied_routing_gradients():
    wl = WL.make_moe(seed=1, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    m = run_bytes(wl, 4, 1, dma_min=1 << 20)
    assert m["dma"] > 0


def test_af_scaled_recycling():
    wl = WL.make_af(seed=1, n_samples=8, act_mib=1, weight_mib=1, blocks=8, budget=64 << 20)
    for t in wl.tensors:
        t.nbytes = min(t.nbytes, 1 << 20)     # MSA/pair state scaled to 1 MiB too
    off = 0
    for t in wl.tensors:
        t.host_off = off
        off += (t.nbytes + 255) // 256 * 256
    run_bytes(wl, 3, 1)


def test_lstm_scaled_small_tensors_zero_copy():
    """Many 2-4 KiB per-timestep / per-sample tensors (R13): fetched and carried by the
    zero-copy and vector-copy kernels; a batch of 4 predictions per plan."""
    wl = WL.make_lstm(n_samples=16, batch=4, max_len=64, hidden=128, budget=4 << 20)
    m = run_bytes(wl, 2, 1, B=4)
    assert m["zc"] > 0


def run_pipelined(wl, steps, policy=None, dma_min=0, staging=0, lookahead=False, spin=0, flags=0):
    """The full event protocol, enqueued asynchronously: emulated compute block j runs on its own
    stream after ready[j]; transition j's EVICT waits end[j-2], its late carries end[j-1].
    Read mismatches are accumulated on the device; the host syncs once per step."""
    d = make_ctx(wl, policy=policy, dma_min_bytes=dma_min, staging_bytes=staging, flags=flags)
    pool = d.host_pool_array()
    for t, ten in enumerate(wl.tensors):
        pool[ten.host_off: ten.host_off + ten.nbytes] = M.content_bytes(t, 0, ten.nbytes)
    arena, H = _arena(d)
    s_copy, s_comp = torch.cuda.Stream(), torch.cuda.Stream()
    ready = [torch.cuda.Event() for _ in range(wl.K_max)]
    end = [torch.cuda.Event() for _ in range(wl.K_max)]
    t0 = torch.cuda.Event()
    for e in ready + end + [t0]:
        e.record(s_copy)
    torch.cuda.synchronize()
    bad = torch.zeros((), dtype=torch.int64, device="cuda")
    st = PL.initial_state(len(wl.tensors))
    table = ()
    ver = [0] * len(wl.tensors)
    cs = torch.cuda.current_stream().cuda_stream

    def plan_step(s, st_, table_):
        r = oracle_step(wl, [s % len(wl.samples)], st_, table_, policy)
        d.predict(wl.samples[[s % len(wl.samples)]].copy(), hist_for(wl, 1), 1, stream=cs)
        K = d.plan(stream=cs)
        assert K == len(r["trs"])
        ents = [d.plan_records(j, "entries").tolist() for j in range(K)]
        for j, tr in enumerate(r["trs"]):
            assert gpu_lists(d, j) == tr_lists(tr)
        return r, K, ents

    pending = plan_step(0, st, table)
    for s in range(steps):
        r, K, ents = pending
        if lookahead and s + 1 < steps:
            # plan the next step BEFORE this step's transitions are enqueued: two plans outstanding
            pending = plan_step(s + 1, r["state"], r["table"])
        t0.record(s_copy)
        fresh = set()
        for j in range(K):
            hf = end[j - 2] if j >= 2 else t0
            pd = end[j - 1] if j >= 1 else t0
            d.migrate(j, s_copy.cuda_stream, hf.cuda_event, pd.cuda_event, ready[j].cuda_event)
            s_comp.wait_event(ready[j])
            with torch.cuda.stream(s_comp):
                if spin:                       # a long block: transition j+1 overlaps it
                    torch.cuda._sleep(spin)
                for (t, mode, rd, dst) in ents[j]:
                    nb = wl.tensors[t].nbytes
                    if rd and (not wl.tensors[t].transient or t in fresh):
                        bad += (arena[dst: dst + nb].view(torch.int32) != _words(t, ver[t], nb)).sum()
                for (t, mode, rd, dst) in ents[j]:
                    if mode & 2:
                        ver[t] += 1
                        fresh.add(t)
                        nb = wl.tensors[t].nbytes
                        arena[dst: dst + nb].view(torch.int32).copy_(_words(t, ver[t], nb))
            end[j].record(s_comp)
        s_copy.wait_stream(s_comp)
        if not lookahead and s + 1 < steps:
            pending = plan_step(s + 1, r["state"], r["table"])
        torch.cuda.synchronize()
        assert int(bad.item()) == 0, f"step {s}: {int(bad.item())} stale words"
        st, table = r["state"], r["table"]
    for t, ten in enumerate(wl.tensors):
        if st.loc[t] == PL.HOST and not ten.transient:
            assert np.array_equal(pool[ten.host_off: ten.host_off + ten.nbytes],
                                  M.content_bytes(t, ver[t], ten.nbytes)), f"host home of {t}"
    d.close()


def test_pipelined_events_tiny_tight():
    wl = WL.make("tiny", seed=2, n_samples=16)
    wl.budget = 384 << 20
    run_pipelined(wl, 5, 0)


def test_pipelined_events_moe_scaled():
    wl = WL.make_moe(seed=2, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    run_pipelined(wl, 4, 1, dma_min=1 << 20)


def _tiny_with_moves():
    wl = WL.make("tiny", seed=2, n_samples=16)
    wl.budget = 448 << 20            # RETAIN at this budget compacts (first fit fails) ~100 times in 6 steps
    from oracle import run as OR
    assert sum(len(t.move) for r in OR.run(wl, 4, policy=1) for t in r.transitions) > 0
    return wl


def test_tiny_compaction_moves():
    run_bytes(_tiny_with_moves(), 4, 1)


def test_moe_scaled_packed_writebacks_small_staging():
    wl = WL.make_moe(seed=3, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    m = run_bytes(wl, 3, 1, dma_min=1 << 20, staging=4 << 20)
    assert m["dma"] > 0


def test_tiny_compaction_moves_small_staging_pipelined():
    run_pipelined(_tiny_with_moves(), 4, 1, staging=8 << 20)   # 4 MiB halves: tensors split into pieces


def test_pipelined_plan_lookahead_moe_scaled():
    """Two plans outstanding: step s+1 is predicted and planned before step s's transitions are
    enqueued; dyo_migrate must continue the older plan (FIFO) and the bytes stay exact."""
    wl = WL.make_moe(seed=4, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    run_pipelined(wl, 4, 1, dma_min=1 << 20, lookahead=True)


def test_pipelined_plan_lookahead_tiny_compaction():
    run_pipelined(_tiny_with_moves(), 4, 1, lookahead=True)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("nbytes,soff,doff", [(1 << 20, 0, 0), ((3 << 20) + 5, 16, 48), (777, 3, 5), (96 << 10, 0, 4096)])
def test_copy_kernels_exact(mode, nbytes, soff, doff):
    """Segment-copy kernels (SM vector path and TMA bulk path) move exactly the bytes, including
    unaligned heads/tails, and touch nothing outside the destination range."""
    wl = WL.make("tiny")
    d = make_ctx(wl, flags=4)
    src = torch.randint(0, 255, (nbytes + 8192,), dtype=torch.uint8, device="cuda")
    dst = torch.zeros(nbytes + 8192, dtype=torch.uint8, device="cuda")
    d.debug_copy(src.data_ptr() + soff, dst.data_ptr() + doff, nbytes, mode, torch.cuda.current_stream().cuda_stream)
    assert torch.equal(dst[doff: doff + nbytes], src[soff: soff + nbytes])
    assert int(dst[:doff].sum()) == 0 and int(dst[doff + nbytes:].sum()) == 0
    d.close()


_RING_CHILD = r"""
import sys, numpy as np, torch
sys.path.insert(0, sys.argv[1])
import workloads as WL
from gpu_harness import make_ctx
wl = WL.make("tiny")
d = make_ctx(wl, flags=4)
s = torch.cuda.current_stream().cuda_stream
n_launch = 0
for nbytes, soff, doff in [((3 << 20) + 5, 16, 48), (777, 3, 5), (40 << 20, 0, 4096)]:
    src = torch.randint(0, 255, (nbytes + 8192,), dtype=torch.uint8, device="cuda")
    dst = torch.zeros(nbytes + 8192, dtype=torch.uint8, device="cuda")
    d.debug_copy(src.data_ptr() + soff, dst.data_ptr() + doff, nbytes, 1, s)
    n_launch += 1
    assert torch.equal(dst[doff: doff + nbytes], src[soff: soff + nbytes])
    assert int(dst[:doff].sum()) == 0 and int(dst[doff + nbytes:].sum()) == 0
st = d.copy_stamps()
lid = (st[:, 0] >> np.uint64(32)).astype(np.int64)
assert sorted(set(lid.tolist())) == list(range(n_launch)), lid
t0, t1, t2 = (st[:, k].astype(np.int64) for k in (1, 2, 3))
assert np.all(t0 <= t1) and np.all(t1 <= t2)
d.copy_stamps(reset=True)
assert len(d.copy_stamps()) == 0
d.close()
print("ok")
"""


@pytest.mark.parametrize("ring,ctas", [("4x16", 1), ("8x16", 2), ("4x32", 1), ("6x32", 1), ("3x64", 3)])
def test_copy_ring_variants_exact_and_stamps(ring, ctas, tmp_path):
    """Every TMA ring shape (DYO_TMA_RING) and grid multiplier moves exactly the bytes, including
    unaligned heads/tails; the DYO_COPY_STAMPS log holds one ordered entry per CTA of each launch
    and empties on reset. Runs in a child process: the knobs are read at the first copy launch."""
    import os, subprocess, sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, DYO_TMA_RING=ring, DYO_TMA_CTAS_PER_SM=str(ctas), DYO_COPY_STAMPS="1",
               PYTHONPATH=os.pathsep.join([root, os.path.join(root, "tests")]))
    r = subprocess.run([sys.executable, "-c", _RING_CHILD, root], env=env, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0 and r.stdout.strip().endswith("ok"), r.stdout[-2000:] + r.stderr[-2000:]


def test_moe_fullsize_bytes():
    """configs[1] at full size (32 MiB expert tensors, 48 GiB pinned host pool, B = 3 GiB): every
    read of every block is compared word for word on the device with the version the oracle's
    plan implies (stronger than the per-tensor FNV digest of survey C6), and every host home of a
    non-resident tensor (the written-back gradients included) is compared at the end (I5)."""
    wl = WL.make("moe", n_samples=8)
    m = run_bytes(wl, 2, 1, gpu_fill=True)
    assert m["dma"] > 0 and m["written_back_versions"] > 0


def test_af_fullsize_bytes():
    """configs[2] at full size (16 MiB activations, 9.6 GiB host pool, B = 2 GiB), one step with
    its recycles: every read of every block and every host home checked as above."""
    wl = WL.make("af", n_samples=4)
    m = run_bytes(wl, 1, 1, gpu_fill=True)
    assert m["dma"] > 0


def test_tree_scaled_nested_bytes():
    """Tree-LSTM with nested per-node sites (R16): the host-resolved paths drive the plan; every
    read of every block and every host home checked (small hidden size, 4 predictions)."""
    wl = WL.make("tree", n_samples=16, batch=4, max_leaves=16, hidden=128, budget=8 << 20)
    m = run_bytes(wl, 2, 1, B=4)
    assert m["zc"] + m["dma"] > 0


def _sysfs_numa_node(dev):
    bus = torch.cuda.get_device_properties(dev)
    pci = "%04x:%02x:%02x.0" % (bus.pci_domain_id, bus.pci_bus_id, bus.pci_device_id)
    try:
        with open(f"/sys/bus/pci/devices/{pci}/numa_node") as f:
            return int(f.read().strip())
    except OSError:
        return -1


def test_host_pool_numa_local_and_exact(monkeypatch):
    """Survey §8(e) / P:L259: the pinned tensor homes sit on the GPU's NUMA node (mbind before
    cudaHostRegister) when the platform reports one; bytes through that pool stay exact; the
    DYO_HOST_NUMA=-1 override falls back to cudaHostAlloc."""
    wl = WL.make("tiny", n_samples=16)
    node = _sysfs_numa_node(0)
    d = make_ctx(wl)
    assert d.query("host_numa") == node
    d.close()
    m = run_bytes(wl, 2, 1)
    assert m["dma"] > 0
    monkeypatch.setenv("DYO_HOST_NUMA", "-1")
    d = make_ctx(wl)
    assert d.query("host_numa") == -1
    d.close()


def _tiny_share_late():
    wl = WL.make("tiny", seed=0, n_samples=32)
    wl.budget = 384 << 20            # RETAIN + SHARE here: ~45 SHARE'd tensors and 9 late_all compactions in 10 steps
    from oracle import run as OR
    trs = [t for r in OR.run(wl, 6, policy=3) for t in r.transitions]
    assert any(t.late_all for t in trs) and any(t.share for t in trs)
    return wl


def test_share_bytes_tiny():
    """R20 SHARE: blocks read SHARE'd tensors in the other half; compactions under the running
    block's tensors wait for its end (late_all); every read sees its latest version."""
    run_bytes(_tiny_share_late(), 6, 3)


def test_share_pipelined_long_blocks():
    """The asynchronous protocol with long emulated blocks (spin before the reads): a late_all
    transition that did not wait for block j-1 would move its tensors under it."""
    run_pipelined(_tiny_share_late(), 6, 3, spin=2_000_000)


def test_share_af_scaled():
    wl = WL.make_af(seed=1, n_samples=8, act_mib=1, weight_mib=1, blocks=8, budget=64 << 20)
    for t in wl.tensors:
        t.nbytes = min(t.nbytes, 1 << 20)
    off = 0
    for t in wl.tensors:
        t.host_off = off
        off += (t.nbytes + 255) // 256 * 256
    run_bytes(wl, 3, 3)
    run_pipelined(wl, 2, 3, spin=200_000)


@pytest.mark.parametrize("strict", [0, 64])
def test_moe_scaled_fetch_after_overlapping_writebacks(strict):
    """R21: with the default per-range order a FETCH DMA waits only for the write-backs it
    overwrites (gradients written back in backward, experts fetched into their slots);
    DYO_F_STRICT_ORDER (64) keeps R12's whole-phase order. Bytes exact both ways, also under the
    asynchronous event protocol."""
    wl = WL.make_moe(seed=5, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    m = run_bytes(wl, 4, 1, flags=strict, dma_min=1 << 20)
    assert m["dma"] > 0
    run_pipelined(wl, 3, 1, dma_min=1 << 20, flags=strict)
    run_pipelined(wl, 3, 1, dma_min=1 << 20, flags=strict, spin=500_000)
