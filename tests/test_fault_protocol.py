"""Reading R17 as a protocol, on version numbers (no GPU): with the oracle's plans, mis-predicted
MoE routing (workloads.actual_choices) executed block by block with R17's rules - slot vs fault
(oracle.fault.classify), fault-area sources, repairs of ALLOC'd slots the actual block does not
write, write-backs after the block - every first read sees the latest version, and at the end
every host home / resident copy of a persistent tensor holds its latest version. (The GPU test
test_gpu_fault.py checks the library against the same expectations on bytes.)"""
import workloads as WL
from workloads import R, W
from oracle import plan as PL, fault as F
from gpu_harness import oracle_step


def test_r17_keeps_every_persistent_tensor_current():
    wl = WL.make_moe(seed=2, n_samples=8, expert_mib=1, act_mib=1, budget=96 << 20)
    T = len(wl.tensors)
    H = PL.half_size(wl.budget, wl.align)
    dev, host = {}, [0] * T                      # device slot -> (t, version); host home version
    loc, off = [-1] * T, [0] * T                  # residency after the last transition
    st, table = PL.initial_state(T), ()
    ver, pending, n_fault = [0] * T, [], 0
    for s in range(4):
        r = oracle_step(wl, [s], st, table, 1)
        pred = r["preds"][0]
        actual, _ = F.actual_sets(wl, WL.actual_choices(wl, s), [v[0] for v in pred.slots if v[0]])
        fresh = set()
        for j, tr in enumerate(r["trs"]):
            m = tr.half
            for t, v in pending:                  # write-backs of the previous block
                host[t] = v
                if loc[t] >= 0:
                    dev[loc[t] * H + off[t]] = (t, v)
            pending = []
            for t, src, ho, nb, wb in tr.evict:
                if wb:
                    assert dev.get(src, (None,))[0] == t
                    host[t] = dev[src][1]
            for t, old, new, nb in tr.move:
                dev[new] = dev.get(old)
            for t, src, dst, nb, late in tr.carry:
                dev[dst] = dev.get(src)
            prev = {}
            for t, *_ in tr.evict:
                loc[t] = -1
            for t, old, new, nb in tr.move:
                off[t] = new - m * H
            for t, src, dst, nb, late in tr.carry:
                loc[t], off[t] = m, dst - m * H
            for t, dst, nb in tr.alloc:
                prev[t] = (loc[t], off[t])
                loc[t], off[t] = m, dst - m * H
                dev[dst] = ("unwritten", t)
            for t, ho, dst, nb in tr.fetch:
                dev[dst] = (t, host[t])
                loc[t], off[t] = m, dst - m * H
            Aj = actual[j] if j < len(actual) else []
            cls = F.classify(r["Ws"][j], Aj)
            where, fa = {}, {}
            for t, md, kind in cls:
                if kind == "slot":
                    where[t] = m * H + off[t]
                else:
                    n_fault += 1
                    l, o = prev.get(t, (loc[t], off[t]))
                    if md & R:
                        fa[t] = dev[l * H + o][1] if l >= 0 else host[t]
            for t, (l, o) in prev.items():           # repairs
                if not any(x == t and (md & W) and kind == "slot" for x, md, kind in cls):
                    dev[m * H + off[t]] = dev[l * H + o] if l >= 0 else (t, host[t])
            first_reads = {t for t, _, rd in Aj if rd}
            for t, md, kind in cls:
                if t in first_reads and (not wl.tensors[t].transient or t in fresh):
                    got = dev.get(where[t]) if t in where else (t, fa.get(t))
                    assert got == (t, ver[t]), (s, j, t, got, ver[t])
            for t, md, kind in cls:
                if md & W:
                    ver[t] += 1
                    fresh.add(t)
                    if t in where:
                        dev[where[t]] = (t, ver[t])
                    else:
                        pending.append((t, ver[t]))
        st, table = r["state"], r["table"]
    for t, v in pending:
        host[t] = v
        if loc[t] >= 0:
            dev[loc[t] * H + off[t]] = (t, v)
    assert n_fault > 0
    for t, ten in enumerate(wl.tensors):
        if ten.transient:
            continue
        if st.loc[t] != PL.HOST:
            assert dev.get(st.loc[t] * H + st.off[t]) == (t, ver[t]), (t, ten.name)
        else:
            assert host[t] == ver[t], (t, ten.name)
