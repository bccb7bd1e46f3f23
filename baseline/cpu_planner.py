"""ctypes binding of baseline/libcpuplan.so - the compiled single-core CPU planner (a bench and
test baseline, not part of libdyo)."""
import ctypes as C
import os

import numpy as np

_LIB = None


def lib():
    global _LIB
    if _LIB is None:
        path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "libcpuplan.so")
        L = C.CDLL(path)
        L.cpu_plan_create.restype = C.c_void_p
        L.cpu_plan_create.argtypes = [C.c_int32]
        L.cpu_plan_destroy.argtypes = [C.c_void_p]
        L.cpu_plan.restype = C.c_int32
        _LIB = L
    return _LIB


def _p(a, t):
    return a.ctypes.data_as(C.POINTER(t))


class CpuPlanner:
    def __init__(self, wl, policy=None):
        self.wl = wl
        self.policy = wl.policy if policy is None else policy
        self.st = lib().cpu_plan_create(len(wl.tensors))
        self.bytes = np.array([t.nbytes for t in wl.tensors], np.int64)
        self.host = np.array([t.host_off for t in wl.tensors], np.int64)
        self.tr = np.array([1 if t.transient else 0 for t in wl.tensors], np.int32)

    def plan(self, Ws, cap=1 << 20):
        """Ws: per group [(t, mode, needs_fetch)]. Returns (status, transitions as oracle-like dicts)."""
        K = len(Ws)
        ptr = np.zeros(K + 1, np.int32)
        for j, Wj in enumerate(Ws):
            ptr[j + 1] = ptr[j] + len(Wj)
        ent = [e for Wj in Ws for e in Wj]
        et = np.array([e[0] for e in ent] or [0], np.int32)
        em = np.array([e[1] for e in ent] or [0], np.int32)
        er = np.array([int(e[2]) for e in ent] or [0], np.int32)
        hdr = np.zeros((K, 10), np.int64)
        ev, mv = np.zeros((cap, 5), np.int64), np.zeros((cap, 4), np.int64)
        ca, al, fe = np.zeros((cap, 5), np.int64), np.zeros((cap, 3), np.int64), np.zeros((cap, 4), np.int64)
        cnt = np.zeros(6, np.int64)
        i64 = C.c_int64
        st = lib().cpu_plan(C.c_void_p(self.st), len(self.bytes), _p(self.bytes, i64), _p(self.host, i64),
                            _p(self.tr, C.c_int32), i64(self.wl.budget), i64(self.wl.align), self.policy, K,
                            _p(ptr, C.c_int32), _p(et, C.c_int32), _p(em, C.c_int32), _p(er, C.c_int32), i64(cap),
                            _p(hdr, i64), _p(ev, i64), _p(mv, i64), _p(ca, i64), _p(al, i64), _p(fe, i64), _p(cnt, i64))
        if st:
            return st, None
        out, o = [], [0] * 5
        for j in range(K):
            h = hdr[j]
            n = [int(h[1]), int(h[2]), int(h[3]), int(h[4]), int(h[5])]
            rec = {}
            for i, (name, arr) in enumerate((("evict", ev), ("move", mv), ("carry", ca), ("alloc", al), ("fetch", fe))):
                rec[name] = arr[o[i]:o[i] + n[i]].tolist()
                o[i] += n[i]
            rec.update(half=int(h[0]), h2d=int(h[6]), d2h=int(h[7]), d2d=int(h[8]), need=int(h[9]))
            out.append(rec)
        return 0, out

    def close(self):
        if self.st:
            lib().cpu_plan_destroy(C.c_void_p(self.st))
            self.st = None
