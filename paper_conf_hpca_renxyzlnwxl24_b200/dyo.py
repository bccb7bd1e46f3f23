"""Thin ctypes binding of libdyo (include/dyo.h): argument marshalling only.

Every step of the hot path runs inside libdyo.so (CUDA kernels for sm_100a + its C++ DMA
engine). This module flattens the workload description into the C structs, passes torch
device pointers / streams through, and raises on any non-zero dyo_status. There is no CPU
fallback: if libdyo.so is missing the import fails.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from workloads import Op, If, Loop

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libdyo.so")

P = C.c_void_p
i32, i64, f32 = C.c_int32, C.c_int64, C.c_float
PI32, PI64, PF32 = C.POINTER(i32), C.POINTER(i64), C.POINTER(f32)


class Config(C.Structure):
    _fields_ = [("budget", i64), ("align", i32), ("policy", i32), ("max_batch", i32),
                ("max_groups", i32), ("max_entries", i32), ("max_records", i32),
                ("staging_bytes", i64), ("dma_min_bytes", i64), ("flags", i32)]


class Arch(C.Structure):
    _fields_ = [("nn_type", i32), ("S_max", i32), ("D_s", i32), ("h", i32), ("K_max", i32),
                ("branch_head", i32), ("n_nodes", i32), ("node_kind", PI32), ("node_a", PI32),
                ("node_b", PI32), ("node_span", PI32), ("node_tie", PI32), ("n_ops", i32),
                ("op_idioms", PI32), ("op_in_ptr", PI32), ("in_dim_ptr", PI32), ("in_dims", PI64),
                ("op_acc_ptr", PI32), ("acc_tensor", PI32), ("acc_mode", PI32), ("n_tensors", i32),
                ("t_bytes", PI64), ("t_host_off", PI64), ("t_flags", PI32),
                ("acc_stride", PI32), ("node_flags", PI32), ("acc_bstride", PI32)]


class PilotDesc(C.Structure):
    _fields_ = [("F", i32), ("O", i32), ("n_feature", i32), ("feat_off", PI32), ("feat_len", PI32),
                ("feat_out", PI32), ("feat_W", C.POINTER(PF32)), ("feat_b", C.POINTER(PF32)),
                ("n_mlp", i32), ("mlp_in", PI32), ("mlp_out", PI32), ("mlp_W", C.POINTER(PF32)),
                ("mlp_b", C.POINTER(PF32)), ("out_in", i32), ("out_W", PF32), ("out_b", PF32),
                ("slope", C.c_double)]


class Sample(C.Structure):
    _fields_ = [("desc", P), ("hist_ids", P)]


class ArchSummary(C.Structure):
    _fields_ = [("n_sites", i32), ("n_branch_logits", i32), ("n_pieces", i32), ("F", i32),
                ("L_max", i64), ("host_pool_bytes", i64)]


class TransitionInfo(C.Structure):
    _fields_ = [("half", i32), ("n_entries", i32), ("n_evict", i32), ("n_move", i32), ("n_carry", i32),
                ("n_alloc", i32), ("n_fetch", i32), ("need", i64), ("h2d", i64), ("d2h", i64), ("d2d", i64),
                ("n_share", i32), ("late_all", i32)]


class Counters(C.Structure):
    _fields_ = [("h2d_dma", i64), ("h2d_zc", i64), ("d2h_dma", i64), ("d2h_zc", i64),
                ("d2h_packed", i64), ("d2d", i64), ("n_dma", i64), ("n_kernels", i64)]


REC_FIELDS = {0: ("t", "src", "host_off", "bytes", "writeback"),
              1: ("t", "src", "dst", "bytes"),
              2: ("t", "src", "dst", "bytes", "late"),
              3: ("t", "dst", "bytes"),
              4: ("t", "host_off", "dst", "bytes"),
              5: ("t", "mode", "needs_fetch", "dst")}
LISTS = ("evict", "move", "carry", "alloc", "fetch", "entries")


class DyoError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"dyo status {status}: {msg}")
        self.status = status


_lib = None


def lib():
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} not built: run __graft_entry__.build()")
        L = C.CDLL(LIB_PATH)
        L.dyo_strerror.restype = C.c_char_p
        L.dyo_last_error.restype = C.c_char_p
        L.dyo_last_error.argtypes = [P]
        for name in ("dyo_create", "dyo_destroy", "dyo_load_arch", "dyo_load_pilot", "dyo_host_pool",
                     "dyo_arena", "dyo_encode_features", "dyo_pilot_predict", "dyo_prediction_get",
                     "dyo_group_entries", "dyo_plan", "dyo_plan_async", "dyo_plan_wait", "dyo_plan_info", "dyo_plan_records", "dyo_migrate",
                     "dyo_residency", "dyo_get_counters", "dyo_get_timings", "dyo_arch_check",
                     "dyo_debug_pilot_stamps", "dyo_debug_plan_stamps", "dyo_debug_copy", "dyo_traverse_check",
                     "dyo_debug_floor", "dyo_memo_config", "dyo_report", "dyo_memo_stats",
                     "dyo_debug_copy_stamps", "dyo_query", "dyo_set_timing", "dyo_prediction_nested", "dyo_nested_check",
                     "dyo_fault_config", "dyo_fault_fetch", "dyo_fault_stats", "dyo_fault_flush", "dyo_fault_inject", "dyo_partition",
                     "dyo_trace_path", "dyo_trainer_create", "dyo_trainer_step", "dyo_trainer_export",
                     "dyo_trainer_destroy"):
            getattr(L, name).restype = C.c_int
        _lib = L
    return _lib


EXPORTS = ("dyo_strerror", "dyo_last_error", "dyo_version", "dyo_create", "dyo_destroy", "dyo_load_arch",
           "dyo_load_pilot", "dyo_host_pool", "dyo_arena", "dyo_encode_features", "dyo_pilot_predict",
           "dyo_prediction_get", "dyo_prediction_matched", "dyo_group_entries", "dyo_plan", "dyo_plan_async", "dyo_plan_wait",
           "dyo_plan_info", "dyo_plan_records",
           "dyo_migrate", "dyo_residency", "dyo_get_counters", "dyo_get_timings", "dyo_arch_check",
           "dyo_debug_pilot_stamps", "dyo_debug_plan_stamps", "dyo_debug_copy", "dyo_traverse_check",
           "dyo_debug_floor", "dyo_memo_config", "dyo_report", "dyo_memo_stats", "dyo_debug_copy_stamps",
           "dyo_query", "dyo_set_timing", "dyo_prediction_nested", "dyo_nested_check",
           "dyo_fault_config", "dyo_fault_fetch", "dyo_fault_stats", "dyo_fault_flush", "dyo_fault_inject", "dyo_partition",
           "dyo_trace_path", "dyo_trainer_create", "dyo_trainer_step", "dyo_trainer_export", "dyo_trainer_destroy")


def _a(x, dt):
    return np.ascontiguousarray(np.asarray(x, dtype=dt))


def _p(arr, ct):
    return arr.ctypes.data_as(C.POINTER(ct))


def flatten_program(program):
    """Preorder node arrays + operator CSR of the program (marshalling into dyo_arch)."""
    kind, na, nb, span, tie, flags = [], [], [], [], [], []
    ops = []

    def rec(items):
        for it in items:
            idx = len(kind)
            if isinstance(it, Op):
                kind.append(0); na.append(len(ops)); nb.append(0); span.append(0); tie.append(-1)
                ops.append(it)
            elif isinstance(it, If):
                kind.append(1); na.append(len(it.branches)); nb.append(0); span.append(0); tie.append(it.tie)
                for br in it.branches:
                    bidx = len(kind)
                    kind.append(3); na.append(0); nb.append(0); span.append(0); tie.append(-1)
                    rec(br)
                    span[bidx] = len(kind) - bidx - 1
                span[idx] = len(kind) - idx - 1
            elif isinstance(it, Loop):
                kind.append(2); na.append(it.lo); nb.append(it.hi); span.append(0); tie.append(it.tie)
                flags.append((idx, 1 if it.rev else 0))
                rec(it.body)
                span[idx] = len(kind) - idx - 1
            else:
                raise TypeError(it)
    rec(program)
    nflags = [0] * len(kind)
    for i, f in flags:
        nflags[i] = f
    idioms, in_ptr, dim_ptr, dims, acc_ptr, acc_t, acc_m, acc_s, acc_sb = [], [0], [0], [], [0], [], [], [], []
    for op in ops:
        idioms.extend(op.idioms)
        for shp in op.inputs:
            dims.extend(shp)
            dim_ptr.append(len(dims))
        in_ptr.append(len(dim_ptr) - 1)
        for a in op.acc:
            acc_t.append(a[0])
            acc_m.append(a[1])
            acc_s.append(a[2] if len(a) > 2 else 0)
            acc_sb.append(a[3] if len(a) > 3 else 0)
        acc_ptr.append(len(acc_t))
    return dict(kind=_a(kind, np.int32), a=_a(na, np.int32), b=_a(nb, np.int32), span=_a(span, np.int32),
                tie=_a(tie, np.int32), n_ops=len(ops), idioms=_a(idioms, np.int32), in_ptr=_a(in_ptr, np.int32),
                dim_ptr=_a(dim_ptr, np.int32), dims=_a(dims, np.int64), acc_ptr=_a(acc_ptr, np.int32),
                acc_t=_a(acc_t, np.int32), acc_m=_a(acc_m, np.int32), acc_s=_a(acc_s, np.int32), acc_sb=_a(acc_sb, np.int32),
                flags=_a(nflags, np.int32))


def _arch_struct(wl, branch_head=None):
    fp = flatten_program(wl.program)
    bh = wl.notes.get("branch_head", True) if branch_head is None else branch_head
    tb = _a([t.nbytes for t in wl.tensors], np.int64)
    th = _a([t.host_off for t in wl.tensors], np.int64)
    tf = _a([1 if t.transient else 0 for t in wl.tensors], np.int32)
    arch = Arch(wl.nn_type, wl.S_max, wl.D_s, wl.h, wl.K_max, 1 if bh else 0, len(fp["kind"]),
                _p(fp["kind"], i32), _p(fp["a"], i32), _p(fp["b"], i32), _p(fp["span"], i32),
                _p(fp["tie"], i32), fp["n_ops"], _p(fp["idioms"], i32), _p(fp["in_ptr"], i32),
                _p(fp["dim_ptr"], i32), _p(fp["dims"], i64), _p(fp["acc_ptr"], i32), _p(fp["acc_t"], i32),
                _p(fp["acc_m"], i32), len(wl.tensors), _p(tb, i64), _p(th, i64), _p(tf, i32),
                _p(fp["acc_s"], i32), _p(fp["flags"], i32), _p(fp["acc_sb"], i32))
    return arch, (fp, tb, th, tf)


def arch_check(wl, align=256, branch_head=None):
    """Host-only parse of the arch by libdyo (no GPU): (status, summary dict, seg_table, op_sig, err)."""
    arch, keep = _arch_struct(wl, branch_head)
    n_ops = keep[0]["n_ops"]
    summ = ArchSummary()
    seg = np.zeros((max(wl.S_max, 1), 10), np.int32)
    sig = np.zeros((max(n_ops, 1), 9), np.int32)
    err = C.create_string_buffer(512)
    st = lib().dyo_arch_check(C.byref(arch), align, C.byref(summ), _p(seg, i32), _p(sig, i32), err, 512)
    return (st, {f: getattr(summ, f) for f, _ in ArchSummary._fields_}, seg[:wl.S_max], sig[:n_ops],
            err.value.decode())


def traverse_check(wl, slots):
    """Host-only traversal decode by libdyo (no GPU): (status, choices, matched, err)."""
    arch, keep = _arch_struct(wl, False)
    n_sites = sum(1 for k in keep[0]["kind"] if k in (1, 2))
    sl = _a(slots, np.int32).reshape(-1)
    assert sl.size == wl.K_max * 10
    ch = np.zeros(max(n_sites, 1), np.int32)
    m = i32()
    err = C.create_string_buffer(512)
    st = lib().dyo_traverse_check(C.byref(arch), _p(sl, i32), _p(ch, i32), C.byref(m), err, 512)
    return st, ch[:n_sites].tolist(), m.value, err.value.decode()


def nested_check(wl, slots, top_choices, cap=1 << 16):
    """Host-only nested-site decode by libdyo (no GPU): (status, nested, path_ops, matched, err)."""
    arch, keep = _arch_struct(wl)
    sl = _a(slots, np.int32).reshape(-1)
    assert sl.size == wl.K_max * 10
    tc = _a([max(c, 0) if c is not None else 0 for c in top_choices] or [0], np.int32)
    nest = np.zeros(cap, np.int32)
    path = np.zeros(cap, np.int32)
    nn, pl, m = i32(), i32(), i32()
    err = C.create_string_buffer(512)
    st = lib().dyo_nested_check(C.byref(arch), _p(sl, i32), _p(tc, i32), _p(nest, i32), cap, C.byref(nn),
                                _p(path, i32), cap, C.byref(pl), C.byref(m), err, 512)
    return st, nest[:nn.value].tolist(), path[:pl.value].tolist(), m.value, err.value.decode()


def _pilot_desc(spec, keep, slope=0.01):
    """dyo_pilot_desc of a PilotSpec (arrays kept alive in `keep`)."""
    w = spec.weights

    def arr(x, dt=np.float32):
        x = _a(x, dt)
        keep.append(x)
        return x

    def ptrs(names):
        lst = [_p(arr(w[n]), f32) for n in names]
        pa = (PF32 * max(1, len(lst)))(*lst)
        keep.append(pa)
        return pa
    nf = len(spec.feature)
    fo = arr([f[0] for f in spec.feature] or [0], np.int32)
    fl = arr([f[1] for f in spec.feature] or [0], np.int32)
    fu = arr([f[2] for f in spec.feature] or [0], np.int32)
    mi = arr([m[0] for m in spec.mlp], np.int32)
    mo = arr([m[1] for m in spec.mlp], np.int32)
    fW = ptrs([f"feat{i}.W" for i in range(nf)])
    fb = ptrs([f"feat{i}.b" for i in range(nf)])
    mW = ptrs([f"mlp{k}.{l}.W" for k in range(3) for l in range(len(spec.mlp))])
    mb = ptrs([f"mlp{k}.{l}.b" for k in range(3) for l in range(len(spec.mlp))])
    oW, ob = arr(w["out.W"]), arr(w["out.b"])
    return PilotDesc(spec.F, spec.O, nf, _p(fo, i32), _p(fl, i32), _p(fu, i32), fW, fb, len(spec.mlp),
                     _p(mi, i32), _p(mo, i32), mW, mb, spec.out_in, _p(oW, f32), _p(ob, f32), slope)


def weight_names(spec):
    """Weight arrays in dyo_pilot_desc / dyo_trainer_export order."""
    names = []
    for i in range(len(spec.feature)):
        names += [f"feat{i}.W", f"feat{i}.b"]
    for k in range(3):
        for l in range(len(spec.mlp)):
            names += [f"mlp{k}.{l}.W", f"mlp{k}.{l}.b"]
    return names + ["out.W", "out.b"]


class Trainer:
    """dyo_trainer: SGD on a pilot's fp64 copy (reading R19)."""

    def __init__(self, spec, nn_type, max_batch, device=0):
        self.L = lib()
        self.spec = spec
        keep = []
        d = _pilot_desc(spec, keep)
        self.tr = P()
        st = self.L.dyo_trainer_create(C.byref(d), int(nn_type), int(max_batch), int(device), C.byref(self.tr))
        if st:
            raise DyoError(st, "dyo_trainer_create")

    def step(self, feat, target, B, lr=0.01, stream=0, want_loss=True):
        loss = C.c_double(0.0)
        st = self.L.dyo_trainer_step(self.tr, P(Dyo._ptr(feat)), P(Dyo._ptr(target)), int(B), C.c_double(lr),
                                     C.byref(loss) if want_loss else None, P(stream))
        if st:
            raise DyoError(st, "dyo_trainer_step")
        return loss.value

    def weights(self):
        """{name: float64 array} of every weight array (trained and untouched)."""
        n = i64()
        self.L.dyo_trainer_export(self.tr, None, 0, C.byref(n))
        blob = np.zeros(n.value, np.float64)
        st = self.L.dyo_trainer_export(self.tr, blob.ctypes.data_as(C.POINTER(C.c_double)), n.value, C.byref(n))
        if st:
            raise DyoError(st, "dyo_trainer_export")
        out, o = {}, 0
        for name in weight_names(self.spec):
            shp = np.shape(self.spec.weights[name])
            k = int(np.prod(shp))
            out[name] = blob[o:o + k].reshape(shp)
            o += k
        return out

    def close(self):
        if self.tr:
            self.L.dyo_trainer_destroy(self.tr)
            self.tr = P()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Dyo:
    """One manager (dyo_ctx) on one GPU."""

    def __init__(self, budget, align=256, policy=1, max_batch=1, device=0, max_groups=0,
                 staging_bytes=0, dma_min_bytes=0, flags=0):
        self.L = lib()
        self.cfg = Config(budget, align, policy, max_batch, max_groups, 0, 0, staging_bytes, dma_min_bytes, flags)
        self.ctx = P()
        self._check(self.L.dyo_create(C.byref(self.cfg), device, C.byref(self.ctx)), create=True)
        self._keep = []
        self.K = 0

    def _check(self, st, create=False):
        if st != 0:
            msg = "" if create else self.L.dyo_last_error(self.ctx).decode()
            raise DyoError(st, f"{self.L.dyo_strerror(st).decode()}: {msg}")

    def close(self):
        if self.ctx:
            self.L.dyo_destroy(self.ctx)
            self.ctx = P()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- loaders --------------------------------------------------------------------------
    def load_arch(self, wl, branch_head=None):
        arch, keep = _arch_struct(wl, branch_head)
        self._check(self.L.dyo_load_arch(self.ctx, C.byref(arch)))
        del keep

    def load_pilot(self, spec, slope=0.01):
        w = spec.weights
        keep = []

        def arr(x, dt=np.float32):
            x = _a(x, dt)
            keep.append(x)
            return x

        def ptrs(names):
            lst = [_p(arr(w[n]), f32) for n in names]
            pa = (PF32 * max(1, len(lst)))(*lst)
            keep.append(pa)
            return pa
        nf = len(spec.feature)
        fo = arr([f[0] for f in spec.feature] or [0], np.int32)
        fl = arr([f[1] for f in spec.feature] or [0], np.int32)
        fu = arr([f[2] for f in spec.feature] or [0], np.int32)
        mi = arr([m[0] for m in spec.mlp], np.int32)
        mo = arr([m[1] for m in spec.mlp], np.int32)
        fW = ptrs([f"feat{i}.W" for i in range(nf)])
        fb = ptrs([f"feat{i}.b" for i in range(nf)])
        mW = ptrs([f"mlp{k}.{l}.W" for k in range(3) for l in range(len(spec.mlp))])
        mb = ptrs([f"mlp{k}.{l}.b" for k in range(3) for l in range(len(spec.mlp))])
        oW, ob = arr(w["out.W"]), arr(w["out.b"])
        d = PilotDesc(spec.F, spec.O, nf, _p(fo, i32), _p(fl, i32), _p(fu, i32), fW, fb, len(spec.mlp),
                      _p(mi, i32), _p(mo, i32), mW, mb, spec.out_in, _p(oW, f32), _p(ob, f32), slope)
        self._check(self.L.dyo_load_pilot(self.ctx, C.byref(d)))

    def load(self, wl):
        self.load_arch(wl)
        self.load_pilot(wl.pilot)

    def host_pool(self):
        base, n = P(), i64()
        self._check(self.L.dyo_host_pool(self.ctx, C.byref(base), C.byref(n)))
        return base.value, n.value

    def host_pool_array(self):
        base, n = self.host_pool()
        return np.ctypeslib.as_array((C.c_uint8 * n).from_address(base))

    def arena(self):
        base, half = P(), i64()
        self._check(self.L.dyo_arena(self.ctx, C.byref(base), C.byref(half)))
        return base.value, half.value

    # -- hot path -------------------------------------------------------------------------
    @staticmethod
    def _ptr(x):
        if x is None:
            return None
        if hasattr(x, "data_ptr"):
            return x.data_ptr()
        if isinstance(x, np.ndarray):
            return x.ctypes.data
        return int(x)

    def encode(self, desc, hist, B, feat, stream=0):
        s = Sample(self._ptr(desc), self._ptr(hist))
        self._check(self.L.dyo_encode_features(self.ctx, C.byref(s), B, P(self._ptr(feat)), P(stream)))

    def predict(self, desc, hist, B, logits=None, feat=None, stream=0):
        s = Sample(self._ptr(desc), self._ptr(hist))
        self._check(self.L.dyo_pilot_predict(self.ctx, P(self._ptr(feat)), C.byref(s), B,
                                             P(self._ptr(logits)), P(stream)))

    def prediction(self, b, K_max, n_sites, stream=0):
        K = i32()
        blocks = np.zeros((K_max, 10), np.int32)
        choices = np.zeros(max(n_sites, 1), np.int32)
        rows = np.zeros((K_max, 2), np.int32)
        self._check(self.L.dyo_prediction_get(self.ctx, b, C.byref(K), _p(blocks, i32), _p(choices, i32),
                                              _p(rows, i32), P(stream)))
        k = K.value
        return k, blocks[:k].copy(), choices[:n_sites].copy(), rows[:k].copy()

    def matched(self, b):
        """Traversal decode: 1 if prediction b matched a path exactly, 0 if the
        closest-count fallback was taken."""
        m = i32()
        self._check(self.L.dyo_prediction_matched(self.ctx, b, C.byref(m)))
        return m.value

    def nested(self, b, cap=4096):
        """Choices of prediction b's nested-site executions in execution order (reading R16)."""
        out = np.zeros(cap, np.int32)
        n = i32()
        self._check(self.L.dyo_prediction_nested(self.ctx, b, _p(out, i32), cap, C.byref(n)))
        return out[: n.value].tolist()

    def group_entries(self, b, g, cap=1024, stream=0):
        out = np.zeros((cap, 3), np.int32)
        n = i32()
        self._check(self.L.dyo_group_entries(self.ctx, b, g, _p(out, i32), cap, C.byref(n), P(stream)))
        return out[: n.value].copy()

    def plan(self, b0=0, n=-1, stream=0):
        K = i32()
        self._check(self.L.dyo_plan(self.ctx, b0, n, C.byref(K), P(stream)))
        self.K = K.value
        return self.K

    def plan_async(self, b0=0, n=-1, stream=0):
        self._check(self.L.dyo_plan_async(self.ctx, b0, n, P(stream)))

    def plan_wait(self):
        K = i32()
        self._check(self.L.dyo_plan_wait(self.ctx, C.byref(K)))
        self.K = K.value
        return self.K

    def plan_info(self, j):
        info = TransitionInfo()
        self._check(self.L.dyo_plan_info(self.ctx, j, C.byref(info)))
        return {f: getattr(info, f) for f, _ in TransitionInfo._fields_}

    def plan_records(self, j, list_id):
        if isinstance(list_id, str):
            list_id = LISTS.index(list_id)
        ptr, n = P(), i32()
        self._check(self.L.dyo_plan_records(self.ctx, j, list_id, C.byref(ptr), C.byref(n)))
        nf = len(REC_FIELDS[list_id])
        if n.value == 0:
            return np.zeros((0, nf), np.int64)
        buf = (C.c_int64 * (n.value * nf)).from_address(ptr.value)
        return np.ctypeslib.as_array(buf).reshape(n.value, nf).copy()

    def migrate(self, j, stream=0, ev_half_free=None, ev_prev_done=None, ev_ready=None):
        """ev_*: cudaEvent_t handles (torch.cuda.Event.cuda_event) or None."""
        self._check(self.L.dyo_migrate(self.ctx, j, P(stream), P(ev_half_free), P(ev_prev_done), P(ev_ready)))

    def trace_path(self, choices, nested=(), cap=1 << 20):
        """(ops, its) of the resolved path for the given site choices / nested choices."""
        ch = _a(list(choices) or [0], np.int32)
        ne = _a(list(nested) or [0], np.int32)
        ops = np.zeros(cap, np.int32)
        its = np.zeros(cap, np.int32)
        L = i32()
        self._check(self.L.dyo_trace_path(self.ctx, _p(ch, i32), _p(ne, i32), len(nested), _p(ops, i32), _p(its, i32),
                                          cap, C.byref(L)))
        return ops[:L.value].copy(), its[:L.value].copy()

    # ---- partition labels (R18) ----
    METHODS = {"overlap": 0, "even_ops": 1, "even_time": 2, "even_size": 3}

    def partition(self, path_ops, path_it, b, op_time_ns, K, method, H, bw, stream=0):
        """(cuts, exposed_ns, feasible) of one trace (R18); method in METHODS."""
        ops = _a(path_ops, np.int32)
        its = _a(path_it, np.int32)
        ons = _a(op_time_ns, np.int64)
        cuts = np.zeros(K + 1, np.int32)
        ex, fe = i64(), i32()
        self._check(self.L.dyo_partition(self.ctx, _p(ops, i32), _p(its, i32), len(ops), int(b), _p(ons, i64), int(K),
                                         self.METHODS[method] if isinstance(method, str) else int(method), i64(H),
                                         i64(bw), _p(cuts, i32), C.byref(ex), C.byref(fe), P(stream)))
        return cuts.tolist(), ex.value, bool(fe.value)

    # ---- on-demand fetch of mis-predicted tensors (R17) ----
    def fault_config(self, area_bytes):
        self._check(self.L.dyo_fault_config(self.ctx, i64(area_bytes)))

    def fault_fetch(self, j, ids, modes, stream=0, ev_done=None):
        """Device addresses for block j's (possibly) missing accesses (list of ints)."""
        ids_a = _a(ids, np.int32)
        md = _a(modes, np.int32)
        n = len(ids_a)
        ptrs = (P * max(n, 1))()
        self._check(self.L.dyo_fault_fetch(self.ctx, int(j), _p(ids_a, i32), _p(md, i32), n, ptrs, P(stream),
                                           P(ev_done)))
        return [ptrs[i] for i in range(n)]

    def fault_inject(self, p, seed=0):
        self._check(self.L.dyo_fault_inject(self.ctx, C.c_double(p), C.c_uint64(seed)))

    def fault_flush(self, stream=0, ev_block_end=None):
        self._check(self.L.dyo_fault_flush(self.ctx, P(stream), P(ev_block_end)))

    def fault_stats(self):
        f, b, r = i64(), i64(), i64()
        self._check(self.L.dyo_fault_stats(self.ctx, C.byref(f), C.byref(b), C.byref(r)))
        return {"faults": f.value, "bytes": b.value, "resident": r.value}

    def residency(self, t):
        p = P()
        self._check(self.L.dyo_residency(self.ctx, t, C.byref(p)))
        return p.value

    TIMING_KINDS = ("pilot", "decode", "plan", "copy_d2d", "copy_zc", "dma_h2d", "dma_d2h")

    def timings(self, reset=False):
        out = {}
        for k, name in enumerate(self.TIMING_KINDS):
            ms, n, b, busy = C.c_double(), i64(), i64(), C.c_double()
            self._check(self.L.dyo_get_timings(self.ctx, k, C.byref(ms), C.byref(n), C.byref(b), C.byref(busy), 0))
            out[name] = {"ms": ms.value, "launches": n.value, "bytes": b.value, "busy_ms": busy.value}
        if reset:
            self._check(self.L.dyo_get_timings(self.ctx, 0, None, None, None, None, 1))
        return out

    def pilot_stamps(self, enable=True):
        out = np.zeros(32, np.uint64)
        self._check(self.L.dyo_debug_pilot_stamps(self.ctx, 1 if enable else 0, out.ctypes.data_as(C.POINTER(C.c_uint64))))
        return out

    def debug_copy(self, src, dst, nbytes, mode, stream=0):
        self._check(self.L.dyo_debug_copy(self.ctx, P(self._ptr(src)), P(self._ptr(dst)), i64(nbytes), mode, P(stream)))

    # ---- mis-prediction record + exact-match memo (R15) ----
    def memo_config(self, capacity):
        self._check(self.L.dyo_memo_config(self.ctx, int(capacity)))

    def report(self, b, actual):
        """Report the control flow prediction b actually ran; returns True on a mis-prediction."""
        a = _a(actual, np.int32)
        out = C.c_int32(0)
        self._check(self.L.dyo_report(self.ctx, int(b), _p(a, C.c_int32), C.byref(out)))
        return bool(out.value)

    def memo_stats(self):
        mp, live, hits = C.c_int64(0), C.c_int32(0), C.c_int64(0)
        self._check(self.L.dyo_memo_stats(self.ctx, C.byref(mp), C.byref(live), C.byref(hits)))
        return {"mispredictions": mp.value, "live": live.value, "hits": hits.value}

    def debug_floor(self, cluster, n_barriers, stream=0):
        self._check(self.L.dyo_debug_floor(self.ctx, cluster, n_barriers, P(stream)))

    def copy_stamps(self, cap=1 << 22, reset=False):
        """DYO_COPY_STAMPS log: uint64 [n, 4] rows {launch<<32 | cta<<8 | smid, t_enter, t_scan, t_end};
        reset=True empties the log."""
        n = C.c_int64(0)
        if reset:
            self._check(self.L.dyo_debug_copy_stamps(self.ctx, None, 0, C.byref(n)))
            return None
        out = np.zeros((cap, 4), np.uint64)
        self._check(self.L.dyo_debug_copy_stamps(self.ctx, out.ctypes.data_as(C.POINTER(C.c_uint64)), cap,
                                                 C.byref(n)))
        return out[:n.value]

    def plan_stamps(self, j):
        out = np.zeros(64, np.uint64)
        self._check(self.L.dyo_debug_plan_stamps(self.ctx, j, out.ctypes.data_as(C.POINTER(C.c_uint64))))
        return out

    def set_timing(self, on):
        self._check(self.L.dyo_set_timing(self.ctx, 1 if on else 0))

    QUERIES = {"pilot_kernel": 0, "decode_fused": 1, "plan_syncs": 2, "host_decode": 3, "host_numa": 4}

    def query(self, what):
        """dyo_query: 'pilot_kernel' (0 K1 cluster GEMV, 1 K1-TC), 'decode_fused', 'plan_syncs'."""
        v = i64()
        self._check(self.L.dyo_query(self.ctx, self.QUERIES[what], C.byref(v)))
        return v.value

    def counters(self, reset=False):
        c = Counters()
        self._check(self.L.dyo_get_counters(self.ctx, C.byref(c), 1 if reset else 0))
        return {f: getattr(c, f) for f, _ in Counters._fields_}
