"""PyTorch integration (survey §8(f) rank 3; §IV-E L176-L180 runtime, §V
"initially allocates all tensors on CPU memory", the operator counter replaced by block-boundary
events): a small real DyNN - a Tree-LSTM over binary parse trees (workloads.make_tree) - trained
with torch operators on the GPU while every one of its tensors lives in libdyo-managed memory.

Allocation is CPU-first: each DyNN tensor's home is in the ctx's pinned host pool (its initial
contents are written there); on the device a tensor only exists as a slot of the arena that the
plan assigns to the block using it, viewed as a torch tensor through __cuda_array_interface__.
Per step: dyo_pilot_predict + dyo_plan, then per block j: dyo_migrate(j) on a copy stream (its
evictions wait for block j-2's end event, its late carries for block j-1's), the compute stream
waits ready[j], dyo_fault_fetch(j) resolves every access of the ACTUAL block (the pilot does not
predict the order of nodes inside a block, so a leaf predicted where an internal node runs
faults in - reading R17), the block's operators run as torch ops on those views, and an event marks
the block's end. `mode="resident"` runs the same operators with every tensor a plain device tensor
(the PyTorch baseline): the two modes compute bit-identical weights.

Operator semantics (by the workload's operator names; fp32, d = hidden):
  embed: pool = 0              leaf: h_k = tanh(W_leaf x_k), c_k = x_k, g_k[:d] = pre, pool += h_k
  compose: h_k = tanh(W_comp [h_{k-1}; h_{k-2}]), c_k = (c_{k-1} + c_{k-2}) / 2, g_k[:d] = pre
  norm: g_k[d:] = h_k, pool += h_k       loss: loss[0] = sum(pool), dpool = 1e-3
  node_bwd: dpre = (1 - h_k^2) dpool; gW_leaf += 1e-3 dpre x_k^T; gW_comp[:, :d] += 1e-3 dpre c_k^T
  optimizer: W -= 0.01 gW; gW = 0
"""
from __future__ import annotations

import numpy as np

import workloads as WL
from .dyo import Dyo


class _Dev:
    def __init__(self, ptr, n):
        self.__cuda_array_interface__ = {"shape": (n,), "typestr": "<f4", "data": (int(ptr), False), "version": 3}


def _ops_of(program):
    ops = []

    def rec(items):
        for it in items:
            if isinstance(it, WL.Op):
                ops.append(it)
            elif isinstance(it, WL.If):
                for br in it.branches:
                    rec(br)
            else:
                rec(it.body)
    rec(program)
    return ops


class TreeLSTMRuntime:
    def __init__(self, wl, mode="dyo", device=0, seed=0, fault_area=256 << 20, timing=False):
        import torch
        self.torch = torch
        self.wl = wl
        self.mode = mode
        self.dev = torch.device("cuda", device)
        self.B = wl.notes["batch"]
        self.d_hidden = 512 if wl.tensors[0].nbytes >= 4 * 512 * 512 * 2 else None
        self.ops = _ops_of(wl.program)
        self.names = [t.name for t in wl.tensors]
        self.idx = {n: i for i, n in enumerate(self.names)}
        hb = wl.tensors[self.idx["pool"]].nbytes
        self.d = hb // 4
        rng = np.random.default_rng(seed)
        d = self.d
        init = {}
        init[self.idx["W_leaf"]] = (rng.standard_normal(d * d) / np.sqrt(d)).astype(np.float32)
        init[self.idx["W_comp"]] = (rng.standard_normal(2 * d * d) / np.sqrt(2 * d)).astype(np.float32)
        for t, ten in enumerate(wl.tensors):
            if ten.name.startswith("x["):
                init[t] = rng.standard_normal(d).astype(np.float32)
        self.init = init
        if mode == "resident":
            self.buf = [torch.zeros(ten.nbytes // 4, dtype=torch.float32, device=self.dev) for ten in wl.tensors]
            for t, v in init.items():
                self.buf[t][:v.size].copy_(torch.from_numpy(v))
        else:
            self.dyo = Dyo(wl.budget, wl.align, wl.policy, max_batch=self.B, device=device,
                           flags=8 if timing else 0)
            self.dyo.load(wl)
            self.dyo.fault_config(fault_area)
            pool = self.dyo.host_pool_array()
            pool[:] = 0
            for t, v in init.items():
                off = wl.tensors[t].host_off
                pool[off: off + v.size * 4] = v.view(np.uint8)
            self.s_copy = torch.cuda.Stream(device=self.dev)
            self.s_comp = torch.cuda.Stream(device=self.dev)
            n_ev = self.B * wl.K_max + 2
            self.ready = [torch.cuda.Event() for _ in range(n_ev)]
            self.end = [torch.cuda.Event() for _ in range(n_ev)]
            self.t0 = torch.cuda.Event()
            for e in self.ready + self.end + [self.t0]:
                e.record(self.s_copy)
            torch.cuda.synchronize()
        self.faults = 0

    # ---- operator semantics -------------------------------------------------------------------
    def _view(self, t, ptrs):
        n = self.wl.tensors[t].nbytes // 4
        if self.mode == "resident":
            return self.buf[t]
        return self.torch.as_tensor(_Dev(ptrs[t], n), device=self.dev)

    def _run_op(self, op, it, b, V):
        torch = self.torch
        d = self.d
        acc = [(a[0] + (a[2] if len(a) > 2 else 0) * it + (a[3] if len(a) > 3 else 0) * b, a[1]) for a in op.acc]
        ts = [t for t, _ in acc]
        name = op.name
        nm = {self.names[t].split("[")[0]: t for t in ts}
        if name == "embed":
            V(nm["pool"])[:d].zero_()
        elif name == "leaf":
            x = V(nm["x"])[:d]
            W = V(nm["W_leaf"])[:d * d].view(d, d)
            pre = W @ x
            h = torch.tanh(pre)
            k = [t for t in ts if self.names[t].startswith("h[")][0]
            V(k)[:d].copy_(h)
            V([t for t in ts if self.names[t].startswith("c[")][0])[:d].copy_(x)
            V([t for t in ts if self.names[t].startswith("g[")][0])[:d].copy_(pre)
            V(nm["pool"])[:d].add_(h)
        elif name == "compose":
            hs = sorted(t for t in ts if self.names[t].startswith("h["))       # h[k-2], h[k-1], h[k]
            cs = sorted(t for t in ts if self.names[t].startswith("c["))
            g = [t for t in ts if self.names[t].startswith("g[")][0]
            u = torch.cat([V(hs[1])[:d], V(hs[0])[:d]])
            W = V(nm["W_comp"])[:2 * d * d].view(d, 2 * d)
            pre = W @ u
            V(hs[2])[:d].copy_(torch.tanh(pre))
            V(cs[2])[:d].copy_((V(cs[1])[:d] + V(cs[0])[:d]) * 0.5)
            V(g)[:d].copy_(pre)
        elif name == "norm":
            h = [t for t in ts if self.names[t].startswith("h[")][0]
            g = [t for t in ts if self.names[t].startswith("g[")][0]
            V(g)[d:2 * d].copy_(V(h)[:d])
            V(nm["pool"])[:d].add_(V(h)[:d])
        elif name == "loss":
            V(nm["loss"])[0:1].copy_(V(nm["pool"])[:d].sum().view(1))
            V(nm["dpool"])[:d].fill_(1e-3)
        elif name == "node_bwd":
            h = V(nm["h"])[:d]
            c = V(nm["c"])[:d]
            x = V(nm["x"])[:d]
            dpre = (1.0 - h * h) * V(nm["dpool"])[:d]
            V(nm["gW_leaf"])[:d * d].view(d, d).add_(torch.outer(dpre, x), alpha=1e-3)
            V(nm["gW_comp"])[:2 * d * d].view(d, 2 * d)[:, :d].add_(torch.outer(dpre, c), alpha=1e-3)
        elif name == "optimizer":
            for w, gw in (("W_leaf", "gW_leaf"), ("W_comp", "gW_comp")):
                n = d * d if w == "W_leaf" else 2 * d * d
                V(nm[w])[:n].sub_(V(nm[gw])[:n], alpha=0.01)
                V(nm[gw])[:n].zero_()
        else:
            raise ValueError(name)

    # ---- the actual (true) path of a sample ----------------------------------------------------
    def _actual_path(self, s):
        wl = self.wl
        tree = wl.notes["trees"][s]
        N = len(tree)
        lo = wl.program[1].lo
        ch = [N - lo, 0, N - lo]                    # loop F, (nested If), tied loop B
        return ch, list(tree)

    def _block_accesses(self, rows, b):
        """(ids, modes) of a block's rows in first-access order, mode union (R8)."""
        order, mode = [], {}
        for op_i, it in rows:
            if op_i < 0:
                continue
            op = self.ops[op_i]
            accs = sorted((a[0] + (a[2] if len(a) > 2 else 0) * it + (a[3] if len(a) > 3 else 0) * b, a[1])
                          for a in op.acc)
            for t, m in accs:
                if t not in mode:
                    order.append(t)
                    mode[t] = m
                else:
                    mode[t] |= m
        return order, [mode[t] for t in order]

    def step(self, sample_ids):
        """One training step over the batch's samples (sample order)."""
        torch = self.torch
        wl = self.wl
        B = len(sample_ids)
        paths = []
        for s in sample_ids:
            ch, nest = self._actual_path(s)
            if self.mode == "resident":
                ops_l, its = self._trace_host(ch, nest)
            else:
                ops_l, its = self.dyo.trace_path(ch, nest)
            paths.append((list(map(int, ops_l)), list(map(int, its))))
        if self.mode == "resident":
            V = lambda t: self.buf[t]
            for b, (ops_l, its) in enumerate(paths):
                for op_i, it in zip(ops_l, its):
                    if op_i >= 0:
                        self._run_op(self.ops[op_i], it, b, V)
            return
        dy = self.dyo
        cs = torch.cuda.current_stream().cuda_stream
        desc = wl.samples[sample_ids].copy()
        hist = np.tile(wl.hist_ids.astype(np.int32), (B, 1))
        dy.predict(desc, hist, B, stream=cs)
        K = dy.plan(stream=cs)
        # the actual blocks: each sample's actual path cut at its predicted group boundaries
        blocks = []
        for b in range(B):
            Kb, _, _, rows = dy.prediction(b, wl.K_max, 4096, cs)
            ops_l, its = paths[b]
            L = len(ops_l)
            for g in range(Kb):
                st_, en = int(rows[g][0]), int(rows[g][1])
                if g == Kb - 1:
                    en = L
                blocks.append((b, [(ops_l[r], its[r]) for r in range(min(st_, L), min(en, L))]))
        assert len(blocks) == K
        self.t0.record(self.s_copy)
        for j in range(K):
            hf = self.end[j - 2] if j >= 2 else self.t0
            pdn = self.end[j - 1] if j >= 1 else self.t0
            dy.migrate(j, self.s_copy.cuda_stream, hf.cuda_event, pdn.cuda_event, self.ready[j].cuda_event)
            self.s_comp.wait_event(self.ready[j])
            b, rows = blocks[j]
            ids, modes = self._block_accesses(rows, b)
            ptr_l = dy.fault_fetch(j, ids, modes, self.s_comp.cuda_stream)
            ptrs = dict(zip(ids, ptr_l))
            with torch.cuda.stream(self.s_comp):
                V = lambda t: self._view(t, ptrs)
                for op_i, it in rows:
                    if op_i >= 0:
                        self._run_op(self.ops[op_i], it, b, V)
            self.end[j].record(self.s_comp)
        dy.fault_flush(self.s_comp.cuda_stream)
        self.s_copy.wait_stream(self.s_comp)
        torch.cuda.current_stream().wait_stream(self.s_copy)

    def _trace_host(self, ch, nest):
        """Resident mode has no libdyo ctx: the same rows from the program (R2 + R16 order)."""
        rows = []
        it_n = iter(nest)
        opi = {id(o): i for i, o in enumerate(self.ops)}

        def rec(items, k):
            for item in items:
                if isinstance(item, WL.Op):
                    rows.append((opi[id(item)], k))
                elif isinstance(item, WL.If):
                    rows.append((-1, k))
                    rec(item.branches[next(it_n)], k)
                else:
                    n = item.lo + ch[0]
                    for i in range(n):
                        rows.append((-1, k))
                        rec(item.body, n - 1 - i if item.rev else i)
                    rows.append((-1, k))
        rec(self.wl.program, 0)
        return [r[0] for r in rows], [r[1] for r in rows]

    def weights(self):
        """Current W_leaf, W_comp (numpy) - from the device slot or the host home."""
        torch = self.torch
        torch.cuda.synchronize()
        out = {}
        d = self.d
        for name, n in (("W_leaf", d * d), ("W_comp", 2 * d * d)):
            t = self.idx[name]
            if self.mode == "resident":
                out[name] = self.buf[t][:n].cpu().numpy()
            else:
                p = self.dyo.residency(t)
                if p:
                    out[name] = torch.as_tensor(_Dev(p, n), device=self.dev).cpu().numpy()
                else:
                    off = self.wl.tensors[t].host_off
                    out[name] = self.dyo.host_pool_array()[off: off + 4 * n].view(np.float32).copy()
        return out

    def close(self):
        if self.mode != "resident":
            self.faults = self.dyo.fault_stats()
            self.dyo.close()
