"""Executing a plan on bytes (§IV-E L180 evict-then-prefetch, §V L199 wait before
compute; R12).

Oracle — test infrastructure only (see oracle/__init__.py).

ByteSim holds a numpy uint8 "device arena" (2H bytes) and "host pool"; it applies a
transition's lists literally in the paper's order (EVICT writebacks -> MOVE (memmove
semantics, ascending destination) -> CARRY -> FETCH) and then emulates block j: every tensor
the block reads first must hold its latest version, every tensor it writes gets the next
version (the counter-based content of workloads.content_words_np).
A transient tensor's contents end with the step (reading R9): a read of a transient tensor
not yet written in the current step has no defined expected value and is not checked;
call new_step() at every step boundary.
VersionSim does the same on version numbers only, for trace sizes whose bytes do not fit.
"""
from __future__ import annotations

import numpy as np

from workloads import W, content_words_np
from .plan import half_size


def content_bytes(t, v, nbytes):
    words = content_words_np(t, v, (nbytes + 3) // 4)
    return words.view(np.uint8)[:nbytes]


class ByteSim:
    def __init__(self, wl):
        self.wl = wl
        self.H = half_size(wl.budget, wl.align)
        pool = max(t.host_off + t.nbytes for t in wl.tensors)
        self.dev = np.zeros(2 * self.H, np.uint8)
        self.host = np.zeros(pool, np.uint8)
        self.ver = [0] * len(wl.tensors)
        self.fresh = set()
        for t, ten in enumerate(wl.tensors):
            self.host[ten.host_off: ten.host_off + ten.nbytes] = content_bytes(t, 0, ten.nbytes)

    def new_step(self):
        self.fresh = set()

    def _checked(self, t):
        return not self.wl.tensors[t].transient or t in self.fresh

    def apply(self, tr):
        for t, src, ho, nb, wb in tr.evict:
            if wb:
                self.host[ho: ho + nb] = self.dev[src: src + nb]
        for t, old, new, nb in tr.move:
            self.dev[new: new + nb] = self.dev[old: old + nb].copy()
        for t, src, dst, nb, late in tr.carry:
            self.dev[dst: dst + nb] = self.dev[src: src + nb]
        for t, ho, dst, nb in tr.fetch:
            self.dev[dst: dst + nb] = self.host[ho: ho + nb]

    def run_block(self, Wj, half, state):
        """Emulated compute of the block (test harness): returns list of mismatching reads."""
        bad = []
        for t, mode, rd in Wj:
            nb = self.wl.tensors[t].nbytes
            base = state.loc[t] * self.H + state.off[t]      # half m, or 1-m when SHARE'd (R20)
            if rd and self._checked(t) and not np.array_equal(self.dev[base: base + nb],
                                                              content_bytes(t, self.ver[t], nb)):
                bad.append(t)
        for t, mode, rd in Wj:
            if mode & W:
                nb = self.wl.tensors[t].nbytes
                base = state.loc[t] * self.H + state.off[t]      # half m, or 1-m when SHARE'd (R20)
                self.fresh.add(t)
                self.ver[t] += 1
                self.dev[base: base + nb] = content_bytes(t, self.ver[t], nb)
        return bad


class VersionSim:
    """Version-number model of the same execution (any trace size)."""

    def __init__(self, wl):
        self.wl = wl
        T = len(wl.tensors)
        self.ver = [0] * T
        self.host_ver = [0] * T
        self.dev_ver = {}          # absolute device offset -> (tensor, version)
        self.fresh = set()

    def new_step(self):
        self.fresh = set()

    def apply(self, tr):
        for t, src, ho, nb, wb in tr.evict:
            if wb:
                tt, v = self.dev_ver[src]
                assert tt == t
                self.host_ver[t] = v
        snap = dict(self.dev_ver)
        for t, old, new, nb in tr.move:
            self.dev_ver[new] = snap[old]
        for t, src, dst, nb, late in tr.carry:
            self.dev_ver[dst] = self.dev_ver[src]
        for t, ho, dst, nb in tr.fetch:
            self.dev_ver[dst] = (t, self.host_ver[t])

    def run_block(self, Wj, half, state, H):
        bad = []
        for t, mode, rd in Wj:
            base = state.loc[t] * H + state.off[t]          # half m, or 1-m when SHARE'd (R20)
            checked = not self.wl.tensors[t].transient or t in self.fresh
            if rd and checked and self.dev_ver.get(base) != (t, self.ver[t]):
                bad.append(t)
        for t, mode, rd in Wj:
            if mode & W:
                self.fresh.add(t)
                self.ver[t] += 1
                self.dev_ver[state.loc[t] * H + state.off[t]] = (t, self.ver[t])
        return bad
