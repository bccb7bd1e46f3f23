"""One oracle step of the hot path: encode -> pilot -> decode -> plan.

Oracle — test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

from dataclasses import dataclass

import numpy as np

from . import encode as E, pilot as P, decode as D, plan as PL


@dataclass
class StepResult:
    feat: np.ndarray
    logits: np.ndarray
    pred: D.Prediction
    transitions: list
    state: PL.State
    error: str = ""


def step(wl, sample, state, group_table=(), branch_head=None, policy=None):
    bh = wl.notes.get("branch_head", True) if branch_head is None else branch_head
    x = E.encode(wl, wl.samples[sample], wl.hist_ids, group_table)
    y = P.forward(wl.pilot, x, wl.nn_type)
    pred = D.decode(wl, y, branch_head=bh)
    try:
        trs, st = PL.plan(state, wl, pred.W, policy)
        return StepResult(x, y, pred, trs, st)
    except PL.BudgetError as e:
        return StepResult(x, y, pred, [], state, str(e))


def run(wl, n_steps, policy=None, branch_head=None):
    """Consecutive steps over samples 0..n_steps-1 with the history table fed forward."""
    st = PL.initial_state(len(wl.tensors))
    table = ()
    out = []
    for s in range(n_steps):
        r = step(wl, s % len(wl.samples), st, table, branch_head, policy)
        out.append(r)
        st = r.state
        table = r.pred.blocks
    return out


def step_batch(wl, samples, state, group_table=(), branch_head=None, policy=None):
    """A batch of predictions planned as one sequence (sample order, reading R13's per-sample
    tensors: prediction b of the batch names its own tensors). Returns (preds, transitions,
    state, error)."""
    bh = wl.notes.get("branch_head", True) if branch_head is None else branch_head
    preds = []
    for b, smp in enumerate(samples):
        x = E.encode(wl, wl.samples[smp], wl.hist_ids, group_table)
        y = P.forward(wl.pilot, x, wl.nn_type)
        preds.append(D.decode(wl, y, branch_head=bh, b=b))
    Ws = [Wj for p in preds for Wj in p.W]
    try:
        trs, st = PL.plan(state, wl, Ws, policy)
        return preds, trs, st, ""
    except PL.BudgetError as e:
        return preds, [], state, str(e)
