"""Misprediction record and exact-match memo (§IV-E "Handling mis-prediction",
P:L184-L187; §VI-H) — oracle, TEST INFRASTRUCTURE ONLY (see oracle/__init__.py).

Paper: when the pilot mis-predicts, DyNN-Offload records the resolved architecture and the
input sample, and "the output of the pilot model is compared with the output where
there is mis-prediction. If the two outputs are exactly the same, then the correct execution
block in the mis-prediction case is used to resolve the control flows for the new DyNN-training
sample".

Readings (R15):
  * the pilot OUTPUT compared "exactly" is the decoded integer output of a prediction: the raw
    block head (K_max x 10 ints, reading R4) and the branch-head choice of every site — integer
    equality, so the comparison does not depend on floating-point summation order;
  * a mis-prediction is a resolved control flow that differs from the predicted one (the
    choices; a different partition of the same path moves no tensor in or out of a group's
    path and is not a mis-prediction of the control flow);
  * the memo maps that output to the ACTUAL choices ("the correct execution block ... resolves
    the control flows"); a hit replaces the predicted choices, and the groups are cut from the
    resolved actual path at the predicted counts (reading R4's cut rule), so the block head
    still partitions the path;
  * a later report for the same output replaces the value (most recent wins); capacity is
    bounded (FIFO replacement of the oldest key).

Plain dict + list; no hashing (the library hashes; the oracle compares keys exactly).
"""
from __future__ import annotations

from . import afm as A
from . import decode as D


def key_of(pred):
    """The exact-match key of a prediction: (raw block head, predicted choices)."""
    return (tuple(v for slot in pred.slots for v in slot), tuple(pred.choices))


class Memo:
    def __init__(self, capacity=4096):
        self.capacity = capacity
        self.table = {}
        self.order = []          # insertion order of live keys (FIFO replacement)
        self.mispredictions = 0
        self.records = []        # (sample index, actual choices): the paper's training record

    def report(self, pred, actual, sample=None):
        """Compare a prediction with the control flow that actually ran; on a mis-prediction
        record it and memoise the actual choices under the prediction's key. Returns True on a
        mis-prediction."""
        actual = tuple(int(c) for c in actual)
        if actual == tuple(pred.choices):
            return False
        self.mispredictions += 1
        self.records.append((sample, actual))
        k = key_of(pred)
        if k in self.table:
            self.order.remove(k)
        elif len(self.order) >= self.capacity:
            del self.table[self.order.pop(0)]
        self.table[k] = actual
        self.order.append(k)
        return True

    def lookup(self, pred):
        return self.table.get(key_of(pred))


def apply(wl, pred, choices, b=0):
    """The prediction with its control flow resolved by `choices` (a memo hit): the actual path,
    cut at the predicted counts (R4), its block vectors and tensor sets."""
    path = A.resolve(wl.program, list(choices), b)
    counts = [v[0] for v in pred.slots if v[0] != 0]
    groups = D.cut(len(path), counts)
    blocks = [A.block10(path[s:e]) for s, e in groups]
    return D.Prediction(list(choices), path, groups, blocks, D.tensor_sets(path, groups), pred.slots,
                        pred.near_ties, pred.matched)


def decode_with_memo(wl, y, memo, b=0):
    """Decode (branch head) and, if the decoded output is a memoised mis-prediction, resolve the
    control flow with the recorded actual choices."""
    pred = D.decode(wl, y, branch_head=True, b=b)
    hit = memo.lookup(pred) if memo is not None else None
    return (apply(wl, pred, hit, b), True) if hit is not None else (pred, False)


def valid_choices(program, choices):
    """Actual choices must be in range and replay their tie targets (reading R6)."""
    sl = A.sites(program)
    if len(choices) != len(sl):
        return False
    for i, s in enumerate(sl):
        if not 0 <= choices[i] < A.n_choices(s):
            return False
        if s.tie >= 0 and choices[i] != choices[s.tie]:
            return False
    return True
