"""On-demand fetch of mis-predicted tensors ("DyNN-Offload checks whether the
tensor is in GPU memory ... migrates the tensors on demand", P:L197 tensor fault handler;
DESIGN.md reading R17).

Oracle — test infrastructure only (see oracle/__init__.py).

When the pilot mis-predicts, execution still follows the ACTUAL control flow, and block j is
the rows [C_j, C_{j+1}) of the actual path cut at the PREDICTED cumulative counts (the
operator counter of P:L178 triggers the migrations at the predicted boundaries; reading R4's
cut rule). An access of actual block j is served from its planned slot when the plan made the
tensor ready for it (residency check), otherwise it faults: the tensor's latest bytes are
copied into a fault area (outside the budget), and a written faulted tensor is written back
after the block to its host home and to its valid device copy. The plan is not changed.
"""
from __future__ import annotations

from workloads import R, W
from . import afm as A, decode as D


def actual_sets(wl, actual_choices, counts, b=0, nested=None):
    """Tensor sets of the actual blocks: the actual path (top-level choices `actual_choices`,
    nested executions `nested`) cut at the predicted counts (R4 cut rule)."""
    path = A.resolve(wl.program, list(actual_choices), b, nested=nested)
    groups = D.cut(len(path), list(counts))
    return D.tensor_sets(path, groups), groups


def classify(planned, actual):
    """planned, actual: one block's [(t, mode, needs_fetch)] (planned W_j, actual W_j).
    Returns [(t, mode, kind)] for the actual accesses in first-access order, kind "slot" when
    the plan made t ready for this access - in the planned set, read first there or written
    first here, and written here only if the plan writes it (otherwise a write the plan does not
    know about would leave a device copy it treats as clean) - else "fault"."""
    plan = {t: (m, rd) for t, m, rd in planned}
    out = []
    for t, m, rd in actual:
        p = plan.get(t)
        ok = p is not None and (p[1] or not rd) and (not (m & W) or (p[0] & W))
        out.append((t, m, "slot" if ok else "fault"))
    return out
