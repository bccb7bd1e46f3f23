"""Pilot-model input features (§IV-A, §IV-C; R1-R3).

Oracle — test infrastructure only (see oracle/__init__.py).

Feature vector layout (reading R3):  [x_t (3) | x_s (D_s) | x_a (10*S_max) | x_h (10*h)],
zero-padded to F = a multiple of 16.
  x_t  one-hot basic NN type {CNN, LSTM, transformer}
  x_s  input-shape descriptors of the sample (stand-in for the embedding; R3)
  x_a  AFM reduced to S_max segment block vectors (R3)
  x_h  block vectors of the h most recently executed groups (north_star "group-ID history")
Scaling by exact powers of two (R3): counts and idiom sums x 2^-4, dimension sums and
shape descriptors x 2^-10, one-hot x 1.
"""
from __future__ import annotations

import numpy as np

from . import afm as A

COUNT_SCALE = 2.0 ** -4
DIM_SCALE = 2.0 ** -10


def feature_width(S_max, D_s, h):
    return (3 + D_s + 10 * S_max + 10 * h + 15) // 16 * 16


def scale_block10(v):
    """Elements 0..6 (operator count, six idiom sums) x 2^-4; 7..9 (dimension sums) x 2^-10."""
    return [float(v[e]) * (COUNT_SCALE if e < 7 else DIM_SCALE) for e in range(10)]


def static_segment_table(wl):
    """S_max block vectors of the AFM segments (zero vector padding); computed once per arch."""
    segs = A.segments(A.afm_rows(wl.program))
    tab = []
    for s in range(wl.S_max):
        tab.append(A.block10_of_sig_rows(segs[s]) if s < len(segs) else (0,) * 10)
    return tab


def resolve_hist(hist_ids, group_table):
    """History group ids -> block vectors. id >= 0 indexes the table; id < 0 counts from its
    end (-1 = most recent group); out-of-range -> zero vector (reading R3)."""
    out = []
    n = len(group_table)
    for gid in hist_ids:
        gid = int(gid)
        idx = gid if gid >= 0 else n + gid
        out.append(tuple(group_table[idx]) if 0 <= idx < n else (0,) * 10)
    return out


def encode(wl, desc, hist_ids=(), group_table=()):
    """Feature vector (float64, values exactly representable in fp32) for one sample."""
    F = feature_width(wl.S_max, wl.D_s, wl.h)
    x = []
    x += [1.0 if k == wl.nn_type else 0.0 for k in range(3)]
    x += [float(A.sat(d)) * DIM_SCALE for d in desc]
    for v in static_segment_table(wl):
        x += scale_block10(v)
    for v in resolve_hist(hist_ids, group_table):
        x += scale_block10(v)
    x += [0.0] * (F - len(x))
    return np.array(x, dtype=np.float64)
