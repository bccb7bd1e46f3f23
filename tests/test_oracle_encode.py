"""Pins for oracle/encode.py: hand-computed feature vector; exact fp32 representability."""
import numpy as np

from oracle import encode as E
from workloads import Workload, PilotSpec
from helpers import load, build_program, num
import workloads as WL


def _wl_from_golden():
    g = load("tree_cnn_node.json")
    e = g["encode"]
    prog = build_program(g["program"], g["ops"])
    return Workload("hand", e["nn_type"], prog, [], e["S_max"], e["D_s"], e["h"], 3, 0, 256, 1,
                    PilotSpec(48, 8, [], [], 0, {}), np.array([e["desc"]]), np.array(e["hist_ids"]), 0), e


def test_hand_feature_vector():
    wl, e = _wl_from_golden()
    x = E.encode(wl, e["desc"], e["hist_ids"], e["group_table"])
    assert len(x) == e["F"] == E.feature_width(wl.S_max, wl.D_s, wl.h)
    assert x.tolist() == [num(v) for v in e["x_num"]]


def test_missing_history_is_zero():
    wl, e = _wl_from_golden()
    x = E.encode(wl, e["desc"], [-5], e["group_table"])
    assert np.all(x[35:45] == 0)
    x2 = E.encode(wl, e["desc"], [0], e["group_table"])
    assert x2[35] == 3 / 16


def test_features_exact_in_fp32():
    for name in ("tiny", "moe", "af"):
        wl = WL.make(name)
        x = E.encode(wl, wl.samples[0], wl.hist_ids, [(100, 7, 0, 3, 9, 1, 2, 70000, 5000, 1)] * 3)
        assert np.array_equal(x.astype(np.float32).astype(np.float64), x)
        assert len(x) == wl.pilot.F
