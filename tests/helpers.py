"""Test helpers: build small programs from golden JSON (input construction only)."""
import json
import os
from fractions import Fraction

from workloads import Op, If, Loop

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden")


def load(name):
    with open(os.path.join(GOLDEN, name)) as f:
        return json.load(f)


def build_program(spec, ops):
    out = []
    for it in spec:
        if isinstance(it, str):
            o = ops[it]
            out.append(Op(tuple(o["idioms"]), tuple(tuple(s) for s in o["inputs"]), tuple(o.get("acc", ())), it))
        elif "if" in it:
            out.append(If([build_program(b, ops) for b in it["if"]]))
        else:
            out.append(Loop(build_program(it["loop"], ops), it["lo"], it["hi"]))
    return out


def num(v):
    return float(Fraction(v)) if isinstance(v, str) else float(v)
