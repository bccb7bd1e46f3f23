"""Pins for nested control flow (reading R16): a site inside a loop body or an If arm
takes its own choice at every execution; the traversal resolves those choices."""
import numpy as np
from hypothesis import given, settings, strategies as st

from oracle import afm as A, decode as D
from workloads import Op, If, Loop, R, W
from helpers import load, build_program


def _name(rows):
    return [r.name if r is not None else "Z" for r in rows]


def _prog():
    g = load("tree_cnn_loop.json")
    return g, build_program(g["program"], g["ops"])


def test_signatures_and_afm_of_the_loop():
    g, prog = _prog()
    ops = [r for r in A.resolve(prog, [0, -1], nested=[1]) if r is not None]
    for op in ops:
        assert list(A.signature(op)) == g["signatures"][op.name]
    # AFM: the loop's control row, the node's four ops, the If's control row, its branch op
    assert [("Z" if c else "op") for c, _ in A.afm_rows(prog)] == ["Z", "op", "op", "op", "op", "Z", "op"]


def test_resolve_per_iteration_choices():
    g, prog = _prog()
    r = g["resolved"]
    assert _name(A.resolve(prog, r["top_choices"], nested=r["nested"])) == r["path"]
    assert A.nested_ids(prog) == {id(prog[0].body[4])}


def test_three_blocks_hand_values_and_traversal():
    g, prog = _prog()
    r = g["resolved"]
    rows = A.resolve(prog, r["top_choices"], nested=r["nested"])
    blocks = [tuple(v) for v in g["three_blocks"]["block10"]]
    cuts = D.cut(len(rows), [v[0] for v in blocks])
    assert [A.block10(rows[s:e]) for s, e in cuts] == blocks
    ch, nest, path, ok = D.traversal_nested(prog, blocks)
    assert ok and ch == r["top_choices"] and nest == r["nested"] and _name(path) == r["path"]
    # with the top-level choice given (branch head), the nested executions alone
    nest2, path2, ok2 = D.nested_traversal(prog, r["top_choices"], blocks)
    assert ok2 and nest2 == r["nested"] and path2 == path


def test_order_within_a_block_is_lexicographically_first():
    g, prog = _prog()
    o = g["one_block"]
    blocks = [tuple(v) for v in o["block10"]]
    for nest in ([1, 0], [0, 1]):
        rows = A.resolve(prog, o["top_choices"], nested=nest)
        assert A.block10(rows) == blocks[0]
    ch, nest, path, ok = D.traversal_nested(prog, blocks)
    assert ok and ch == o["top_choices"] and nest == o["nested"]


def test_fallback_closest_count():
    g, prog = _prog()
    f = g["fallback"]
    ch, nest, path, ok = D.traversal_nested(prog, [tuple(v) for v in f["block10"]])
    assert not ok and ch == f["top_choices"] and nest == f["nested"] and len(path) == f["rows"]


# ---- brute force: the pruned, memoised search = the first match of the plain enumeration ----

def _brute_first(program, ch, blocks, b=0):
    for nest, rows in D._all_resolutions(D._atoms(program, ch, b)):
        cuts = D.cut(len(rows), [v[0] for v in blocks])
        if sum(v[0] for v in blocks) == len(rows) and len(cuts) == len(blocks) and \
                all(A.block10(rows[s:e]) == tuple(blocks[i]) for i, (s, e) in enumerate(cuts)):
            return nest, rows
    return None


@st.composite
def nested_programs(draw):
    def op(i):
        idi = tuple(draw(st.integers(0, 2)) for _ in range(6))
        return Op(idi, ((draw(st.integers(1, 3)), draw(st.integers(1, 3))),), ((i, R),), f"o{i}")
    n = [0]

    def nxt():
        n[0] += 1
        return op(n[0])
    body = [nxt() for _ in range(draw(st.integers(0, 2)))]
    arms = [[nxt() for _ in range(draw(st.integers(0, 2)))] for _ in range(draw(st.integers(2, 3)))]
    body.append(If(arms))
    if draw(st.booleans()):
        body.append(If([[nxt()], []]))
    prog = [nxt(), Loop(body, 1, draw(st.integers(2, 4)))]
    if draw(st.booleans()):
        prog.append(If([[nxt()], [nxt(), nxt()]]))
    return prog


@settings(max_examples=60, deadline=None)
@given(nested_programs(), st.data())
def test_exact_search_equals_brute_force(prog, data):
    tops = list(D.top_choice_vectors(prog))
    ch = data.draw(st.sampled_from(tops))
    res = list(D._all_resolutions(D._atoms(prog, ch, 0)))
    nest, rows = data.draw(st.sampled_from(res))
    L = len(rows)
    k = data.draw(st.integers(1, min(4, L)))
    cuts = sorted(data.draw(st.sets(st.integers(1, L - 1), min_size=k - 1, max_size=k - 1))) if L > 1 else []
    bounds = [0] + cuts + [L]
    blocks = [A.block10(rows[bounds[i]:bounds[i + 1]]) for i in range(len(bounds) - 1)]
    got = D.nested_exact(D._atoms(prog, ch, 0), blocks)
    want = _brute_first(prog, ch, blocks)
    assert want is not None and got is not None
    assert got[0] == want[0] and got[1] == want[1]
    # round trip (T5 analogue): the decoded path reproduces the predicted vectors
    c2 = D.cut(len(got[1]), [v[0] for v in blocks])
    assert [A.block10(got[1][s:e]) for s, e in c2] == blocks


def test_branch_head_skips_nested_sites():
    g, prog = _prog()
    # one free top-level site (the loop, 3 trip logits); the nested If has none
    from workloads import n_branch_logits
    assert n_branch_logits(prog) == 3
    y = np.zeros(10 + 3)
    y[10 + 2] = 1.0
    near = []
    assert D.decode_branch_head(y, prog, 1, near) == [2, -1]


@settings(max_examples=80, deadline=None)
@given(nested_programs(), st.data())
def test_closest_flat_equals_exhaustive_fallback(prog, data):
    """The suffix-set fallback (P:L147 for flat choice points) = the exhaustive enumeration's
    first closest resolution."""
    ch = data.draw(st.sampled_from(list(D.top_choice_vectors(prog))))
    atoms = D._atoms(prog, ch, 0)
    if not D._flat(atoms):
        return
    total = data.draw(st.integers(0, 40))
    best = None
    for nest, rows in D._all_resolutions(atoms):
        d = abs(len(rows) - total)
        if best is None or d < best[0]:
            best = (d, nest, rows)
    assert D.closest_flat(atoms, total) == (best[1], best[2])
