"""Pilot output -> resolved control flow, execution blocks and per-block tensor sets
(§IV-B; readings R4, R6).

Oracle — test infrastructure only (see oracle/__init__.py).

Logit layout (reading R4): [block head: K_max x 10 | branch head: one logit per choice of
every free (untied) control-flow site, sites in preorder | zero padding].
  block head: n = rint(y * 2^sigma) (round half to even), clamped to [0, 2^24-1];
              sigma = 4 for the count and idiom sums, 10 for the dimension sums;
              slot k is empty iff its count n_0 = 0 (P:L143 vector format).
  branch head: choice = argmax (lowest index on ties) over the site's logits; a tied site
              replays the choice of the site it names (reading R6).
Without a branch head the paper's traversal match resolves the path.
"""
from __future__ import annotations

from dataclasses import dataclass, field
import math

import numpy as np

from workloads import Op, If, Loop, R, W
from . import afm as A

NEAR_TIE = 1e-6


@dataclass
class Prediction:
    choices: list
    path: list              # executed rows: Op or None (control)
    groups: list            # [(start_row, end_row)]
    blocks: list            # block10 of every group (the executed block vectors)
    W: list                 # per group: [(tensor_id, mode_union, needs_fetch)]
    slots: list             # raw decoded block head, K_max x 10 ints
    near_ties: list = field(default_factory=list)
    matched: bool = True    # traversal: exact match found
    nested: list = field(default_factory=list)   # nested-site executions' choices (R16)


def decode_block_head(y, K_max, near):
    """Block head -> K_max x 10 integer slot vectors (reading R4)."""
    slots = []
    for k in range(K_max):
        v = []
        for e in range(10):
            sigma = 4 if e < 7 else 10
            t = float(y[10 * k + e]) * (2.0 ** sigma)
            frac = t - math.floor(t)
            if abs(frac - 0.5) < NEAR_TIE:
                near.append(("slot", k, e))
            n = int(np.rint(t))
            v.append(min(max(n, 0), A.SAT))
        slots.append(tuple(v))
    return slots


def decode_branch_head(y, program, K_max, near):
    """Branch head -> choice index for every site in preorder (reading R4, R6)."""
    sl = A.sites(program)
    inner = A.nested_ids(program)
    off = 10 * K_max
    choices = [0] * len(sl)
    for i, s in enumerate(sl):
        if id(s) in inner:
            choices[i] = -1            # R16: resolved per execution by the traversal
            continue
        if s.tie >= 0:
            choices[i] = choices[s.tie]
            continue
        b = A.n_choices(s)
        logits = [float(v) for v in y[off:off + b]]
        best = 0
        for c in range(1, b):
            if logits[c] > logits[best]:
                best = c
        srt = sorted(logits, reverse=True)
        if b > 1 and srt[0] - srt[1] < NEAR_TIE * max(1.0, abs(srt[0])):
            near.append(("site", i))
        choices[i] = best
        off += b
    return choices


def cut(L, counts):
    """Partition rows [0, L) at the cumulative predicted counts (reading R4): group g covers
    [C_g, C_{g+1}) clipped to L; groups starting at or past L are dropped; if the counts sum
    to less than L the last group absorbs the remainder; no non-empty slot -> one group."""
    if not counts or L == 0:
        return [(0, L)] if L > 0 else []
    groups, c = [], 0
    for n in counts:
        if c >= L:
            break
        groups.append((c, min(c + n, L)))
        c += n
    if groups[-1][1] < L:
        groups[-1] = (groups[-1][0], L)
    return groups


def enumerate_paths(program, b=0):
    """All resolved paths in lexicographic order of branch choices (program order; lower
    branch index / lower trip count first). Yields (choices_by_site_index, rows)."""
    sl = A.sites(program)
    index = {id(s): i for i, s in enumerate(sl)}

    def rec(items, pos, choices, k=None):
        # yields (choices, rows) for items[pos:]; k = iteration index of the innermost loop (R13)
        if pos == len(items):
            yield choices, []
            return
        it = items[pos]
        if isinstance(it, Op):
            for ch, rows in rec(items, pos + 1, choices, k):
                yield ch, [A.bind(it, k, b)] + rows
            return
        si = index[id(it)]
        opts = [choices[it.tie]] if it.tie >= 0 else list(range(A.n_choices(it)))
        for c in opts:
            ch0 = dict(choices)
            ch0[si] = c
            if isinstance(it, If):
                body_items = it.branches[c]
                for ch1, brows in rec(body_items, 0, ch0, k):
                    for ch2, rest in rec(items, pos + 1, ch1, k):
                        yield ch2, [None] + brows + rest
            else:
                n = it.lo + c
                yield from _loop_iter(it, n, items, pos, ch0, rec, k)

    def _loop_iter(it, n, items, pos, ch, rec_, k_out):
        def iters(i, chk):
            if i == n:
                yield chk, [None]
                return
            for ch1, brows in rec_(it.body, 0, chk, n - 1 - i if it.rev else i):
                for ch2, rest in iters(i + 1, ch1):
                    yield ch2, [None] + brows + rest
        for ch1, lrows in iters(0, ch):
            for ch2, rest in rec_(items, pos + 1, ch1, k_out):
                yield ch2, lrows + rest

    for ch, rows in rec(program, 0, {}):
        yield [ch.get(i, 0) for i in range(len(sl))], rows


def traversal(program, pred_blocks, b=0):
    """The paper's mapping: find the first path (lexicographic order) whose
    rows, cut at the predicted cumulative counts, give exactly the predicted block vectors;
    otherwise pick the path closest in operator count (first on ties)."""
    total = sum(v[0] for v in pred_blocks)
    best = None
    for choices, rows in enumerate_paths(program, b):
        if len(rows) == total:
            groups = cut(len(rows), [v[0] for v in pred_blocks])
            if len(groups) == len(pred_blocks) and all(
                    A.block10(rows[s:e]) == tuple(pred_blocks[g]) for g, (s, e) in enumerate(groups)):
                return choices, rows, True
        d = abs(len(rows) - total)
        if best is None or d < best[0]:
            best = (d, choices, rows)
    return best[1], best[2], False


# ---- nested sites (reading R16) ---------------------------------------------------------
# A site nested in another site's arm or loop body executes once per execution of its
# enclosure, each time with its own choice, and carries no branch-head logits. With the
# top-level choices fixed, the path is a sequence of rows and choice points (one per nested
# execution, in execution order). The paper's mapping "enumerates and traverses each possible
# branch" whenever a control flow is met: the executions' choices are visited in
# lexicographic order of the execution-ordered choice sequence (lower branch index / trip count
# first); the first path whose cut at the predicted cumulative counts gives exactly the
# predicted vectors wins; otherwise the path with the closest operator count, first in
# the same order.

def _atoms(program, choices, b):
    """The path of fixed top-level `choices` as atoms: ('row', op_or_None) and
    ('choice', [arm_atoms, ...]) for every nested execution; arm c of a nested If is its
    branch c, arm c of a nested Loop is its execution with trip count lo + c."""
    sl = A.sites(program)
    index = {id(s): i for i, s in enumerate(sl)}
    inner = A.nested_ids(program)

    def loop_rows(it, n, k_out):
        out = []
        for i in range(n):
            out.append(("row", None))
            out.extend(rec(it.body, n - 1 - i if it.rev else i))
        out.append(("row", None))
        return out

    def rec(items, k):
        out = []
        for it in items:
            if isinstance(it, Op):
                out.append(("row", A.bind(it, k, b)))
            elif id(it) in inner:
                if it.tie >= 0:
                    raise ValueError("a nested site cannot replay another site (R6, R16)")
                if isinstance(it, If):
                    out.append(("row", None))
                    out.append(("choice", [rec(br, k) for br in it.branches]))
                else:
                    out.append(("choice", [loop_rows(it, it.lo + c, k) for c in range(A.n_choices(it))]))
            else:
                i = index[id(it)]
                c = choices[it.tie if it.tie >= 0 else i]
                if isinstance(it, If):
                    out.append(("row", None))
                    out.extend(rec(it.branches[c], k))
                else:
                    out.extend(loop_rows(it, it.lo + c, k))
        return out
    return rec(program, None)


def _feed(g, acc, row, pred):
    """One row into the running block vector of group g (R4 cut); None when no extension of
    the prefix can match (every element is >= 0, so running sums only grow)."""
    if g >= len(pred):
        return None
    sig = A.row_sig(row)
    acc = (acc[0] + 1,) + tuple(acc[1 + e] + sig[e] for e in range(9))
    p = pred[g]
    sat = tuple(A.sat(x) for x in acc)
    if any(sat[e] > p[e] for e in range(10)):
        return None
    if acc[0] == p[0]:
        if sat != tuple(p):
            return None
        return g + 1, (0,) * 10
    return g, acc


def nested_exact(atoms, pred):
    """First (lexicographic) resolution of the choice points whose rows, cut at the predicted
    cumulative counts, give exactly the predicted vectors: (nested choices, rows) or None.
    Depth-first in execution order; a prefix is abandoned as soon as it cannot match (_feed);
    a failed state (continuation, group, running vector) is remembered - the search from it is
    deterministic - so the search is polynomial on repetitive programs (both are
    result-preserving)."""
    failed = set()
    rows, nested = [], []
    zero = (0,) * 10

    def go(stack, g, acc):
        while stack:
            lst, i = stack[-1]
            if i == len(lst):
                stack = stack[:-1]
                continue
            atom = lst[i]
            stack = stack[:-1] + ((lst, i + 1),)
            if atom[0] == "row":
                r = _feed(g, acc, atom[1], pred)
                if r is None:
                    return False
                g, acc = r
                rows.append(atom[1])
            else:
                key = (tuple((id(l), j) for l, j in stack), g, acc)
                if key in failed:
                    return False
                mr, mn = len(rows), len(nested)
                for c, arm in enumerate(atom[1]):
                    nested.append(c)
                    if go(stack + ((arm, 0),), g, acc):
                        return True
                    del rows[mr:]
                    del nested[mn:]
                failed.add(key)
                return False
        return g == len(pred) and acc == zero

    if go(((atoms, 0),), 0, zero):
        return list(nested), list(rows)
    return None


def _all_resolutions(atoms, cap=200_000):
    """Every resolution of the choice points in lexicographic order: (nested, rows)."""
    count = [0]

    def rec(stack, rows, nest):
        rows = list(rows)
        while stack:
            lst, i = stack[-1]
            if i == len(lst):
                stack = stack[:-1]
                continue
            atom = lst[i]
            stack = stack[:-1] + ((lst, i + 1),)
            if atom[0] == "choice":
                for c, arm in enumerate(atom[1]):
                    yield from rec(stack + ((arm, 0),), rows, nest + [c])
                return
            rows.append(atom[1])
        count[0] += 1
        if count[0] > cap:
            raise RuntimeError("too many resolutions for the exhaustive fallback")
        yield nest, rows
    yield from rec(((atoms, 0),), [], [])


def closest_flat(atoms, total):
    """P:L147's fallback for a path whose choice points are flat (arms hold rows only): the
    first resolution, in lexicographic order, among those whose row count is closest to
    `total`. The row count is the fixed rows plus the chosen arms' lengths, so the reachable
    counts after each choice point are sets (suffix sums); choosing at every point the lowest
    arm from which a closest count stays reachable gives the lexicographically first such
    resolution. (tests/test_oracle_nested.py checks it against the exhaustive enumeration.)"""
    fixed = sum(1 for a in atoms if a[0] == "row")
    points = [[len(arm) for arm in a[1]] for a in atoms if a[0] == "choice"]
    suffix = [set() for _ in range(len(points) + 1)]
    suffix[-1] = {0}
    for i in range(len(points) - 1, -1, -1):
        suffix[i] = {v + l for v in suffix[i + 1] for l in points[i]}
    dbest = min(abs(fixed + v - total) for v in suffix[0])
    targets = {total - dbest, total + dbest}
    nest, used = [], fixed
    for i, lens in enumerate(points):
        for c, l in enumerate(lens):
            if any((t - used - l) in suffix[i + 1] for t in targets):
                nest.append(c)
                used += l
                break
    it = iter(nest)
    rows = []
    for a in atoms:
        if a[0] == "row":
            rows.append(a[1])
        else:
            rows.extend(r[1] for r in a[1][next(it)])
    return nest, rows


def _flat(atoms):
    return all(a[0] == "row" or all(x[0] == "row" for arm in a[1] for x in arm) for a in atoms)


def nested_traversal(program, choices, pred_blocks, b=0):
    """Reading R16 with the top-level choices fixed (branch head): (nested, rows, matched)."""
    atoms = _atoms(program, choices, b)
    pred = [tuple(v) for v in pred_blocks]
    hit = nested_exact(atoms, pred)
    if hit is not None:
        return hit[0], hit[1], True
    total = sum(v[0] for v in pred)
    if _flat(atoms):
        nest, rows = closest_flat(atoms, total)
        return nest, rows, False
    best = None
    for nest, rows in _all_resolutions(atoms):
        d = abs(len(rows) - total)
        if best is None or d < best[0]:
            best = (d, nest, rows)
    return best[1], best[2], False


def top_choice_vectors(program):
    """Top-level choice vectors in lexicographic order (preorder; nested sites -1; a tied site
    replays its target)."""
    sl = A.sites(program)
    inner = A.nested_ids(program)
    free = [i for i, s in enumerate(sl) if id(s) not in inner and s.tie < 0]

    def rec(k, cur):
        if k == len(free):
            v = [-1 if id(s) in inner else 0 for s in sl]
            for i, s in enumerate(sl):
                if id(s) in inner:
                    continue
                v[i] = cur[free.index(s.tie)] if s.tie >= 0 else cur[free.index(i)]
            yield v
            return
        for c in range(A.n_choices(sl[free[k]])):
            yield from rec(k + 1, cur + [c])
    yield from rec(0, [])


def traversal_nested(program, pred_blocks, b=0):
    """Reading R16 without a branch head: top-level vectors in lexicographic order, each with
    its nested executions in lexicographic order; first exact match, else the closest count
    (first in the same order). Returns (choices, nested, rows, matched)."""
    pred = [tuple(v) for v in pred_blocks]
    for ch in top_choice_vectors(program):
        hit = nested_exact(_atoms(program, ch, b), pred)
        if hit is not None:
            return ch, hit[0], hit[1], True
    total = sum(v[0] for v in pred)
    best = None
    for ch in top_choice_vectors(program):
        for nest, rows in _all_resolutions(_atoms(program, ch, b)):
            d = abs(len(rows) - total)
            if best is None or d < best[0]:
                best = (d, ch, nest, rows)
    return best[1], best[2], best[3], False


def tensor_sets(path, groups):
    """W_j (reading R8): tensors accessed by the group's operators, in order of first access
    (row order; within an operator ascending tensor id); mode = union of the group's accesses;
    needs_fetch = the first access reads the tensor."""
    out = []
    for (s, e) in groups:
        order, mode, fetch = [], {}, {}
        for r in path[s:e]:
            if r is None:
                continue
            for t, m in r.acc:
                if t not in mode:
                    order.append(t)
                    mode[t] = m
                    fetch[t] = bool(m & R)
                else:
                    mode[t] |= m
        out.append([(t, mode[t], fetch[t]) for t in order])
    return out


def decode(wl, y, branch_head=True, b=0):
    """Decode prediction b of a batch (b selects its per-sample tensors, reading R13)."""
    near = []
    slots = decode_block_head(y, wl.K_max, near)
    counts_slots = [v for v in slots if v[0] != 0]
    matched = True
    nested = []
    has_nested = bool(A.nested_ids(wl.program))
    if branch_head:
        choices = decode_branch_head(y, wl.program, wl.K_max, near)
        if has_nested:
            nested, path, matched = nested_traversal(wl.program, choices, counts_slots, b)
        else:
            path = A.resolve(wl.program, choices, b)
    elif has_nested:
        choices, nested, path, matched = traversal_nested(wl.program, counts_slots, b)
    else:
        choices, path, matched = traversal(wl.program, counts_slots, b)
    groups = cut(len(path), [v[0] for v in counts_slots])
    blocks = [A.block10(path[s:e]) for s, e in groups]
    return Prediction(choices, path, groups, blocks, tensor_sets(path, groups), slots, near, matched, nested)
