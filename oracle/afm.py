"""Idiom-based representation (§IV-A2) and the block vector (§IV-B).

Oracle — test infrastructure only (see oracle/__init__.py).
"""
from __future__ import annotations

from workloads import Op, If, Loop

SAT = (1 << 24) - 1   # reading R1(iii): counts saturate at 2^24-1 (exact in fp32)
ZERO_ROW = (0,) * 9   # P:L110 "a row full of dummy values (all 0s)"; reading R1(ii)


def sat(x):
    return min(max(int(x), 0), SAT)


def signature(op: Op):
    """Nine-element operator signature: six idiom counts followed by three
    input-dimension elements. Fig. 3: matmul(a:(ar,ac), b:(br,bc)) ->
    [1,0,0,0,1,0, ar+br, ac+bc, 0], i.e. element 6+k = sum over the operator's inputs of
    shape[k] (reading R1(i): axes >= 3 ignored, shorter ranks contribute 0)."""
    idi = [sat(c) for c in op.idioms]
    dims = []
    for k in range(3):
        s = 0
        for shape in op.inputs:
            if len(shape) > k:
                s += int(shape[k])
        dims.append(sat(s))
    return tuple(idi + dims)


def afm(program):
    """Rows of afm_rows() without the control flag."""
    return [sig for _, sig in afm_rows(program)]


def afm_rows(program):
    """Architecture feature matrix: one row per operator in program order;
    operators of every branch included (P:L110 'operators in multiple branches are placed
    into AFM following the program order'); a control statement is an all-zero row at its
    position; a loop body appears once. Rows are (is_control, sig): the flag keeps an
    all-zero-signature operator distinct from a control row (reading R1(ii))."""
    rows = []
    for it in program:
        if isinstance(it, Op):
            rows.append((False, signature(it)))
        elif isinstance(it, If):
            rows.append((True, ZERO_ROW))
            for br in it.branches:
                rows.extend(afm_rows(br))
        elif isinstance(it, Loop):
            rows.append((True, ZERO_ROW))
            rows.extend(afm_rows(it.body))
        else:
            raise TypeError(it)
    return rows


def sites(program):
    """Control-flow sites (If/Loop) in preorder: list of the site objects."""
    out = []
    for it in program:
        if isinstance(it, If):
            out.append(it)
            for br in it.branches:
                out.extend(sites(br))
        elif isinstance(it, Loop):
            out.append(it)
            out.extend(sites(it.body))
    return out


def n_choices(site):
    return len(site.branches) if isinstance(site, If) else site.hi - site.lo + 1


def nested_ids(program):
    """ids of the sites nested inside another site's arm or body (reading R16): such a site
    executes once per execution of its enclosing arm / loop iteration, each time with its own
    choice; only top-level sites carry branch-head logits."""
    out = set()

    def rec(items, inside):
        for it in items:
            if isinstance(it, If):
                if inside:
                    out.add(id(it))
                for br in it.branches:
                    rec(br, True)
            elif isinstance(it, Loop):
                if inside:
                    out.add(id(it))
                rec(it.body, True)
    rec(program, False)
    return out


def bind(op, k, b=0):
    """The operator as executed in iteration k of its innermost enclosing loop by prediction b
    of its batch (reading R13): an access (t, m, stride_k, stride_b) names tensor
    t + stride_k * k + stride_b * b (missing strides are 0); accesses sorted by tensor id (the
    order W_j uses within an operator, reading R8). k = None outside loops (stride_k must be 0)."""
    acc = []
    plain = True
    for a in op.acc:
        t, m = a[0], a[1]
        sk = a[2] if len(a) > 2 else 0
        sb = a[3] if len(a) > 3 else 0
        if sk:
            if k is None:
                raise ValueError("strided access outside a loop")
            t = t + sk * k
        t = t + sb * b
        plain = plain and len(a) == 2
        acc.append((t, m))
    acc.sort()
    if len({t for t, _ in acc}) != len(acc):
        raise ValueError("an operator accesses a tensor twice in one iteration")
    if plain and tuple(acc) == tuple(op.acc):
        return op
    return Op(op.idioms, op.inputs, tuple(acc), op.name)


def resolve(program, choices, b=0, nested=None):
    """Executed row sequence for given site choices (choices[i] = choice index of preorder
    site i; If -> branch index, Loop -> trip count lo + index).

    Each row is (op or None). An executed If contributes one control row followed by the
    chosen branch; a Loop with n iterations contributes n+1 control rows (n continue tests
    plus the exit test, reading R2): [Z, body, Z, body, ..., Z]. b = the prediction's index in
    its batch (per-sample tensors, reading R13). nested: the choices of the nested sites'
    executions in execution order (reading R16; their entries in `choices` are unused)."""
    site_list = sites(program)
    index = {id(s): i for i, s in enumerate(site_list)}
    inner = nested_ids(program)
    it_nested = iter(nested or ())

    def choice_of(s):
        if id(s) in inner:
            return next(it_nested)
        i = index[id(s)]
        if s.tie >= 0:
            i = s.tie
        return choices[i]

    def rec(prog, k):
        out = []
        for it in prog:
            if isinstance(it, Op):
                out.append(bind(it, k, b))
            elif isinstance(it, If):
                out.append(None)
                out.extend(rec(it.branches[choice_of(it)], k))
            else:
                n = it.lo + choice_of(it)
                for i in range(n):
                    out.append(None)
                    out.extend(rec(it.body, n - 1 - i if it.rev else i))
                out.append(None)
        return out

    return rec(program, None)


def row_sig(row):
    return ZERO_ROW if row is None else signature(row)


def block10(rows):
    """Execution-block vector: [number of operators and control flows,
    six idiom sums, three dimension sums] over the block's rows (control rows count 1
    and add zeros). Saturating (reading R1(iii))."""
    v = [len(rows)] + [0] * 9
    for r in rows:
        s = row_sig(r)
        for k in range(9):
            v[1 + k] += s[k]
    return tuple(sat(x) for x in v)


def segments(rows):
    """Reading R3: split the AFM (afm_rows() output) before every control row; each
    control row starts a new segment. Returns a list of signature-row lists."""
    segs, cur = [], []
    for ctrl, r in rows:
        if ctrl and cur:
            segs.append(cur)
            cur = []
        cur.append(r)
    if cur:
        segs.append(cur)
    return segs


def block10_of_sig_rows(sig_rows):
    v = [len(sig_rows)] + [0] * 9
    for s in sig_rows:
        for k in range(9):
            v[1 + k] += s[k]
    return tuple(sat(x) for x in v)
