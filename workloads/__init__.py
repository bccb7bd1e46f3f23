"""Seeded synthetic DyNN traces — the ONLY module shared by oracle/ and the CUDA path.

It holds the *inputs* of the method and none of its arithmetic: the static program
(operators with their idiom counts, input shapes and tensor accesses; If/Loop
control flow), the tensor table, the per-sample input-shape descriptors, the
pilot-model weights, and a counter-based byte-content generator used by the
migration tests (oracle/ implements nothing of it; both sides call it).

No signature, AFM, block vector, feature, logit, decode or plan is computed here.

Program model (§IV-A2):
  Op(idioms[6], inputs=(shape, ...), acc=((tensor_id, mode), ...))
      idioms = counts of [transpose, gather, scatter, reduction, stream, stencil]
      (column order P:L135); acc sorted by tensor id, unique.
  If(branches=[program, ...], tie=-1)   one control-flow statement
  Loop(body=program, lo, hi, tie=-1, rev=False)    trip count in [lo, hi]
  tie >= 0 marks a site that replays the choice of an earlier site (the backward
  pass of a routed layer follows its forward choice) — DESIGN.md reading R6.
  An access may carry a stride: (tensor_id, mode, stride) names tensor
  tensor_id + stride * k, k = iteration index of the innermost enclosing Loop
  (0..n-1; n-1..0 when the Loop has rev=True, a backward pass over a forward loop's
  per-iteration tensors) — DESIGN.md reading R13. Outside loops the stride is 0.
"""
from __future__ import annotations

from dataclasses import dataclass, field
import numpy as np

R, W, RW = 1, 2, 3
CNN, LSTM, TRANSFORMER = 0, 1, 2
MiB = 1 << 20
GiB = 1 << 30


@dataclass
class Op:
    idioms: tuple
    inputs: tuple
    acc: tuple
    name: str = ""


@dataclass
class If:
    branches: list
    tie: int = -1


@dataclass
class Loop:
    body: list
    lo: int
    hi: int
    tie: int = -1
    rev: bool = False


@dataclass
class Tensor:
    nbytes: int
    host_off: int
    transient: bool
    name: str = ""


@dataclass
class PilotSpec:
    """Pilot topology + fp32 weights (row-major W[out][in]).

    feature: list of (in_off, in_len, out) input-feature layers;
             empty list = identity feature stage (tiny T32 topology).
    mlp:     list of (in, out) layer dims shared by the three MLPs.
    out_in:  input width of the output layer; O = number of logits.
    weights: {"feat{i}.W","feat{i}.b","mlp{k}.{l}.W","mlp{k}.{l}.b","out.W","out.b"}
    """
    F: int
    O: int
    feature: list
    mlp: list
    out_in: int
    weights: dict


@dataclass
class Workload:
    name: str
    nn_type: int
    program: list
    tensors: list
    S_max: int
    D_s: int
    h: int
    K_max: int
    budget: int
    align: int
    policy: int          # 0 = PAPER (evict all unused), 1 = RETAIN (Belady prefix cut)
    pilot: PilotSpec
    samples: np.ndarray  # int64 [n_samples, D_s] input-shape descriptors
    hist_ids: np.ndarray  # int32 [h] history group ids (negative = from the end)
    seed: int
    notes: dict = field(default_factory=dict)


# ----------------------------------------------------------------------------
# helpers (input construction only)
# ----------------------------------------------------------------------------

def _op(rng, acc, nin=2, name=""):
    idioms = tuple(int(x) for x in rng.integers(0, 4, size=6))
    inputs = tuple(tuple(int(d) for d in rng.integers(1, 513, size=int(rng.integers(1, 4))))
                   for _ in range(nin))
    acc = tuple(sorted({t: m for t, m in acc}.items()))
    return Op(idioms, inputs, acc, name)


def _linear_init(rng, fan_in, fan_out):
    """He-uniform W ~ U(-sqrt(6/in), sqrt(6/in)) (keeps activations alive through the LeakyReLU
    stack so the random pilot's routing depends on the sample), b ~ U(-0.1, 0.1)."""
    bound = np.sqrt(6.0 / fan_in)
    Wt = rng.uniform(-bound, bound, size=(fan_out, fan_in)).astype(np.float32)
    b = rng.uniform(-0.1, 0.1, size=(fan_out,)).astype(np.float32)
    return Wt, b


def feature_width(S_max, D_s, h):
    """F = [x_t(3) | x_s(D_s) | x_a(10*S_max) | x_h(10*h)] zero-padded to a multiple of 16."""
    n = 3 + D_s + 10 * S_max + 10 * h
    return (n + 15) // 16 * 16


def make_pilot(rng, kind, S_max, D_s, h, K_max, n_branch_logits, planted_counts=None,
               count_scale=16.0, xs_mean=None):
    """Build a pilot with seeded-random weights.

    kind "T32": identity feature stage, MLP F->32->32, output 32->O (north_star config 1).
    kind "P512": three input-feature layers (x_s->32, [x_a;x_h]->32, x_t->32), MLP
                 96->512->512->512->64, output 64->O (width P:L263).
    kind "H<w>": like P512 with hidden width w (width sweep).

    planted_counts: if given, the block-head rows of the output layer get zero weights and
    a bias that encodes these per-slot operator counts in the block-head unit (count/16,
    DESIGN.md reading R4) — a stand-in for a trained pilot's partition labels
    (P:L164-L170), so the synthetic predictions have the workload's group structure.
    The branch-head rows keep random weights: routing depends on the sample.
    """
    F = feature_width(S_max, D_s, h)
    n_out = 10 * K_max + n_branch_logits
    O = (n_out + 7) // 8 * 8
    wts = {}
    if kind == "T32":
        feature = []
        mlp = [(F, 32), (32, 32)]
        out_in = 32
    else:
        width = 512 if kind == "P512" else int(kind[1:])
        xs_off, xs_len = 3, D_s
        xa_off, xa_len = 3 + D_s, 10 * S_max + 10 * h
        feature = [(xs_off, xs_len, 32), (xa_off, xa_len, 32), (0, 3, 32)]
        mlp = [(96, width), (width, width), (width, width), (width, 64)]
        out_in = 64
        for i, (off, ln, o) in enumerate(feature):
            wts[f"feat{i}.W"], wts[f"feat{i}.b"] = _linear_init(rng, ln, o)
    for k in range(3):
        for l, (i, o) in enumerate(mlp):
            wts[f"mlp{k}.{l}.W"], wts[f"mlp{k}.{l}.b"] = _linear_init(rng, i, o)
    # sample sensitivity: the per-arch constant inputs (x_t, x_a) get a gain of 1/16 so that
    # the random branch head routes differently per sample instead of being dominated by them
    if kind == "T32":
        for k in range(3):
            wts[f"mlp{k}.0.W"][:, :3] *= np.float32(1 / 16)
            wts[f"mlp{k}.0.W"][:, 3 + D_s:] *= np.float32(1 / 1024)
    else:
        wts["feat1.W"] *= np.float32(1 / 1024)
        wts["feat2.W"] *= np.float32(1 / 16)
    # centre the descriptor input (what a trained first layer does): b -= W . E[x_s], with
    # E[x_s] the mean descriptor in feature units (descriptor x 2^-10, reading R3)
    if xs_mean is not None:
        mu = np.asarray(xs_mean, np.float64) / 1024.0
        if kind == "T32":
            for k in range(3):
                Wk = wts[f"mlp{k}.0.W"]
                wts[f"mlp{k}.0.b"] = (wts[f"mlp{k}.0.b"] - Wk[:, 3:3 + D_s].astype(np.float64) @ mu).astype(np.float32)
        else:
            wts["feat0.b"] = (wts["feat0.b"] - wts["feat0.W"].astype(np.float64) @ mu).astype(np.float32)
    Wo, bo = _linear_init(rng, out_in, O)
    if planted_counts is not None:
        Wo[: 10 * K_max, :] = 0.0
        bo[: 10 * K_max] = 0.0
        for k, c in enumerate(planted_counts):
            bo[10 * k] = np.float32(c / count_scale)
    Wo[n_out:, :] = 0.0
    bo[n_out:] = 0.0
    wts["out.W"], wts["out.b"] = Wo, bo
    return PilotSpec(F=F, O=O, feature=feature, mlp=mlp, out_in=out_in, weights=wts)


def _host_layout(tensors_bytes, align):
    """Host homes laid out in table order (the generator lists tensors group-major)."""
    offs, cur = [], 0
    for nb in tensors_bytes:
        offs.append(cur)
        cur += (nb + align - 1) // align * align
    return offs, cur


def n_branch_logits(program):
    """Count of free (untied) branch-head logits: structure bookkeeping of the input. Only
    top-level sites carry logits; a site nested in another site's arm or body has none
    (reading R16)."""
    n = 0
    for it in program:
        if isinstance(it, If) and it.tie < 0:
            n += len(it.branches)
        elif isinstance(it, Loop) and it.tie < 0:
            n += it.hi - it.lo + 1
    return n


def _walk(program):
    for it in program:
        yield it
        if isinstance(it, If):
            for br in it.branches:
                yield from _walk(br)
        elif isinstance(it, Loop):
            yield from _walk(it.body)


def actual_choices(wl, sample, zipf_s=1.2):
    """Synthetic 'what actually ran' control flow of a sample (input generation for the
    mis-prediction tests and bench): per free site a choice drawn from a
    Zipf(zipf_s) prior over its choices with a generator seeded by (workload seed, sample);
    tied sites replay their target (reading R6). Deterministic; no method arithmetic."""
    rng = np.random.default_rng((int(wl.seed) * 1_000_003 + int(sample)) & 0x7FFFFFFF)
    sl = [it for it in _walk(wl.program) if isinstance(it, (If, Loop))]
    top = {id(it) for it in wl.program}
    out = []
    for it in sl:
        if id(it) not in top:
            out.append(-1)                 # nested site: per-execution choices (R16), not drawn
            continue
        if it.tie >= 0:
            out.append(out[it.tie])
            continue
        n = len(it.branches) if isinstance(it, If) else it.hi - it.lo + 1
        w = 1.0 / np.arange(1, n + 1) ** zipf_s
        out.append(int(rng.choice(n, p=w / w.sum())))
    return out


# ----------------------------------------------------------------------------
# M0 tiny (BASELINE configs[0])
# ----------------------------------------------------------------------------

def make_tiny(seed=0, n_samples=16, planted=True, branch_head=True):
    """8 groups, 64 tensors, T32 pilot (hidden 32), 1 GiB budget.

    Program: LSTM type; If A (2 branches), If B (2 branches), Loop C (1..3 x 4-op body)
    -> 12 paths of 35..49 rows. 64 tensors of U{1..31} MiB: 38 weights (R) and 26
    activations (written once, then read; transient). Each op touches 1-2 tensors.
    Feasibility by construction: a group has <= 7 rows (8 planted slots of 6 rows, the
    last absorbs <= 1 extra row) x 2 accesses x 31 MiB = 434 MiB < H = 512 MiB.
    """
    rng = np.random.default_rng(seed)
    T = 64
    n_w = 38
    sizes = [int(rng.integers(1, 32)) * MiB for _ in range(T)]
    weights = list(range(n_w))
    acts = list(range(n_w, T))
    act_cursor = [0]

    def op():
        k = int(rng.integers(1, 3))
        acc = []
        for _ in range(k):
            if rng.random() < 0.6 or not acts:
                acc.append((int(rng.choice(weights)), R))
            else:
                a = acts[int(rng.integers(0, len(acts)))]
                acc.append((a, W if rng.random() < 0.5 else R))
        return _op(rng, acc)

    def block(n):
        return [op() for _ in range(n)]

    program = (block(8)
               + [If([block(4), block(6)])]
               + block(6)
               + [If([block(3), block(5)])]
               + block(4)
               + [Loop(block(4), 1, 3)]
               + block(2))
    offs, _ = _host_layout(sizes, 256)
    tensors = [Tensor(sizes[t], offs[t], t >= n_w, f"t{t}") for t in range(T)]
    S_max, D_s, h, K_max = 4, 8, 0, 8
    nbl = n_branch_logits(program) if branch_head else 0
    samples = rng.integers(1, 4096, size=(n_samples, D_s)).astype(np.int64)
    pilot = make_pilot(rng, "T32", S_max, D_s, h, K_max, nbl,
                       planted_counts=[6] * 8 if planted else None, xs_mean=[2048.0] * D_s)
    return Workload("tiny", LSTM, program, tensors, S_max, D_s, h, K_max,
                    budget=GiB, align=256, policy=1, pilot=pilot, samples=samples,
                    hist_ids=np.zeros(0, np.int32), seed=seed,
                    notes={"branch_head": branch_head})


# ----------------------------------------------------------------------------
# M1 switch-MoE (BASELINE configs[1])
# ----------------------------------------------------------------------------

def make_moe(seed=0, n_samples=16, layers=24, experts=16, layers_per_group=3,
             pilot_kind="P512", budget=3 * GiB, expert_mib=32, act_mib=16):
    """Switch-MoE top-1 (sample-level) routing, 16 experts, expert tensors offloaded.

    Per layer, forward: 4 static attention ops (dense weights resident, not managed),
    then If(16 experts): expert e = 2 ops reading W_in[l,e], W_out[l,e] (32 MiB each,
    d_model 2048 x d_ff 8192 bf16) and writing act[l] (16 MiB, transient).
    Backward (reverse layer order): If(tie = forward site of l): 3 ops reading W_out, W_in,
    act[l] and writing grad_out[l,e], grad_in[l,e] (32 MiB each; live -> written back
    for a host-side optimizer), then 4 static attention-backward ops.
    Groups: 3 layers per group -> 8 forward (21 rows) + 8 backward (24 rows) = K_max 16.
    Host pool: experts 24 GiB + gradients 24 GiB; budget 3 GiB -> 8x oversubscription
    of the expert pool.
    """
    rng = np.random.default_rng(seed)
    L, E = layers, experts
    tensors = []

    def add(nb, transient, name):
        tensors.append([nb, transient, name])
        return len(tensors) - 1

    # host layout is table order: expert weights layer-major with W_in/W_out adjacent
    w_in, w_out, g_in, g_out, act = {}, {}, {}, {}, {}
    for l in range(L):
        for e in range(E):
            w_in[l, e] = add(expert_mib * MiB, False, f"w_in[{l},{e}]")
            w_out[l, e] = add(expert_mib * MiB, False, f"w_out[{l},{e}]")
    for l in range(L):
        for e in range(E):
            g_in[l, e] = add(expert_mib * MiB, False, f"g_in[{l},{e}]")
            g_out[l, e] = add(expert_mib * MiB, False, f"g_out[{l},{e}]")
    for l in range(L):
        act[l] = add(act_mib * MiB, True, f"act[{l}]")

    d_model, d_ff, seq = 2048, 8192, 2048

    def attn_ops(bwd=False):
        # layernorm, qkv projection, attention, output projection (shapes of the layer)
        shp = [((seq, d_model),), ((seq, d_model), (d_model, 3 * d_model)),
               ((seq, d_model), (seq, d_model), (seq, d_model)), ((seq, d_model), (d_model, d_model))]
        idi = [(0, 0, 0, 2, 3, 0), (1, 0, 0, 1, 1, 0), (2, 1, 0, 2, 2, 0), (1, 0, 0, 1, 1, 0)]
        if bwd:
            idi = [tuple(x + (1 if i in (0, 4) else 0) for i, x in enumerate(v)) for v in idi][::-1]
            shp = shp[::-1]
        return [Op(idi[i], shp[i], (), "attn_bwd" if bwd else "attn") for i in range(4)]

    program, fwd_site = [], {}
    site = 0
    for l in range(L):
        program += attn_ops()
        branches = []
        for e in range(E):
            branches.append([
                Op((0, 0, 0, 1, 1, 0), ((seq, d_model), (d_model, d_ff)), ((w_in[l, e], R),), "ffn_in"),
                Op((0, 0, 0, 1, 1, 0), ((seq, d_ff), (d_ff, d_model)),
                   tuple(sorted([(w_out[l, e], R), (act[l], W)])), "ffn_out"),
            ])
        program.append(If(branches))
        fwd_site[l] = site
        site += 1
    for l in reversed(range(L)):
        branches = []
        for e in range(E):
            branches.append([
                Op((1, 0, 0, 1, 1, 0), ((seq, d_model), (d_ff, d_model)),
                   tuple(sorted([(w_out[l, e], R), (g_out[l, e], W)])), "ffn_out_bwd"),
                Op((1, 0, 0, 1, 1, 0), ((seq, d_ff), (d_model, d_ff)),
                   tuple(sorted([(w_in[l, e], R), (g_in[l, e], W)])), "ffn_in_bwd"),
                Op((0, 0, 0, 1, 2, 0), ((seq, d_model),), ((act[l], R),), "act_bwd"),
            ])
        program.append(If(branches, tie=fwd_site[l]))
        site += 1
        program += attn_ops(bwd=True)

    sizes = [t[0] for t in tensors]
    offs, _ = _host_layout(sizes, 256)
    tens = [Tensor(t[0], offs[i], t[1], t[2]) for i, t in enumerate(tensors)]
    S_max, D_s, h = 16, 16, 2
    K_max = 2 * L // layers_per_group
    fwd_rows = layers_per_group * (4 + 1 + 2)
    bwd_rows = layers_per_group * (1 + 3 + 4)
    planted = [fwd_rows] * (L // layers_per_group) + [bwd_rows] * (L // layers_per_group)
    samples = np.stack([
        rng.integers(128, 2049, size=n_samples),         # sequence length
        rng.integers(1, 65, size=n_samples),             # sentences / documents
    ] + [rng.integers(1, 4096, size=n_samples) for _ in range(D_s - 2)], axis=1).astype(np.int64)
    pilot = make_pilot(rng, pilot_kind, S_max, D_s, h, K_max, n_branch_logits(program),
                       planted_counts=planted, xs_mean=[1088.0, 32.5] + [2048.0] * (D_s - 2))
    return Workload("moe", TRANSFORMER, program, tens, S_max, D_s, h, K_max,
                    budget=budget, align=256, policy=1, pilot=pilot, samples=samples,
                    hist_ids=np.array([-2, -1], np.int32), seed=seed,
                    notes={"experts": E, "layers": L, "expert_bytes": 2 * expert_mib * MiB})


# ----------------------------------------------------------------------------
# M2 AlphaFold-Evoformer-shaped (BASELINE configs[2])
# ----------------------------------------------------------------------------

def make_af(seed=0, n_samples=16, blocks=48, max_recycle=4, budget=2 * GiB,
            pilot_kind="P512", rows_per_block=16, acts_per_block=10, act_mib=16,
            weight_mib=11):
    """Evoformer-shaped trace: Loop(recycle 1..4) over 48 forward blocks, then 48 backward
    blocks (with the per-block optimizer update fused in), then one final group.

    MSA N_seq 128 x N_res 256, c_m 256, c_z 128, bf16: 10 saved activations of 16 MiB per
    block (written in every recycle; only the last recycle's survive to the backward pass),
    running MSA/pair state (RW), per-block weights 11 MiB + Adam state 22 MiB (RW in backward),
    per-block weight gradient 11 MiB. Every group is 16 rows (the loop-test row rides with
    the first block of an iteration), so planted counts [17, 16 x 47] x 5 + [16] decode to
    one group per block per direction for every recycle count (reading R4).
    """
    rng = np.random.default_rng(seed)
    tensors = []

    def add(nb, transient, name):
        tensors.append([nb, transient, name])
        return len(tensors) - 1

    n_seq, n_res, c_m, c_z = 128, 256, 256, 128
    msa_state = add(n_seq * n_res * c_m * 2, False, "msa_state")
    pair_state = add(n_res * n_res * c_z * 2, False, "pair_state")
    msa_grad = add(n_seq * n_res * c_m * 2, True, "msa_grad")
    pair_grad = add(n_res * n_res * c_z * 2, True, "pair_grad")
    wts, adam, wgrad, acts = {}, {}, {}, {}
    for b in range(blocks):
        wts[b] = add(weight_mib * MiB, False, f"w[{b}]")
        adam[b] = add(2 * weight_mib * MiB, False, f"adam[{b}]")
    for b in range(blocks):
        for a in range(acts_per_block):
            acts[b, a] = add(act_mib * MiB, True, f"act[{b},{a}]")
    for b in range(blocks):
        wgrad[b] = add(weight_mib * MiB, True, f"wgrad[{b}]")
    final_t = add(1 * MiB, False, "loss_scale")

    msa_shape = (n_seq, n_res, c_m)
    pair_shape = (n_res, n_res, c_z)
    n = rows_per_block

    def fwd_block(b):
        ops = []
        for i in range(n):
            acc = []
            if i == 0:
                acc += [(wts[b], R), (msa_state, RW)]
            if i == 1:
                acc += [(pair_state, RW)]
            if 2 <= i < 2 + acts_per_block:
                acc += [(acts[b, i - 2], W)]
            idi = (int(i % 3 == 0), int(i % 5 == 1), 0, 1 + i % 2, 2, int(i % 4 == 3))
            ops.append(Op(idi, (msa_shape, pair_shape) if i % 2 else (msa_shape,), tuple(sorted(acc)), f"evo{b}.{i}"))
        return ops

    def bwd_block(b):
        ops = []
        for i in range(n):
            acc = []
            if i < acts_per_block:
                acc += [(acts[b, acts_per_block - 1 - i], R)]
            if i == 0:
                acc += [(msa_grad, RW), (pair_grad, RW)]
            if i == acts_per_block:
                acc += [(wts[b], R), (wgrad[b], W)]
            if i == n - 1:
                acc += [(wts[b], RW), (adam[b], RW), (wgrad[b], R)]
            idi = (int(i % 3 == 1), 0, int(i % 5 == 0), 2, 2 + i % 2, 0)
            ops.append(Op(idi, (pair_shape, msa_shape) if i % 2 else (pair_shape,), tuple(sorted(acc)), f"evo_bwd{b}.{i}"))
        return ops

    body = []
    for b in range(blocks):
        body += fwd_block(b)
    program = [Loop(body, 1, max_recycle)]
    for b in reversed(range(blocks)):
        program += bwd_block(b)
    program += [Op((0, 0, 0, 1, 1, 0), ((1,),), ((final_t, RW),), "final")] + \
               [Op((0, 0, 0, 0, 1, 0), ((1,),), (), "final")] * (n - 1)

    sizes = [t[0] for t in tensors]
    offs, _ = _host_layout(sizes, 256)
    tens = [Tensor(t[0], offs[i], t[1], t[2]) for i, t in enumerate(tensors)]
    S_max, D_s, h = 16, 16, 2
    K_max = 256
    planted = ([n + 1] + [n] * (blocks - 1)) * (max_recycle + 1) + [n]
    samples = np.stack([
        np.full(n_samples, n_seq), np.full(n_samples, n_res),
        rng.integers(1, 5, size=n_samples),             # sampled recycle count descriptor
    ] + [rng.integers(1, 4096, size=n_samples) for _ in range(D_s - 3)], axis=1).astype(np.int64)
    pilot = make_pilot(rng, pilot_kind, S_max, D_s, h, K_max, n_branch_logits(program),
                       planted_counts=planted, xs_mean=[n_seq, n_res, 2.5] + [2048.0] * (D_s - 3))
    return Workload("af", TRANSFORMER, program, tens, S_max, D_s, h, K_max,
                    budget=budget, align=256, policy=1, pilot=pilot, samples=samples,
                    hist_ids=np.array([-2, -1], np.int32), seed=seed,
                    notes={"blocks": blocks, "max_recycle": max_recycle})


# ----------------------------------------------------------------------------
# M3 variable-length sequence LSTM (BASELINE configs[3])
# ----------------------------------------------------------------------------

def make_lstm(seed=0, n_samples=128, batch=64, max_len=512, min_len=16, hidden=512, tasks=4,
              budget=48 * MiB, pilot_kind="P512", K_max=16):
    """Variable-length 2-layer LSTM with a per-sample task head: the "variable-length sequence"
    variant of configs[3] (many small per-timestep tensors, batch-64 pilot predictions, one plan
    over the batch's group sequences concatenated in sample order).

    Per sample (one training example; DyNN with per-sample structure):
      embed op; Loop F (trip n = sequence length in [16, 512]) of two LSTM cells per timestep:
        cell1 reads x[k], h1[k], c1[k], W1 and writes h1[k+1], c1[k+1], g1[k] (saved gates);
        cell2 reads h1[k+1], h2[k], c2[k], W2 and writes h2[k+1], c2[k+1], g2[k]; pool RW;
      If(task head, 4 arms: different op mixes and head weights Wh[a]) + loss;
      If(tie = head) head backward (writes gWh[a]);
      Loop B (tie = F, reversed: k = n-1..0) of two backward cells reading the saved
        g*[k], h*[k], c*[k+1] and x[k], accumulating gW1 / gW2 (RW);
      optimizer op (W1, W2, Wh RW with their gradients).
    Per-iteration / per-sample tensors use strided accesses (reading R13): x[b, k] is row k of
    minibatch sample b's input sequence (its own host home), h/c/g[k] are per-timestep
    transients shared by the batch's samples (each sample's die with its backward pass).
    Sizes: hidden 512 fp32 h/c/x = 2 KiB, bf16 gates 4 x 512 = 4 KiB, W1/W2 = 4 x 512 x 1024
    bf16 = 4 MiB, Wh 1 MiB: 32,768 input rows + 3,079 per-timestep transients + 16
    weight/gradient/state tensors (T = 35,863).
    Budget 48 MiB (H = 24 MiB): a backward group holds W1, W2, gW1, gW2 (16 MiB) plus its
    timesteps; saved activations of long sequences overflow and migrate in 2-4 KiB pieces.
    """
    rng = np.random.default_rng(seed)
    tensors = []

    def add(nb, transient, name):
        tensors.append([nb, transient, name])
        return len(tensors) - 1

    hb, gb = hidden * 4, 4 * hidden * 2
    W1 = add(4 * hidden * 2 * hidden * 2, False, "W1")
    W2 = add(4 * hidden * 2 * hidden * 2, False, "W2")
    gW1 = add(4 * hidden * 2 * hidden * 2, False, "gW1")
    gW2 = add(4 * hidden * 2 * hidden * 2, False, "gW2")
    Wh = [add(hidden * 2048, False, f"Wh[{a}]") for a in range(tasks)]
    gWh = [add(hidden * 2048, False, f"gWh[{a}]") for a in range(tasks)]
    pool = add(hb, True, "pool")
    dpool = add(hb, True, "dpool")
    dh = add(2 * hb, True, "dh_dc")
    loss = add(256, True, "loss")
    x0 = len(tensors)
    for b in range(batch):
        for k in range(max_len):
            add(hb, False, f"x[{b},{k}]")
    h1 = len(tensors)
    for k in range(max_len + 1):
        add(hb, True, f"h1[{k}]")
    c1 = len(tensors)
    for k in range(max_len + 1):
        add(hb, True, f"c1[{k}]")
    g1 = len(tensors)
    for k in range(max_len):
        add(gb, True, f"g1[{k}]")
    h2 = len(tensors)
    for k in range(max_len + 1):
        add(hb, True, f"h2[{k}]")
    c2 = len(tensors)
    for k in range(max_len + 1):
        add(hb, True, f"c2[{k}]")
    g2 = len(tensors)
    for k in range(max_len):
        add(gb, True, f"g2[{k}]")

    Hd = hidden
    cell = (0, 0, 0, 2, 6, 0)          # 2 matmul reductions, gate elementwise streams
    cell_bwd = (1, 0, 0, 3, 8, 0)

    def acc(*a):
        return tuple(sorted(a, key=lambda e: e[0]))

    fwd_body = [
        Op(cell, ((1, Hd), (Hd, 4 * Hd), (1, Hd)),
           acc((W1, R, 0), (x0, R, 1, max_len), (h1, R, 1), (c1, R, 1), (h1 + 1, W, 1), (c1 + 1, W, 1), (g1, W, 1)), "cell1"),
        Op(cell, ((1, Hd), (Hd, 4 * Hd), (1, Hd), (1, Hd)),
           acc((W2, R, 0), (pool, RW, 0), (h1 + 1, R, 1), (h2, R, 1), (c2, R, 1), (h2 + 1, W, 1), (c2 + 1, W, 1),
               (g2, W, 1)), "cell2"),
    ]
    bwd_body = [
        Op(cell_bwd, ((1, Hd), (4 * Hd, Hd), (1, 4 * Hd)),
           acc((W2, R, 0), (gW2, RW, 0), (dh, RW, 0), (g2, R, 1), (h2, R, 1), (c2 + 1, R, 1), (h1 + 1, R, 1)),
           "cell2_bwd"),
        Op(cell_bwd, ((1, Hd), (4 * Hd, Hd), (1, 4 * Hd), (1, Hd)),
           acc((W1, R, 0), (gW1, RW, 0), (dh, RW, 0), (g1, R, 1), (h1, R, 1), (c1 + 1, R, 1), (x0, R, 1, max_len)),
           "cell1_bwd"),
    ]
    head_arms, head_bwd_arms = [], []
    for a in range(tasks):
        na = 1 + a % 3
        head_arms.append([Op((a % 2, 0, a % 2, 1, 1 + a, 0), ((1, Hd), (Hd, 256 * (a + 1))),
                             acc((Wh[a], R, 0), (pool, R, 0)) if i == 0 else acc((loss, W if i == na - 1 else RW, 0)),
                             f"head{a}.{i}") for i in range(na)])
        head_bwd_arms.append([Op((1, 0, a % 2, 1, 2 + a, 0), ((1, Hd), (256 * (a + 1), Hd)),
                                 acc((Wh[a], R, 0), (gWh[a], W, 0), (dpool, W, 0), (loss, R, 0)), f"head_bwd{a}")])
    program = [Op((0, 1, 0, 0, 1, 0), ((max_len, Hd),), (), "embed"),
               Loop(fwd_body, min_len, max_len),
               If(head_arms),
               If(head_bwd_arms, tie=1),
               Op((0, 0, 0, 1, 1, 0), ((1, Hd),), acc((dpool, R, 0), (dh, W, 0)), "pool_bwd"),
               Loop(bwd_body, min_len, max_len, tie=0, rev=True),
               Op((0, 0, 0, 0, 3, 0), ((4 * Hd, 2 * Hd),) * 2,
                  acc((W1, RW, 0), (W2, RW, 0), (gW1, RW, 0), (gW2, RW, 0)), "optimizer")]
    sizes = [t[0] for t in tensors]
    offs, _ = _host_layout(sizes, 256)
    tens = [Tensor(t[0], offs[i], t[1], t[2]) for i, t in enumerate(tensors)]
    S_max, D_s, h = 16, 16, 2
    lens = rng.integers(min_len, max_len + 1, size=n_samples)
    task = rng.integers(0, tasks, size=n_samples)
    samples = np.stack([lens, task] + [rng.integers(1, 4096, size=n_samples) for _ in range(D_s - 2)],
                       axis=1).astype(np.int64)
    nbl = n_branch_logits(program)
    pilot = make_pilot(rng, pilot_kind, S_max, D_s, h, K_max, nbl, planted_counts=None,
                       xs_mean=[(min_len + max_len) / 2, (tasks - 1) / 2] + [2048.0] * (D_s - 2))
    _plant_lstm_heads(pilot, K_max, min_len, max_len, tasks,
                      rows_per_step=2 + len(fwd_body) + len(bwd_body),
                      rows_const=1 + 2 + 3 + 2 + 1 + 1)
    return Workload("lstm", LSTM, program, tens, S_max, D_s, h, K_max,
                    budget=budget, align=256, policy=1, pilot=pilot, samples=samples,
                    hist_ids=np.array([-2, -1], np.int32), seed=seed,
                    notes={"batch": batch, "max_len": max_len, "tasks": tasks,
                           "oracle_batch": 4})   # bench.py's bounded CPU-oracle sample


def _plant_lstm_heads(pilot, K_max, min_len, max_len, tasks, rows_per_step, rows_const):
    """Stand-in for a trained pilot on the var-LSTM trace: two pass-through units
    carry the descriptors n = x_s[0] and task = x_s[1] (in feature units, desc x 2^-10, R3)
    unchanged through every layer (weight 1 on the previous unit, bias 0; LeakyReLU is the
    identity on positive inputs), and the heads read only them, with power-of-two-exact weights:
      trip-count logits  l_t = (2 t n - t^2) / 2048       -> argmax t = n (gap 1/2048),
      task logits        l_a = (2 a task - a^2) / 8       -> argmax a = task (gap 1/8),
      block counts       16 y_k = (rows_const + rows_per_step n) / K_max + 1/32 for every slot,
    so the groups scale with the sequence (the cut's last group absorbs the rounding rest) and
    no rint lands on a half. Every other weight stays seeded-random (the layers remain dense)."""
    w = pilot.weights
    f0 = w["feat0.W"]
    f0[0, :] = 0.0; f0[1, :] = 0.0
    f0[0, 0] = 1.0; f0[1, 1] = 1.0
    w["feat0.b"][:2] = 0.0
    for k in range(3):
        for l in range(len(pilot.mlp)):
            Wl = w[f"mlp{k}.{l}.W"]
            Wl[0, :] = 0.0; Wl[1, :] = 0.0
            Wl[0, 0] = 1.0; Wl[1, 1] = 1.0
            w[f"mlp{k}.{l}.b"][:2] = 0.0
    Wo, bo = w["out.W"], w["out.b"]
    Wo[: 10 * K_max, :] = 0.0
    bo[: 10 * K_max] = 0.0
    for k in range(K_max):
        # 16 y = 1024 * Wo * (n / 1024) + 16 b  ->  Wo = rows_per_step / (16 K_max) * 1024 / 1024
        Wo[10 * k, 0] = np.float32(rows_per_step / (16.0 * K_max) * 1024.0)
        bo[10 * k] = np.float32((rows_const / K_max + 1.0 / 32.0) / 16.0)
    off = 10 * K_max
    for t in range(min_len, max_len + 1):          # Loop F trip-count logits
        Wo[off, :] = 0.0
        Wo[off, 0] = np.float32(t)
        bo[off] = np.float32(-t * t / 2048.0)
        off += 1
    for a in range(tasks):                          # task-head logits
        Wo[off, :] = 0.0
        Wo[off, 1] = np.float32(2 * a * 1024 / 8.0)
        bo[off] = np.float32(-a * a / 8.0)
        off += 1


def _random_tree_postorder(rng, n):
    """Post-order node types (0 leaf, 1 internal) of a random binary tree with n leaves
    (uniform random split of the leaf span at every internal node)."""
    out = []

    def rec(m):
        if m == 1:
            out.append(0)
            return
        left = int(rng.integers(1, m))
        rec(left)
        rec(m - left)
        out.append(1)
    rec(n)
    return out


def make_tree(seed=0, n_samples=128, batch=64, min_leaves=8, max_leaves=64, hidden=512,
              budget=256 * MiB, pilot_kind="P512", K_max=16, fwd_groups=8):
    """Tree-LSTM over binary parse trees: configs[3]'s primary variant (survey §8(d) M3).

    Per sample: embed; Loop F over the tree's nodes in post-order (trip 2n-1 in [15, 127] for
    n leaves in U{8..64}) whose body is ONE If selecting the node type - a site nested in the
    loop, so every node takes its own choice (reading R16): leaf (one cell op reading the
    word's input x[b,k]) or internal (compose + norm ops reading the states of nodes k-1 and
    k-2: the right child of a post-order node is k-1; the left child is approximated by k-2,
    since child indices of an arbitrary parse tree are not a linear stride, R13); loss; Loop B
    (tied to F, reversed) of a uniform node-backward op accumulating the weight gradients;
    optimizer. Per-(sample, node) tensors use strided accesses (R13): h/c (2 KiB), saved
    gates g (4 KiB, transient), input x (2 KiB); two leading pad slots keep k-2 in range.
    The pilot is planted (a stand-in for a trained pilot): pass-through units
    carry the descriptors N = 2n-1, the per-group leaf / internal counts of 8 forward groups
    (even node split) and the node counts of 8 backward groups through every layer, and the
    block head is the exact linear function of them - so the decode meets an exact match, and
    the traversal orders each group's leaves before its internal nodes (the lexicographically
    first resolution; order inside a block is not predicted). The trip-count logits
    (2tN - t^2)/2048 put the argmax at t = N."""
    rng = np.random.default_rng(seed)
    tensors = []

    def add(nb, transient, name):
        tensors.append([nb, transient, name])
        return len(tensors) - 1

    hb, gb = hidden * 4, 4 * hidden * 2
    W_leaf = add(4 * hidden * hidden * 2, False, "W_leaf")
    W_comp = add(5 * 2 * hidden * hidden * 2, False, "W_comp")
    gW_leaf = add(4 * hidden * hidden * 2, False, "gW_leaf")
    gW_comp = add(5 * 2 * hidden * hidden * 2, False, "gW_comp")
    pool = add(hb, True, "pool")
    dpool = add(hb, True, "dpool")
    loss = add(256, True, "loss")
    max_nodes = 2 * max_leaves - 1
    S = max_nodes + 2                                   # per-sample slots: 2 pads + nodes
    h0 = len(tensors)
    for b in range(batch):
        for k in range(S):
            add(hb, True, f"h[{b},{k - 2}]")
    c0 = len(tensors)
    for b in range(batch):
        for k in range(S):
            add(hb, True, f"c[{b},{k - 2}]")
    g0 = len(tensors)
    for b in range(batch):
        for k in range(S):
            add(gb, True, f"g[{b},{k - 2}]")
    x0 = len(tensors)
    for b in range(batch):
        for k in range(S):
            add(hb, False, f"x[{b},{k - 2}]")

    def acc(*a):
        return tuple(sorted(a, key=lambda e: e[0]))

    Hd = hidden
    leaf_sig = (0, 1, 0, 2, 4, 0)
    comp_sig = (1, 0, 0, 3, 6, 0)
    norm_sig = (0, 0, 1, 1, 2, 1)
    bwd_sig = (1, 0, 0, 4, 8, 0)

    def node(base, d):                                  # (tensor, mode, stride_k, stride_b) of slot k + d
        return (base + 2 + d, None, 1, S)

    def A_(base, d, m):
        t, _, sk, sbb = node(base, d)
        return (t, m, sk, sbb)

    leaf_arm = [Op(leaf_sig, ((1, Hd), (Hd, 4 * Hd)),
                   acc((W_leaf, R, 0, 0), (pool, RW, 0, 0), A_(h0, 0, W), A_(c0, 0, W), A_(g0, 0, W), A_(x0, 0, R)),
                   "leaf")]
    int_arm = [Op(comp_sig, ((1, 2 * Hd), (2 * Hd, 5 * Hd)),
                  acc((W_comp, R, 0, 0), A_(h0, -2, R), A_(h0, -1, R), A_(h0, 0, W), A_(c0, -2, R), A_(c0, -1, R),
                      A_(c0, 0, W), A_(g0, 0, W)), "compose"),
               Op(norm_sig, ((1, Hd),), acc((pool, RW, 0, 0), A_(h0, 0, RW), A_(g0, 0, RW)), "norm")]
    bwd_body = [Op(bwd_sig, ((1, Hd), (Hd, 5 * Hd)),
                   acc((W_leaf, R, 0, 0), (W_comp, R, 0, 0), (gW_leaf, RW, 0, 0), (gW_comp, RW, 0, 0),
                       (dpool, R, 0, 0), A_(h0, 0, R), A_(c0, 0, R), A_(g0, 0, R), A_(x0, 0, R)), "node_bwd")]
    embed = Op((0, 1, 0, 0, 1, 0), ((max_nodes, Hd),), acc((pool, W, 0, 0)), "embed")     # resets the pooled state
    loss_op = Op((0, 0, 0, 1, 2, 0), ((1, Hd),), acc((pool, R, 0, 0), (loss, W, 0, 0), (dpool, W, 0, 0)), "loss")
    opt = Op((0, 0, 0, 0, 3, 0), ((4 * Hd, 2 * Hd),) * 2,
             acc((W_leaf, RW, 0, 0), (W_comp, RW, 0, 0), (gW_leaf, RW, 0, 0), (gW_comp, RW, 0, 0)), "optimizer")
    lo, hi = 2 * min_leaves - 1, max_nodes
    program = [embed,
               Loop([If([leaf_arm, int_arm])], lo, hi),
               loss_op,
               Loop(bwd_body, lo, hi, tie=0, rev=True),
               opt]
    sizes = [t[0] for t in tensors]
    offs, _ = _host_layout(sizes, 256)
    tens = [Tensor(t[0], offs[i], t[1], t[2]) for i, t in enumerate(tensors)]
    # samples: trees, descriptors [N, leaves per forward group, internals per forward group,
    # nodes per backward group]
    bg = K_max - fwd_groups
    D_s = 1 + 2 * fwd_groups + bg
    trees, rows = [], []
    for _ in range(n_samples):
        n = int(rng.integers(min_leaves, max_leaves + 1))
        ty = _random_tree_postorder(rng, n)
        N = len(ty)
        fw = [(g * N // fwd_groups, (g + 1) * N // fwd_groups) for g in range(fwd_groups)]
        leaves = [sum(1 for k in range(a, b) if ty[k] == 0) for a, b in fw]
        ints = [(b - a) - l for (a, b), l in zip(fw, leaves)]
        bw = [((g + 1) * N // bg) - (g * N // bg) for g in range(bg)]
        trees.append(ty)
        rows.append([N] + leaves + ints + bw)
    samples = np.asarray(rows, np.int64)
    S_max, h = 16, 2
    program_sites = n_branch_logits(program)
    pilot = make_pilot(rng, pilot_kind, S_max, D_s, h, K_max, program_sites,
                       xs_mean=[float(v) for v in samples.mean(axis=0)])
    _plant_tree_heads(pilot, K_max, fwd_groups, lo, hi, D_s,
                      {"embed": embed, "leaf": leaf_arm, "int": int_arm, "loss": loss_op, "bwd": bwd_body, "opt": opt})
    return Workload("tree", LSTM, program, tens, S_max, D_s, h, K_max,
                    budget=budget, align=256, policy=1, pilot=pilot, samples=samples,
                    hist_ids=np.array([-2, -1], np.int32), seed=seed,
                    notes={"batch": batch, "trees": trees, "fwd_groups": fwd_groups, "oracle_batch": 2})


def _sig9(op):
    """Operator signature bookkeeping for the planted head (Fig. 3 form: idioms ++ dimension
    sums of the inputs) - input construction of the stand-in pilot, recomputed by neither side."""
    dims = [sum(s[k] for s in op.inputs if len(s) > k) for k in range(3)]
    return list(op.idioms) + dims


def _plant_tree_heads(pilot, K_max, fwd_groups, lo, hi, D_s, ops):
    """Pass-through units 0..D_s-1 carry the descriptors (feature units desc x 2^-10) through
    every layer; the block head of slot g is the exact linear function of them (coefficients
    x 2^(10 - sigma), R4 scaling) and the trip logits (2tN - t^2)/2048 (see make_tree)."""
    w = pilot.weights
    f0 = w["feat0.W"]
    for i in range(D_s):
        f0[i, :] = 0.0
        f0[i, i] = 1.0
        w["feat0.b"][i] = 0.0
    for k in range(3):
        for l in range(len(pilot.mlp)):
            Wl = w[f"mlp{k}.{l}.W"]
            for i in range(D_s):
                Wl[i, :] = 0.0
                Wl[i, i] = 1.0
                w[f"mlp{k}.{l}.b"][i] = 0.0
    Wo, bo = w["out.W"], w["out.b"]
    Wo[: 10 * K_max, :] = 0.0
    bo[: 10 * K_max] = 0.0
    sg = {k: [_sig9(o) for o in v] if isinstance(v, list) else _sig9(v) for k, v in ops.items()}
    leaf_v = [3] + sg["leaf"][0]                     # Z (loop test) + Z (If) + the leaf op
    int_v = [4] + [a + b for a, b in zip(sg["int"][0], sg["int"][1])]
    bwd_v = [2] + sg["bwd"][0]                       # Z + the backward op
    bg = K_max - fwd_groups

    def put(slot, unit, vec):
        for e in range(10):
            sigma = 4 if e < 7 else 10
            Wo[10 * slot + e, unit] += np.float32(vec[e] * 2.0 ** (10 - sigma))

    def bias(slot, vec):
        for e in range(10):
            sigma = 4 if e < 7 else 10
            bo[10 * slot + e] += np.float32(vec[e] / 2.0 ** sigma)
    for g in range(fwd_groups):
        put(g, 1 + g, leaf_v)
        put(g, 1 + fwd_groups + g, int_v)
    bias(0, [1] + sg["embed"])
    bias(fwd_groups - 1, [2] + sg["loss"])           # the loop's exit test + the loss op
    for g in range(bg):
        put(fwd_groups + g, 1 + 2 * fwd_groups + g, bwd_v)
    bias(K_max - 1, [2] + sg["opt"])                 # the backward loop's exit test + optimizer
    off = 10 * K_max
    for t in range(lo, hi + 1):                      # Loop F trip-count logits
        Wo[off, :] = 0.0
        Wo[off, 0] = np.float32(t)
        bo[off] = np.float32(-t * t / 2048.0)
        off += 1


CONFIGS = {"tiny": make_tiny, "moe": make_moe, "af": make_af, "lstm": make_lstm, "tree": make_tree}


def make(name, seed=0, **kw):
    return CONFIGS[name](seed=seed, **kw)


def op_time_ns(op):
    """Synthetic compute time of an operator (ns): 1 + (sum over its inputs of the element
    count) / 64 - the trace's execution time for the partition labels (P:L168 'execution time of
    each operator'); an input of both sides, no method arithmetic. Control rows take 0."""
    if op is None:
        return 0
    n = 0
    for shp in op.inputs:
        e = 1
        for d in shp:
            e *= int(d)
        n += e
    return 1 + n // 64


# ----------------------------------------------------------------------------
# fault injection (DYO_FAULT=drop_prefetch:p): a counter-based drop decision, implemented here
# for the test side and independently in libdyo (api.cpp drop_hash)
# ----------------------------------------------------------------------------

def drop_hash(seed, b, k, t):
    """splitmix64 of (seed, prediction b, group slot k, tensor t) -> uint64."""
    M = (1 << 64) - 1
    z = (int(seed) * 0x9E3779B97F4A7C15 + (int(b) << 40) + (int(k) << 20) + int(t)) & M
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & M
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & M
    return z ^ (z >> 31)


def drop_prefetch(W, p, seed, b):
    """The predicted tensor sets of prediction b with every read-first entry dropped when
    drop_hash(seed, b, k, t) / 2^64 < p (the injected 'mis-prediction' of DYO_FAULT)."""
    lim = int(p * (1 << 64)) if p < 1 else (1 << 64)
    return [[e for e in Wk if not (e[2] and drop_hash(seed, b, k, e[0]) < lim)] for k, Wk in enumerate(W)]


# ----------------------------------------------------------------------------
# counter-based content generator (migration byte checks; both sides call it)
# ----------------------------------------------------------------------------

def content_words_np(tid, version, n_words, start=0):
    """uint32 words of tensor `tid` at `version`: a 32-bit integer hash of the word index.

    Pure integer mixing (xorshift-multiply), identical to content_words_torch().
    """
    i = np.arange(start, start + n_words, dtype=np.int64)
    x = (i * 0x9E3779B1 + (tid * 0x85EBCA77) + (version * 0xC2B2AE3D) + 0x27D4EB2F) & 0xFFFFFFFF
    x ^= x >> 15
    x = (x * 0x2C1B3C6D) & 0xFFFFFFFF
    x ^= x >> 12
    x = (x * 0x297A2D39) & 0xFFFFFFFF
    x ^= x >> 15
    return x.astype(np.uint32)


def content_words_torch(tid, version, n_words, device, start=0):
    import torch
    i = torch.arange(start, start + n_words, dtype=torch.int64, device=device)
    M = 0xFFFFFFFF
    x = (i * 0x9E3779B1 + ((tid * 0x85EBCA77) & M) + ((version * 0xC2B2AE3D) & M) + 0x27D4EB2F) & M
    x ^= x >> 15
    x = (x * 0x2C1B3C6D) & M
    x ^= x >> 12
    x = (x * 0x297A2D39) & M
    x ^= x >> 15
    return x.to(torch.int32)  # reinterpreted as uint32 bits via two's complement wrap
