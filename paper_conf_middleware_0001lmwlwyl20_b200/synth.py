"""Seeded synthetic inputs: training-graph-shaped DAGs, cost tables, link
models and memory caps for configs C1-C5 plus random
fuzz DAGs.

This module is the ONE piece shared by the oracle side (tests, bench
cpu_baseline) and the CUDA side (the product binding, bench).  It draws
random numbers and lays out arrays; it contains none of the method's
arithmetic (no ranks, no schedule, no split semantics).

Graph shape: forward ops, one backward grad-input op
per forward op and one grad-weight op per (parametric op, variable), one
apply op per variable and replica, data-parallel replication xR with a
cross-replica AddN per variable.  Costs are integer ns, log-normal around
op-type means, ~5-15% zero-cost ops (Var/Identity/Reshape);
bytes come from fp32 tensor shapes.  The recipe is restated in DESIGN.md.
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional

import numpy as np

INT64_MAX = np.iinfo(np.int64).max

DIM_BATCH_BIT = 1
DIM_CHANNEL_BIT = 2

# link presets (R10): alpha ns, beta fs/byte
LINK_PAPER = (10_000, 40_000)   # V100 NVLink-shaped, ~25 GB/s effective
LINK_B200 = (5_000, 1_111)      # NVLink 5 / NVSwitch, 900 GB/s per direction


@dataclasses.dataclass
class GraphDesc:
    name: str
    n_ops: int
    n_devices: int
    src: np.ndarray          # int32 [E]
    dst: np.ndarray          # int32 [E]
    bytes: np.ndarray        # int64 [E]
    eparam: np.ndarray       # uint8 [E], 1 = parameter tensor
    cost: np.ndarray         # int64 [V, G] ns
    mem: np.ndarray          # int64 [V] bytes
    param: np.ndarray        # int64 [V] bytes (<= mem)
    split_mask: np.ndarray   # uint8 [V]
    cap: np.ndarray          # int64 [G]
    link_class: np.ndarray   # uint8 [G, G]
    alpha: np.ndarray        # int64 [K]
    beta: np.ndarray         # int64 [K]
    copy_fs: int = 0
    seed: int = 0
    op_type: Optional[List[str]] = None

    @property
    def n_edges(self):
        return int(len(self.src))

    def summary(self):
        return {"name": self.name, "V": self.n_ops, "E": self.n_edges, "G": self.n_devices,
                "K": int(len(self.alpha)), "seed": self.seed}


def _finish(name, G, srcs, dsts, byts, eprm, cost, mem, prm, smask, cap=None, link=LINK_PAPER, classes=None,
            copy_fs=0, seed=0, types=None):
    V = len(mem)
    if classes is None:
        lc = np.zeros((G, G), np.uint8)
        alpha = np.array([link[0]], np.int64)
        beta = np.array([link[1]], np.int64)
    else:
        lc, alpha, beta = classes
    if cap is None:
        cap = np.full(G, INT64_MAX, np.int64)
    return GraphDesc(name=name, n_ops=V, n_devices=G, src=np.asarray(srcs, np.int32), dst=np.asarray(dsts, np.int32),
                     bytes=np.asarray(byts, np.int64), eparam=np.asarray(eprm, np.uint8),
                     cost=np.ascontiguousarray(np.asarray(cost, np.int64).reshape(V, G)),
                     mem=np.asarray(mem, np.int64), param=np.asarray(prm, np.int64),
                     split_mask=np.asarray(smask, np.uint8), cap=np.asarray(cap, np.int64),
                     link_class=np.ascontiguousarray(np.asarray(lc, np.uint8).reshape(G, G)),
                     alpha=np.asarray(alpha, np.int64), beta=np.asarray(beta, np.int64), copy_fs=int(copy_fs),
                     seed=int(seed), op_type=types)


# --------------------------------------------------------------- hand graphs

def diamond():
    """A->B, A->C, B->D, C->D; bytes 4,6,3,7; G=2;
    one link class alpha=0, beta=1e6 fs/B (comm = bytes ns); costs 10,20,15,5."""
    G = 2
    cost = np.array([[10, 10], [20, 20], [15, 15], [5, 5]], np.int64)
    return _finish("diamond", G, [0, 0, 1, 2], [1, 2, 3, 3], [4, 6, 3, 7], [0, 0, 0, 0], cost, [0] * 4, [0] * 4,
                   [0] * 4, link=(0, 1_000_000))


def split_chain():
    """P(1) -> X(100, batch-splittable) -> Q(1); G=2; zero comm."""
    G = 2
    cost = np.array([[1, 1], [100, 100], [1, 1]], np.int64)
    return _finish("split_chain", G, [0, 1], [1, 2], [64, 64], [0, 0], cost, [0] * 3, [0] * 3,
                   [0, DIM_BATCH_BIT, 0], link=(0, 0))


def append_vs_insert():
    """A(10) -> B(10) with comm 20; Z(5) isolated; G=2."""
    G = 2
    cost = np.array([[10, 10], [10, 10], [5, 5]], np.int64)
    return _finish("append_vs_insert", G, [0], [1], [20], [0], cost, [0] * 3, [0] * 3, [0] * 3,
                   link=(0, 1_000_000))


def stop_rule_chain():
    """tests/golden/alg2_stop_rule.json: P(1) -> X(100) -> Q(1) -> Y(60) -> R(1),
    X and Y batch-splittable; bytes 1000, 1000, 0, 0; G=2; one link class
    alpha=0, beta=1e6 fs/B (comm = bytes ns)."""
    G = 2
    cost = np.repeat(np.array([1, 100, 1, 60, 1], np.int64)[:, None], G, axis=1)
    return _finish("stop_rule_chain", G, [0, 1, 2, 3], [1, 2, 3, 4], [1000, 1000, 0, 0], [0] * 4, cost, [0] * 5,
                   [0] * 5, [0, DIM_BATCH_BIT, 0, DIM_BATCH_BIT, 0], link=(0, 1_000_000))


def r9_average_pair():
    """tests/golden/r9_exact_average.json: A -> B (5 bytes); costs A (3, 3),
    B (4, 100); mem 10 each; caps (20, 10); G=2; comm = bytes ns."""
    G = 2
    cost = np.array([[3, 3], [4, 100]], np.int64)
    return _finish("r9_average_pair", G, [0], [1], [5], [0], cost, [10, 10], [0, 0], [0, 0], cap=[20, 10],
                   link=(0, 1_000_000))


# ------------------------------------------------------------ random fuzz

def random_dag(seed, V=None, G=None, K=None, p_edge=None, zero_frac=None, caps="random", homogeneous=None,
               max_in=None):
    """Random DAG for fuzzing: ids in topological order, random costs with a
    zero-cost fraction (ties), random bytes, random caps (some infeasible),
    1-3 link classes, random split masks."""
    rng = np.random.default_rng(seed)
    V = int(rng.integers(1, 300)) if V is None else V
    G = int(rng.integers(1, 9)) if G is None else G
    K = int(rng.integers(1, 4)) if K is None else K
    zero_frac = float(rng.uniform(0, 0.3)) if zero_frac is None else zero_frac
    homogeneous = bool(rng.integers(0, 2)) if homogeneous is None else homogeneous
    max_in = int(rng.integers(1, 7)) if max_in is None else max_in
    srcs, dsts = [], []
    for j in range(1, V):
        n_in = int(rng.integers(0, max_in + 1))
        if p_edge is not None:
            n_in = int(rng.binomial(min(j, 8), p_edge))
        lo = max(0, j - int(rng.integers(1, 64)))
        for _ in range(n_in):
            i = int(rng.integers(lo, j))
            srcs.append(i)
            dsts.append(j)
    # a few duplicate (parallel) edges exercise the merge rule R11
    for _ in range(int(rng.integers(0, 3))):
        if srcs:
            q = int(rng.integers(0, len(srcs)))
            srcs.append(srcs[q])
            dsts.append(dsts[q])
    E = len(srcs)
    byts = rng.integers(0, 1 << 20, E).astype(np.int64)
    byts[rng.random(E) < 0.1] = 0
    eprm = (rng.random(E) < 0.2).astype(np.uint8)
    base = rng.integers(0, 1000, V).astype(np.int64)
    base[rng.random(V) < zero_frac] = 0
    if homogeneous:
        cost = np.repeat(base[:, None], G, axis=1)
    else:
        jit = rng.integers(0, 200, (V, G)).astype(np.int64)
        cost = base[:, None] + jit * (base[:, None] > 0)
    mem = rng.integers(0, 1000, V).astype(np.int64)
    prm = (mem * rng.random(V) * (rng.random(V) < 0.3)).astype(np.int64)
    smask = rng.integers(0, 4, V).astype(np.uint8) * (rng.random(V) < 0.3)
    if caps == "random":
        mode = int(rng.integers(0, 3))
        if mode == 0:
            cap = np.full(G, INT64_MAX, np.int64)
        else:
            tot = int(mem.sum())
            frac = 1.3 if mode == 1 else 0.9
            cap = np.array([int(tot * frac / G) + int(rng.integers(0, 2000)) for _ in range(G)], np.int64)
    elif caps == "none":
        cap = np.full(G, INT64_MAX, np.int64)
    else:
        cap = np.asarray(caps, np.int64)
    lc = rng.integers(0, K, (G, G)).astype(np.uint8)
    alpha = rng.integers(0, 200, K).astype(np.int64)
    beta = rng.integers(0, 2000, K).astype(np.int64)
    copy_fs = int(rng.integers(0, 3)) * 100
    return _finish("random_%d" % seed, G, srcs, dsts, byts, eprm, cost, mem, prm, smask, cap=cap,
                   classes=(lc, alpha, beta), copy_fs=copy_fs, seed=seed)


# ---------------------------------------------------- training-graph builder

# per-op-type relative cost weights (V100-era shapes; rescaled per model)
_TYPE_W = {
    "Var": 0.0, "Data": 0.0, "Identity": 0.0, "Reshape": 0.0, "Shape": 0.0,
    "MatMul": 10.0, "BatchMatMul": 6.0, "Conv2D": 12.0, "BiasAdd": 0.6, "Relu": 0.5, "Gelu": 0.8,
    "Add": 0.5, "Mul": 0.5, "Sub": 0.5, "Mean": 0.6, "Rsqrt": 0.3, "Square": 0.4, "Softmax": 1.2,
    "Dropout": 0.7, "RandomUniform": 0.4, "Transpose": 0.8, "BatchNorm": 1.5, "MaxPool": 1.0, "AvgPool": 1.0,
    "ConcatV2": 0.8, "Loss": 0.5, "Embedding": 1.0, "Tanh": 0.4, "Pow": 0.4, "Cast": 0.2,
}
_ZERO = {"Var", "Data", "Identity", "Reshape", "Shape"}
_SPLITTABLE = {"MatMul", "Conv2D", "BatchMatMul"}


class _TB:
    """Tiny training-graph builder for one model replica description."""

    def __init__(self):
        self.ops = []      # dict(type, inputs: [(op, bytes, is_param)], out_bytes, param_bytes, w)
        self.vars = []     # op ids of Var ops

    def var(self, nbytes):
        i = len(self.ops)
        self.ops.append(dict(type="Var", inputs=[], out=nbytes, param=nbytes, w=0.0))
        self.vars.append(i)
        return i

    def op(self, typ, inputs, out, w=None, scale=1.0):
        i = len(self.ops)
        ins = []
        for x in inputs:
            is_p = self.ops[x]["type"] == "Var"
            ins.append((x, self.ops[x]["out"], is_p))
        self.ops.append(dict(type=typ, inputs=ins, out=int(out), param=0, w=(_TYPE_W[typ] if w is None else w) * scale))
        return i


def _replicate_training(tb: _TB, R, G, rng, name, total_cost_ns, link=LINK_PAPER, hetero_ppm=0, caps=None,
                        cap_frac=None, seed=0, loss_op=None):
    """Expand a forward description into a DP-replicated training DAG:
    fwd + bwd (grad-input per op, grad-weight per (op, var)) + per-variable
    cross-replica AddN + per-replica apply.  Returns a GraphDesc."""
    n = len(tb.ops)
    consumers = [[] for _ in range(n)]
    for j, o in enumerate(tb.ops):
        for (x, b, p) in o["inputs"]:
            consumers[x].append(j)
    ids_types, costw, outb, prmb, smask = [], [], [], [], []
    edges = []  # (s, d, bytes, param)

    def new(typ, w, out, param=0, split=0):
        ids_types.append(typ)
        costw.append(w)
        outb.append(int(out))
        prmb.append(int(param))
        smask.append(split)
        return len(ids_types) - 1

    rd = {}  # (replica, var) -> Identity read op (TF 1.x reads variables through Identity)

    var_grads = {v: [] for v in tb.vars}   # var -> list over replicas of grad op ids
    var_ops = {v: [] for v in tb.vars}
    loss = loss_op if loss_op is not None else n - 1
    for r in range(R):
        f = {}
        for j, o in enumerate(tb.ops):
            sm = (DIM_BATCH_BIT | DIM_CHANNEL_BIT) if o["type"] in _SPLITTABLE else 0
            pb = sum(b for (x, b, p) in o["inputs"] if p)
            f[j] = new(o["type"], o["w"], o["out"], param=o["param"] if o["type"] == "Var" else pb, split=sm)
            if o["type"] == "Var":
                var_ops[j].append(f[j])
                rd[j] = new("Identity", 0.0, 0)
                edges.append((f[j], rd[j], o["out"], 1))
            for (x, b, p) in o["inputs"]:
                edges.append((rd[x] if p else f[x], f[j], b, int(p)))
        # backward in reverse order: dY[j] = gradient of op j's output
        dY = {loss: None}
        gin = {}
        for j in range(n - 1, -1, -1):
            o = tb.ops[j]
            if o["type"] in ("Var", "Data"):
                continue
            if j != loss:
                contrib = [gin[c] for c in consumers[j] if c in gin]
                if not contrib:
                    continue
                if len(contrib) == 1:
                    dY[j] = contrib[0]
                else:
                    a = new("AddN", 0.4 * o["w"] / max(1.0, _TYPE_W.get(o["type"], 1.0)) + 0.3, o["out"])
                    for c in contrib:
                        edges.append((c, a, o["out"], 0))
                    dY[j] = a
            act_in = [(x, b) for (x, b, p) in o["inputs"] if not p]
            par_in = [(x, b) for (x, b, p) in o["inputs"] if p]
            needs_gi = any(tb.ops[x]["type"] not in ("Var", "Data") for (x, b) in act_in)
            sm = (DIM_BATCH_BIT | DIM_CHANNEL_BIT) if o["type"] in _SPLITTABLE else 0
            if needs_gi:
                gi = new(o["type"] + "Grad", o["w"] if o["w"] > 0 else 0.3, max(b for (x, b) in act_in), split=sm)
                if dY[j] is not None:
                    edges.append((dY[j], gi, o["out"], 0))
                for (x, b) in act_in:                  # saved activations (long fwd->bwd edges)
                    edges.append((f[x], gi, b, 0))
                for (x, b) in par_in:
                    edges.append((rd[x], gi, b, 1))
                gin[j] = gi
            for (x, b) in par_in:
                gw = new(o["type"] + "GradW", o["w"] if o["w"] > 0 else 0.3, b, split=sm)
                if dY[j] is not None:
                    edges.append((dY[j], gw, o["out"], 0))
                for (y, bb) in act_in:
                    edges.append((f[y], gw, bb, 0))
                var_grads[x].append(gw)
        # the loss op needs the label input; gradients start there
    for v in tb.vars:
        b = tb.ops[v]["out"]
        grads = var_grads[v]
        if not grads:
            continue
        if R > 1:
            agg = new("AddN", 0.3, b)
            for gop in grads:
                edges.append((gop, agg, b, 1))
        else:
            agg = grads[0]
        for r in range(R):
            ap = new("Apply", 0.3, 0)
            edges.append((agg, ap, b, 1))
            edges.append((var_ops[v][r], ap, b, 1))
    V = len(ids_types)
    w = np.asarray(costw, np.float64)
    # log-normal jitter, zero-cost types stay zero, a few extra zero-cost ops
    jit = rng.lognormal(0.0, 0.35, V)
    w = w * jit
    zero_extra = rng.random(V) < 0.03
    w[zero_extra] = 0.0
    if w.sum() > 0:
        w = w * (total_cost_ns * R / w.sum())
    base = np.rint(w).astype(np.int64)
    cost = np.repeat(base[:, None], G, axis=1)
    if hetero_ppm:
        jd = rng.integers(-hetero_ppm, hetero_ppm + 1, (V, G))
        cost = cost + (cost * jd) // 1_000_000
    outb = np.asarray(outb, np.int64)
    prmb = np.asarray(prmb, np.int64)
    mem = outb + prmb
    types = ids_types
    e = np.asarray(edges, dtype=np.int64).reshape(-1, 4)
    cap = None
    if cap_frac is not None:
        per = -(-int(mem.sum()) // G)
        cap = np.full(G, int(per * cap_frac), np.int64)
    elif caps is not None:
        cap = caps
    return _finish(name, G, e[:, 0], e[:, 1], e[:, 2], e[:, 3], cost, mem, prmb, np.asarray(smask, np.uint8),
                   cap=cap, link=link, seed=seed, types=types)


F32 = 4


def _layernorm(tb, x, nbytes, hid):
    g = tb.var(hid * F32)
    b = tb.var(hid * F32)
    m = tb.op("Mean", [x], nbytes // hid)
    d = tb.op("Sub", [x, m], nbytes)
    s = tb.op("Square", [d], nbytes)
    v = tb.op("Mean", [s], nbytes // hid)
    e = tb.op("Add", [v], nbytes // hid, w=0.1)
    r = tb.op("Rsqrt", [e], nbytes // hid)
    nrm = tb.op("Mul", [d, r], nbytes)
    sc = tb.op("Mul", [nrm, g], nbytes)
    return tb.op("Add", [sc, b], nbytes)


def _dropout(tb, x, nbytes):
    u = tb.op("RandomUniform", [], nbytes)
    k = tb.op("Cast", [u], nbytes)
    return tb.op("Mul", [x, k], nbytes, w=_TYPE_W["Dropout"])


def _dense(tb, x, din, dout, rows, act=None):
    W = tb.var(din * dout * F32)
    b = tb.var(dout * F32)
    y = tb.op("MatMul", [x, W], rows * dout * F32, scale=din * dout / (1024 * 1024))
    y = tb.op("BiasAdd", [y, b], rows * dout * F32)
    if act == "relu":
        y = tb.op("Relu", [y], rows * dout * F32)
    return y


def bert_large(G=8, R=4, seed=0xFA57_0004, layers=24, hid=1024, heads=16, seq=64, batch=16, ffn=4096,
               link=LINK_PAPER, hetero_ppm=0, iter_s=0.19, cap_frac=None):
    """C5: BERT-large training DAG (~20k ops), seq 64, batch 16
    (P:930), Sigma cost per replica ~0.19 s.  cap_frac (test
    variants only): per-device caps = cap_frac x ceil(Sigma mem / G)."""
    rng = np.random.default_rng(seed)
    tb = _TB()
    rows = batch * seq // R if R > 1 else batch * seq
    act = rows * hid * F32
    ids = tb.op("Data", [], rows * 4)
    emb = tb.var(30522 * hid * F32)
    pos = tb.var(512 * hid * F32)
    typ = tb.var(2 * hid * F32)
    x = tb.op("Embedding", [ids, emb], act)
    p = tb.op("Embedding", [ids, pos], act, w=0.3)
    t = tb.op("Embedding", [ids, typ], act, w=0.3)
    x = tb.op("Add", [x, p], act)
    x = tb.op("Add", [x, t], act)
    x = _layernorm(tb, x, act, hid)
    x = _dropout(tb, x, act)
    mask = tb.op("Data", [], rows * seq * F32 // hid + 4)
    bsz = max(1, rows // seq)
    sc_bytes = bsz * heads * seq * seq * F32
    for _ in range(layers):
        q = _dense(tb, x, hid, hid, rows)
        k = _dense(tb, x, hid, hid, rows)
        v = _dense(tb, x, hid, hid, rows)
        q = tb.op("Transpose", [tb.op("Reshape", [q], act)], act)
        k = tb.op("Transpose", [tb.op("Reshape", [k], act)], act)
        v = tb.op("Transpose", [tb.op("Reshape", [v], act)], act)
        s = tb.op("BatchMatMul", [q, k], sc_bytes, scale=0.5)
        s = tb.op("Mul", [s], sc_bytes, w=0.3)
        s = tb.op("Add", [s, mask], sc_bytes)
        s = tb.op("Softmax", [s], sc_bytes)
        s = _dropout(tb, s, sc_bytes)
        c = tb.op("BatchMatMul", [s, v], act, scale=0.5)
        c = tb.op("Reshape", [tb.op("Transpose", [c], act)], act)
        o = _dense(tb, c, hid, hid, rows)
        o = _dropout(tb, o, act)
        x = _layernorm(tb, tb.op("Add", [o, x], act), act, hid)
        h = _dense(tb, x, hid, ffn, rows)
        hb = rows * ffn * F32
        # GELU (tanh approximation) decomposed as in TF 1.x graphs
        g3 = tb.op("Pow", [h], hb)
        g3 = tb.op("Mul", [g3], hb, w=0.2)
        g3 = tb.op("Add", [h, g3], hb)
        g3 = tb.op("Mul", [g3], hb, w=0.2)
        g3 = tb.op("Tanh", [g3], hb)
        g3 = tb.op("Add", [g3], hb, w=0.2)
        g3 = tb.op("Mul", [g3], hb, w=0.2)
        h = tb.op("Mul", [h, g3], hb)
        o = _dense(tb, h, ffn, hid, rows)
        o = _dropout(tb, o, act)
        x = _layernorm(tb, tb.op("Add", [o, x], act), act, hid)
    pool = _dense(tb, x, hid, hid, rows)
    pool = tb.op("Tanh", [pool], act)
    logits = _dense(tb, pool, hid, 2, rows)
    lbl = tb.op("Data", [], rows * 4)
    tb.op("Loss", [logits, lbl], 4)
    return _replicate_training(tb, R, G, rng, "C5_bert_large", int(iter_s * 1e9), link=link, hetero_ppm=hetero_ppm,
                               cap_frac=cap_frac, seed=seed)


def _conv(tb, x, cin, cout, k, hw_out, bs, stride_w=1.0, bn=True, relu=True):
    W = tb.var(k * k * cin * cout * F32)
    ob = bs * hw_out * hw_out * cout * F32
    flops = bs * hw_out * hw_out * cout * cin * k * k
    y = tb.op("Conv2D", [x, W], ob, scale=flops / 2.0e9 * stride_w)
    if bn:
        g = tb.var(cout * F32)
        b = tb.var(cout * F32)
        m = tb.op("Mean", [y], cout * F32)
        y = tb.op("BatchNorm", [y, m, g, b], ob)
    if relu:
        y = tb.op("Relu", [y], ob)
    return y


def resnet50(G=4, R=4, seed=0xFA57_0001, batch=32, link=LINK_PAPER, hetero_ppm=0, iter_s=0.25):
    """C2: ResNet-50 training DAG (~5k ops) on 4 simulated GPUs."""
    rng = np.random.default_rng(seed)
    tb = _TB()
    bs = max(1, batch // R)
    x = tb.op("Data", [], bs * 224 * 224 * 3 * F32)
    x = _conv(tb, x, 3, 64, 7, 112, bs)
    x = tb.op("MaxPool", [x], bs * 56 * 56 * 64 * F32)
    cin, hw = 64, 56
    for (nblk, mid, out, hwo) in [(3, 64, 256, 56), (4, 128, 512, 28), (6, 256, 1024, 14), (3, 512, 2048, 7)]:
        for bi in range(nblk):
            y = _conv(tb, x, cin, mid, 1, hwo, bs)
            y = _conv(tb, y, mid, mid, 3, hwo, bs)
            y = _conv(tb, y, mid, out, 1, hwo, bs, relu=False)
            sc = _conv(tb, x, cin, out, 1, hwo, bs, relu=False) if bi == 0 else x
            x = tb.op("Relu", [tb.op("Add", [y, sc], bs * hwo * hwo * out * F32)], bs * hwo * hwo * out * F32)
            cin = out
    x = tb.op("AvgPool", [x], bs * 2048 * F32)
    x = _dense(tb, x, 2048, 1000, bs)
    lbl = tb.op("Data", [], bs * 4)
    tb.op("Loss", [x, lbl], 4)
    return _replicate_training(tb, R, G, rng, "C2_resnet50", int(iter_s * 1e9), link=link, hetero_ppm=hetero_ppm,
                               seed=seed)


def inception_v3(G=8, R=4, seed=0xFA57_0002, batch=64, link=LINK_PAPER, hetero_ppm=0, iter_s=0.335):
    """C3: Inception-v3 training DAG (~8-10k ops, wide 4-tower modules),
    Sigma cost per replica calibrated to 0.335 s (Table 1)."""
    rng = np.random.default_rng(seed)
    tb = _TB()
    bs = max(1, batch // R)
    x = tb.op("Data", [], bs * 299 * 299 * 3 * F32)

    def cv(x, ci, co, k, hw, bn=True):
        return _conv(tb, x, ci, co, k, hw, bs, bn=False) if not bn else _conv(tb, x, ci, co, k, hw, bs)

    x = cv(x, 3, 32, 3, 149)
    x = cv(x, 32, 32, 3, 147)
    x = cv(x, 32, 64, 3, 147)
    x = tb.op("MaxPool", [x], bs * 73 * 73 * 64 * F32)
    x = cv(x, 64, 80, 1, 73)
    x = cv(x, 80, 192, 3, 71)
    x = tb.op("MaxPool", [x], bs * 35 * 35 * 192 * F32)
    cin = 192

    def module(x, cin, hw, towers):
        outs, cout = [], 0
        for tw in towers:
            y, c = x, cin
            for (co, k) in tw:
                if co == 0:
                    y = tb.op("AvgPool", [y], bs * hw * hw * c * F32)
                else:
                    y = cv(y, c, co, k, hw)
                    c = co
            outs.append(y)
            cout += c
        return tb.op("ConcatV2", outs, bs * hw * hw * cout * F32), cout

    for _ in range(3):
        x, cin = module(x, cin, 35, [[(64, 1)], [(48, 1), (64, 5)], [(64, 1), (96, 3), (96, 3)], [(0, 3), (32, 1)]])
    x, cin = module(x, cin, 17, [[(384, 3)], [(64, 1), (96, 3), (96, 3)], [(0, 3)]])
    for _ in range(4):
        x, cin = module(x, cin, 17, [[(192, 1)], [(128, 1), (128, 7), (192, 7)],
                                     [(128, 1), (128, 7), (128, 7), (128, 7), (192, 7)], [(0, 3), (192, 1)]])
    x, cin = module(x, cin, 8, [[(192, 1), (320, 3)], [(192, 1), (192, 7), (192, 7), (192, 3)], [(0, 3)]])
    for _ in range(2):
        x, cin = module(x, cin, 8, [[(320, 1)], [(384, 1), (384, 3)], [(448, 1), (384, 3), (384, 3)],
                                    [(0, 3), (192, 1)]])
    x = tb.op("AvgPool", [x], bs * cin * F32)
    x = _dense(tb, x, cin, 1000, bs)
    lbl = tb.op("Data", [], bs * 4)
    tb.op("Loss", [x, lbl], 4)
    return _replicate_training(tb, R, G, rng, "C3_inception_v3", int(iter_s * 1e9), link=link,
                               hetero_ppm=hetero_ppm, seed=seed)


# Table 5: per-op V100 times anchor VGG-19's cost scale
VGG_TABLE5_MS = {"conv1_1": 1.847, "conv1_2": 11.14, "conv1_2bp": 26.744, "relu": 1.08, "pool": 0.737, "fc6": 1.374}


def vgg19(G=8, R=8, seed=0xFA57_0003, batch=64, link=LINK_PAPER, hetero_ppm=0, cap_frac=1.25, iter_s=0.496):
    """C4: VGG-19 training DAG (~2k ops) with large FC layers (fc6 has
    102,764,544 params, Table 5) and per-device memory caps
    cap = cap_frac * ceil(Sigma mem / G) (1.25, or 1.05 for infeasible
    candidates)."""
    rng = np.random.default_rng(seed)
    tb = _TB()
    bs = max(1, batch // R)
    x = tb.op("Data", [], bs * 224 * 224 * 3 * F32)
    cin, hw = 3, 224
    for (nconv, cout) in [(2, 64), (2, 128), (4, 256), (4, 512), (4, 512)]:
        for _ in range(nconv):
            W = tb.var(3 * 3 * cin * cout * F32)
            b = tb.var(cout * F32)
            ob = bs * hw * hw * cout * F32
            y = tb.op("Conv2D", [x, W], ob, scale=bs * hw * hw * cout * cin * 9 / 2.0e9)
            y = tb.op("BiasAdd", [y, b], ob)
            x = tb.op("Relu", [y], ob)
            cin = cout
        hw //= 2
        x = tb.op("MaxPool", [x], bs * hw * hw * cin * F32)
    x = tb.op("Reshape", [x], bs * 7 * 7 * 512 * F32)
    x = _dense(tb, x, 7 * 7 * 512, 4096, bs, act="relu")
    x = _dropout(tb, x, bs * 4096 * F32)
    x = _dense(tb, x, 4096, 4096, bs, act="relu")
    x = _dropout(tb, x, bs * 4096 * F32)
    x = _dense(tb, x, 4096, 1000, bs)
    lbl = tb.op("Data", [], bs * 4)
    tb.op("Loss", [x, lbl], 4)
    return _replicate_training(tb, R, G, rng, "C4_vgg19", int(iter_s * 1e9), link=link, hetero_ppm=hetero_ppm,
                               cap_frac=cap_frac, seed=seed)


def mlp2(G=2, R=2, seed=0xFA57_0000, batch=64, din=784, dh=256, dout=10, link=LINK_PAPER):
    """C1: 2-layer MLP (MatMul-BiasAdd-Relu x2, softmax-xent) training DAG,
    ~50 ops on 2 simulated devices; microsecond-scale costs."""
    rng = np.random.default_rng(seed)
    tb = _TB()
    bs = max(1, batch // R)
    x = tb.op("Data", [], bs * din * F32)
    x = _dense(tb, x, din, dh, bs, act="relu")
    x = _dense(tb, x, dh, dout, bs)
    lbl = tb.op("Data", [], bs * 4)
    tb.op("Loss", [x, lbl], 4)
    return _replicate_training(tb, R, G, rng, "C1_mlp2", 400_000, link=link, seed=seed)


CONFIGS = {
    "C1": mlp2,
    "C2": resnet50,
    "C3": inception_v3,
    "C4": vgg19,
    "C5": bert_large,
    # C5 with the model replicated once per device (OS-DPOS starts
    # from a data-parallel graph with one replica per GPU): ~38k ops, past the
    # ready-set kernel's 32,768 positions (topological priority order)
    "C5R8": lambda **kw: bert_large(**dict({"R": 8}, **kw)),
}


def config(name, **kw):
    return CONFIGS[name](**kw)


def edge_csr(desc: GraphDesc):
    """Edge list -> CSR by source (stable), the layout the C-ABI takes.  Pure
    array marshalling."""
    order = np.argsort(desc.src, kind="stable")
    succ_dst = np.ascontiguousarray(desc.dst[order].astype(np.int32))
    byts = np.ascontiguousarray(desc.bytes[order].astype(np.int64))
    prm = np.ascontiguousarray(desc.eparam[order].astype(np.uint8))
    counts = np.bincount(desc.src, minlength=desc.n_ops) if desc.n_edges else np.zeros(desc.n_ops, np.int64)
    off = np.zeros(desc.n_ops + 1, np.int32)
    off[1:] = np.cumsum(counts)
    return off, succ_dst, byts, prm
