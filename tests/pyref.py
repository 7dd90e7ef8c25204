"""A second, independent re-implementation of DPOS (Alg. 1), SplitOperation
and OS-DPOS (Alg. 2) plus the sweep's candidate stream (R21), in plain
Python, written from PAPER.md and the readings in DESIGN.md -- used only to
PIN the C oracle (tests only).

It shares nothing with ``oracle/fastt_oracle.c`` beyond the paper: different
data structures (dict adjacency, a heap ready set, ``fractions.Fraction`` for
the R9 averages, memoised recursion for ranks, per-op split rewriting by
edge dictionaries) and no call into the oracle library.  The things the
three round-1 mutations changed are each written here from the text:

  * Alg. 2 line 12 and P:845 "stops the loop": the OS-DPOS loop
    ends at the first split-eligible CP op whose best split does not
    strictly improve (``split_search`` ... ``break``);
  * Alg. 2 line 5 "sort ... in descending order of computation
    time": ``sorted(..., key=(-cost, id))``;
  * P:600-609 (R9) "the smallest average computation time": averages are
    exact rationals (``Fraction``), ties to the lowest device id.

"P:<n>" = line n of /root/reference/PAPER.md.
"""
from __future__ import annotations

import heapq
import sys
from fractions import Fraction

INF = (1 << 63) - 1
MASK64 = (1 << 64) - 1
GOLDEN = 0x9E3779B97F4A7C15


def _cdiv(a, b):
    return -(-a // b)


class PG:
    """A DAG with devices, memory caps and cost models.
    edges: {(src, dst): (bytes, param)} (parallel edges merged, R11)."""

    def __init__(self, V, G, edges, cost, mem, param, smask, cap, lc, alpha, beta, copy_fs=0, alive=None):
        self.V, self.G = V, G
        self.edges = dict(edges)
        self.cost = [list(r) for r in cost]
        self.mem, self.param, self.smask = list(mem), list(param), list(smask)
        self.cap = list(cap)
        self.lc = [list(r) for r in lc]
        self.alpha, self.beta = list(alpha), list(beta)
        self.copy_fs = copy_fs
        self.alive = list(alive) if alive is not None else [True] * V
        self.succ = {i: [] for i in range(V)}
        self.pred = {i: [] for i in range(V)}
        for (s, d) in sorted(self.edges):
            self.succ[s].append(d)
            self.pred[d].append(s)

    @classmethod
    def from_desc(cls, desc):
        e = {}
        for s, d, b, p in zip(desc.src.tolist(), desc.dst.tolist(), desc.bytes.tolist(), desc.eparam.tolist()):
            ob, op_ = e.get((s, d), (0, 0))
            e[(s, d)] = (ob + b, op_ | (1 if p else 0))
        return cls(int(desc.n_ops), int(desc.n_devices), e, desc.cost.tolist(), desc.mem.tolist(),
                   desc.param.tolist(), desc.split_mask.tolist(), desc.cap.tolist(), desc.link_class.tolist(),
                   desc.alpha.tolist(), desc.beta.tolist(), int(desc.copy_fs))

    # R10: comm(b, s, t) = 0 on one device, else alpha_k + ceil(b * beta_k / 1e6)
    def comm(self, b, s, t):
        if s == t:
            return 0
        k = self.lc[s][t]
        return self.alpha[k] + _cdiv(b * self.beta[k], 1_000_000)


# ----------------------------------------------------------------- Alg. 1

def ranks(g: PG, pin=None, dset=None):
    """rank_u with w_i / c_ij as maxima over the allowed devices
    (R5): {pin} if pinned, else the candidate's devices."""
    pin = pin or {}
    devs = [d for d in range(g.G) if dset is None or d in dset]

    def allowed(i):
        return [pin[i]] if i in pin else devs

    memo = {}
    sys.setrecursionlimit(max(10000, 4 * g.V + 100))

    def ru(i):
        if i in memo:
            return memo[i]
        w = max(g.cost[i][d] for d in allowed(i)) if allowed(i) else 0
        best = 0
        for j in g.succ[i]:
            b = g.edges[(i, j)][0]
            c = max([g.comm(b, s, t) for s in allowed(i) for t in allowed(j) if s != t] or [0])
            best = max(best, c + ru(j))
        memo[i] = w + best
        return memo[i]

    return {i: ru(i) for i in range(g.V) if g.alive[i]}


def critical_path(g: PG, rk):
    """P:595-598, R4, R7: from the highest-(rank, -id) entry op, step to the
    successor with the largest rank (ties: lowest id)."""
    srcs = [i for i in range(g.V) if g.alive[i] and not g.pred[i]]
    if not srcs:
        return []
    cur = max(srcs, key=lambda i: (rk[i], -i))
    cp = [cur]
    while g.succ[cur]:
        cur = max(g.succ[cur], key=lambda j: (rk[j], -j))
        cp.append(cur)
    return cp


def cp_devices(g: PG, rk, pin=None, dset=None):
    """Alg. 1 lines 4-5 (R9): for every remaining
    device, the longest prefix of the remaining free CP ops that fits its
    memory; pick the device with the smallest exact average computation time
    (ties: lowest id); pin that prefix there; repeat on the other devices."""
    pin = pin or {}
    free = [o for o in critical_path(g, rk) if o not in pin]
    left = [d for d in range(g.G) if dset is None or d in dset]
    out = {}
    k = 0
    while k < len(free) and left:
        best = None
        for d in left:
            m, tot = 0, 0
            while k + m < len(free) and tot + g.mem[free[k + m]] <= g.cap[d]:
                tot += g.mem[free[k + m]]
                m += 1
            if m == 0:
                continue
            avg = Fraction(sum(g.cost[free[k + q]][d] for q in range(m)), m)
            if best is None or avg < best[0]:
                best = (avg, d, m)
        if best is None:
            break
        _, d, m = best
        for q in range(m):
            out[free[k + q]] = d
        left.remove(d)
        k += m
    return out


def dpos(g: PG, pin=None, dset=None, cp_pin=False):
    """DPOS (Alg. 1) under APPEND (R1), ready-set dequeue (R2),
    static memory (R8), hard perturbation pins.  Returns a dict or, if no
    device fits some op, {"status": 1, "makespan": INF}."""
    pin = pin or {}
    devs = [d for d in range(g.G) if dset is None or d in dset]
    rk = ranks(g, pin, dset)
    cpd = cp_devices(g, rk, pin, dset) if cp_pin else {}
    reserved = [0] * g.G
    for i, d in cpd.items():
        reserved[d] += g.mem[i]
    used, avail = [0] * g.G, [0] * g.G
    indeg = {i: len(g.pred[i]) for i in range(g.V) if g.alive[i]}
    heap = [(-rk[i], i) for i, n in indeg.items() if n == 0]
    heapq.heapify(heap)
    place, start, fin, deq = {}, {}, {}, []

    def est(i, d):
        return max([avail[d]] + [fin[m] + g.comm(g.edges[(m, i)][0], place[m], d) for m in g.pred[i]])

    while heap:
        _, i = heapq.heappop(heap)
        if i in pin:
            d = pin[i]
            if used[d] + reserved[d] + g.mem[i] > g.cap[d]:
                return {"status": 1, "makespan": INF}
        elif i in cpd:
            d = cpd[i]
            reserved[d] -= g.mem[i]
        else:
            opts = [(est(i, d) + g.cost[i][d], d) for d in devs if used[d] + reserved[d] + g.mem[i] <= g.cap[d]]
            if not opts:
                return {"status": 1, "makespan": INF}
            d = min(opts)[1]
        start[i] = est(i, d)
        fin[i] = start[i] + g.cost[i][d]
        place[i] = d
        avail[d] = fin[i]
        used[d] += g.mem[i]
        deq.append(i)
        for j in g.succ[i]:
            indeg[j] -= 1
            if indeg[j] == 0:
                heapq.heappush(heap, (-rk[j], j))
    seq = {i: q for q, i in enumerate(deq)}
    order = sorted(deq, key=lambda i: (start[i], seq[i]))
    return {"status": 0, "makespan": max(fin.values(), default=0), "place": place, "start": start, "order": order,
            "rank": rk, "cp_dev": cpd, "peak": used, "dequeue": deq}


# ------------------------------------------------- SplitOperation (Alg. 2)

def split_view(g: PG, op, dim, n):
    """SplitOperation(G, op, dim, n) (Alg. 2 lines 16-30) under
    R13: one split node per predecessor (ascending id), n sub-ops, one
    concat node per successor (ascending id), appended in that order; op
    becomes a tombstone.  Batch split cuts activation edges and replicates
    parameter edges, channel split the reverse; partitions
    floor(b/n) + (k < b mod n); sub-op cost ceil(cost/n); split/concat node
    cost ceil(b * copy_fs / 1e6), memory 0."""
    preds, succs = list(g.pred[op]), list(g.succ[op])
    V2 = g.V + len(preds) + n + len(succs)
    sp = {p: g.V + a for a, p in enumerate(preds)}
    subs = [g.V + len(preds) + k for k in range(n)]
    con = {s: g.V + len(preds) + n + a for a, s in enumerate(succs)}

    def part(b, k):
        return b // n + (1 if k < b % n else 0)

    def cut(p):
        return (not p) if dim == 0 else bool(p)

    edges = {(s, d): v for (s, d), v in g.edges.items() if op not in (s, d)}
    cost = [list(r) for r in g.cost] + [[0] * g.G for _ in range(V2 - g.V)]
    mem = list(g.mem) + [0] * (V2 - g.V)
    param = list(g.param) + [0] * (V2 - g.V)
    smask = list(g.smask) + [0] * (V2 - g.V)
    alive = list(g.alive) + [True] * (V2 - g.V)
    alive[op] = False
    cost[op] = [0] * g.G
    mem[op] = param[op] = smask[op] = 0
    act = g.mem[op] - g.param[op]
    for k, s in enumerate(subs):
        cost[s] = [_cdiv(c, n) for c in g.cost[op]]
        prm = g.param[op] if dim == 0 else part(g.param[op], k)
        mem[s] = part(act, k) + prm
        param[s] = prm
    for p in preds:
        b, pr = g.edges[(p, op)]
        cost[sp[p]] = [_cdiv(b * g.copy_fs, 1_000_000)] * g.G
        edges[(p, sp[p])] = (b, pr)
        for k, s in enumerate(subs):
            edges[(sp[p], s)] = (part(b, k) if cut(pr) else b, pr)
    for s_ in succs:
        b, pr = g.edges[(op, s_)]
        cost[con[s_]] = [_cdiv(b * g.copy_fs, 1_000_000)] * g.G
        for k, s in enumerate(subs):
            edges[(s, con[s_])] = (part(b, k), pr)
        edges[(con[s_], s_)] = (b, pr)
    return PG(V2, g.G, edges, cost, mem, param, smask, g.cap, g.lc, g.alpha, g.beta, g.copy_fs, alive)


def split_list(g: PG, place):
    """Alg. 2 lines 4-5 (R15): the critical path of the placed graph -- rank
    with the cost on the assigned device and the transfer time between the
    assigned devices -- keeping the ops with a splittable dimension, sorted
    by descending computation time on the assigned device (ties: lower id)."""
    memo = {}

    def rp(i):
        if i not in memo:
            memo[i] = g.cost[i][place[i]] + max(
                [g.comm(g.edges[(i, j)][0], place[i], place[j]) + rp(j) for j in g.succ[i]] or [0])
        return memo[i]

    sys.setrecursionlimit(max(10000, 4 * g.V + 100))
    rk = {i: rp(i) for i in range(g.V) if g.alive[i]}
    cp = [o for o in critical_path(g, rk) if g.smask[o]]
    return sorted(cp, key=lambda o: (-g.cost[o][place[o]], o))


def split_counts(G, pow2_only=False):
    """R14: n in 2..G (powers of two only with n_pow2_only)."""
    return [n for n in range(2, G + 1) if not pow2_only or (n & (n - 1)) == 0]


def split_search(g: PG, cp_pin=False, pow2_only=False):
    """OS-DPOS (Alg. 2, R15): DPOS of G0; the sorted list of
    split-eligible ops of its placed critical path (computed once); for each
    op the best of its splits (dims ascending, n ascending; smallest FT, first
    wins ties) is accepted if strictly better, otherwise the loop STOPS
    (Alg. 2 line 12; "stops the loop")."""
    r = dpos(g, cp_pin=cp_pin)
    if r["status"] != 0:
        return {"sp": [], "makespan": INF, "status": r["status"]}
    cur, ft_old, best_r = g, r["makespan"], r
    sp = []
    for op in split_list(g, r["place"]):
        best = None
        for dim in (0, 1):
            if not cur.smask[op] & (1 << dim):
                continue
            for n in split_counts(g.G, pow2_only):
                gv = split_view(cur, op, dim, n)
                rr = dpos(gv, cp_pin=cp_pin)
                if rr["status"] == 0 and (best is None or rr["makespan"] < best[0]):
                    best = (rr["makespan"], dim, n, gv, rr)
        if best is not None and best[0] < ft_old:
            ms, dim, n, gv, rr = best
            ft_old, cur, best_r = ms, gv, rr
            sp.append((op, dim, n))
        else:
            break
    return {"sp": sp, "makespan": ft_old, "status": 0, "place": best_r["place"], "start": best_r["start"],
            "n_ops_final": cur.V}


def split_search_best(g: PG, cp_pin=False, pow2_only=False):
    """Reading R23 (NEXT N2, a variant of Alg. 2): the list of R15 computed
    once on G0; every round evaluates every split (dims asc, n asc) of every
    list op not split yet, on the current graph, and accepts the smallest
    makespan (ties: list order, dim, n) iff strictly below the current one;
    stops when no split improves."""
    r = dpos(g, cp_pin=cp_pin)
    if r["status"] != 0:
        return {"sp": [], "makespan": INF, "status": r["status"]}
    lst = split_list(g, r["place"])
    cur, ft_old, best_r, sp, done = g, r["makespan"], r, [], set()
    while True:
        cands = []
        for li, op in enumerate(lst):
            if op in done:
                continue
            for dim in (0, 1):
                if cur.smask[op] & (1 << dim):
                    for n in split_counts(g.G, pow2_only):
                        gv = split_view(cur, op, dim, n)
                        rr = dpos(gv, cp_pin=cp_pin)
                        if rr["status"] == 0:
                            cands.append(((rr["makespan"], li, dim, n), op, gv, rr))
        if not cands:
            break
        key, op, gv, rr = min(cands, key=lambda x: x[0])
        if key[0] >= ft_old:
            break
        ft_old, cur, best_r = key[0], gv, rr
        done.add(op)
        sp.append((op, key[2], key[3]))
    return {"sp": sp, "makespan": ft_old, "status": 0, "place": best_r["place"], "start": best_r["start"],
            "n_ops_final": cur.V}


def split_search_multi(g: PG, cp_pin=False, pow2_only=False):
    """Reading R27 (NEXT N2 multi-split candidates, on top of R23): per round,
    every op's best improving split (smallest makespan, ties dim, n); the
    improving ops ranked by (makespan, list order); candidates C_j = the
    first j ranked ops' best splits applied in rank order, j = 1..min(4, k);
    accept the C_j of smallest makespan (ties: smaller j) -- written from the
    definition: each C_j built from scratch from the round's graph."""
    r = dpos(g, cp_pin=cp_pin)
    if r["status"] != 0:
        return {"sp": [], "makespan": INF, "status": r["status"]}
    lst = split_list(g, r["place"])
    cur, ft_old, best_r, sp, done, rounds = g, r["makespan"], r, [], set(), []
    while True:
        per_op = {}
        for li, op in enumerate(lst):
            if op in done or not any(cur.smask[op] & (1 << dim) for dim in (0, 1)):
                continue
            best = None
            for dim in (0, 1):
                if cur.smask[op] & (1 << dim):
                    for n in split_counts(g.G, pow2_only):
                        rr = dpos(split_view(cur, op, dim, n), cp_pin=cp_pin)
                        if rr["status"] == 0 and (best is None or rr["makespan"] < best[0]):
                            best = (rr["makespan"], dim, n)
            if best is not None and best[0] < ft_old:
                per_op[li] = best
        if not per_op:
            break
        ranked = sorted(per_op, key=lambda li: (per_op[li][0], li))[:4]
        choice = None
        for j in range(1, len(ranked) + 1):
            gj = cur
            for li in ranked[:j]:
                gj = split_view(gj, lst[li], per_op[li][1], per_op[li][2])
            rr = dpos(gj, cp_pin=cp_pin)
            if rr["status"] == 0 and (choice is None or rr["makespan"] < choice[0]):
                choice = (rr["makespan"], j, gj, rr)
        ms, j, gj, rr = choice
        for li in ranked[:j]:
            sp.append((lst[li], per_op[li][1], per_op[li][2]))
            done.add(lst[li])
        rounds.append(j)
        cur, ft_old, best_r = gj, ms, rr
    return {"sp": sp, "makespan": ft_old, "status": 0, "place": best_r["place"], "start": best_r["start"],
            "n_ops_final": cur.V, "rounds": rounds}


# ---------------------------------------------------- the sweep stream (R21)

def splitmix64(state):
    """One splitmix64 step (Steele, Lea, Flood 2014): returns (output, state)."""
    state = (state + GOLDEN) & MASK64
    z = state
    z = ((z ^ (z >> 30)) * 0xBF58476D1CE4E5B9) & MASK64
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & MASK64
    return z ^ (z >> 31), state


def stream(g: PG, seed, first, n, kmin=1, kmax=4, cp_pin=True, pow2_only=False, subsets=False):
    """Candidates first..first+n-1 of the R21 stream as tuples
    (kind, n_pins, split_dim, split_n, split_op, pin_op[4], pin_dev[4], dev_mask)."""
    base = dpos(g, cp_pin=cp_pin)
    bp = base["place"] if base["status"] == 0 else {i: 0 for i in range(g.V)}
    splits = []
    if base["status"] == 0:
        for op in split_list(g, base["place"]):
            for dim in (0, 1):
                if g.smask[op] & (1 << dim):
                    splits += [(op, dim, m) for m in split_counts(g.G, pow2_only)]
    nsub = g.G - 1 if subsets else 0
    live = [i for i in range(g.V) if g.alive[i]]
    out = []
    for c in range(first, first + n):
        if c == 0:
            out.append((0, 0, 0, 0, -1, [-1] * 4, [0] * 4, 0))
        elif c <= len(splits):
            op, dim, m = splits[c - 1]
            out.append((2, 0, dim, m, op, [-1] * 4, [0] * 4, 0))
        elif c <= len(splits) + nsub:
            k = c - len(splits)
            out.append((0, 0, 0, 0, -1, [-1] * 4, [0] * 4, (1 << k) - 1))
        else:
            st = seed ^ ((c * GOLDEN) & MASK64)
            x0, st = splitmix64(st)
            K = min(kmin + x0 % (kmax - kmin + 1), len(live))
            ops, devs = [-1] * 4, [0] * 4
            for k in range(K):
                xo, st = splitmix64(st)
                idx = xo % len(live)
                while live[idx] in ops[:k]:
                    idx = (idx + 1) % len(live)
                xd, st = splitmix64(st)
                ops[k] = live[idx]
                devs[k] = (bp[live[idx]] + 1 + xd % (g.G - 1)) % g.G
            out.append((1, K, 0, 0, -1, ops, devs, 0))
    return out
