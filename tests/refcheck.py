"""Independent pure-Python checkers used to PIN the oracle (tests only).

Nothing here calls the oracle's arithmetic: these are written directly from
the paper's definitions as brute force / verification routines.
  * merged adjacency (R11) from a GraphDesc,
  * rank by explicit enumeration of all paths,
  * an APPEND evaluator of a fixed (placement, order) (R1, R6),
  * brute force over all placements x all topological orders,
  * schedule invariants,
  * a greedy-step replay checker, APPEND or INSERT (R1i, EST by
    brute force over time), static or liveness memory (R24), device subsets
    (R25),
  * liveness peaks by their definition (R24).
"""
from __future__ import annotations

import itertools

INF = (1 << 63) - 1


class G:
    def __init__(self, desc):
        self.V = int(desc.n_ops)
        self.G = int(desc.n_devices)
        e = {}
        for s, d, b, p in zip(desc.src.tolist(), desc.dst.tolist(), desc.bytes.tolist(), desc.eparam.tolist()):
            if (s, d) in e:
                e[(s, d)] = (e[(s, d)][0] + b, e[(s, d)][1] | (1 if p else 0))
            else:
                e[(s, d)] = (b, 1 if p else 0)
        self.edges = e
        self.succ = [[] for _ in range(self.V)]
        self.pred = [[] for _ in range(self.V)]
        for (s, d), (b, p) in sorted(e.items()):
            self.succ[s].append((d, b))
            self.pred[d].append((s, b))
        for l in self.pred:
            l.sort()
        self.cost = desc.cost.tolist()
        self.mem = desc.mem.tolist()
        self.param = desc.param.tolist()
        self.cap = desc.cap.tolist()
        self.lc = desc.link_class.tolist()
        self.alpha = desc.alpha.tolist()
        self.beta = desc.beta.tolist()

    def comm(self, b, s, t):
        if s == t:
            return 0
        k = self.lc[s][t]
        return self.alpha[k] + -(-(b * self.beta[k]) // 1_000_000)

    def w(self, i, pin=None, dset=None):
        if pin and i in pin:
            return self.cost[i][pin[i]]
        return max(self.cost[i][d] for d in range(self.G) if dset is None or d in dset)

    def c(self, i, j, b, pin=None, dset=None):
        best = 0
        for s in range(self.G):
            if pin and i in pin and s != pin[i]:
                continue
            if not (pin and i in pin) and dset is not None and s not in dset:
                continue
            for t in range(self.G):
                if pin and j in pin and t != pin[j]:
                    continue
                if not (pin and j in pin) and dset is not None and t not in dset:
                    continue
                if s != t:
                    best = max(best, self.comm(b, s, t))
        return best


def rank_by_paths(g: G, pin=None, dset=None):
    """rank_u(i) = max over all paths i -> sink of sum(w) + sum(c), by explicit
    enumeration of paths (exponential; small graphs only).  dset: the
    candidate's device subset (R25) as the allowed set of unpinned ops."""
    out = []
    for i in range(g.V):
        best = -1
        stack = [(i, g.w(i, pin, dset))]
        while stack:
            u, acc = stack.pop()
            if not g.succ[u]:
                best = max(best, acc)
            for (v, b) in g.succ[u]:
                stack.append((v, acc + g.c(u, v, b, pin, dset) + g.w(v, pin, dset)))
        out.append(best)
    return out


def evaluate(g: G, place, order):
    """APPEND evaluator: process ops in `order`, op i on place[i];
    ST = max(avail[d], max_pred FT + comm), FT = ST + cost."""
    avail = [0] * g.G
    ST, FT = {}, {}
    for i in order:
        d = place[i]
        st = avail[d]
        for (p, b) in g.pred[i]:
            st = max(st, FT[p] + g.comm(b, place[p], d))
        ST[i] = st
        FT[i] = st + g.cost[i][d]
        avail[d] = FT[i]
    return ST, FT, (max(FT.values()) if FT else 0)


def topo_orders(g: G, limit=None):
    indeg = [len(g.pred[i]) for i in range(g.V)]
    res = []

    def rec(cur, indeg):
        if limit is not None and len(res) >= limit:
            return
        if len(cur) == g.V:
            res.append(list(cur))
            return
        for i in range(g.V):
            if indeg[i] == 0 and i not in cur:
                cur.append(i)
                for (v, _) in g.succ[i]:
                    indeg[v] -= 1
                rec(cur, indeg)
                for (v, _) in g.succ[i]:
                    indeg[v] += 1
                cur.pop()

    rec([], indeg)
    return res


def brute_force_opt(g: G, zero_comm=False, dset=None):
    """Optimum of the APPEND schedule space: all placements x all
    topological orders (every left-shifted schedule is one of these);
    dset restricts the placements to a device subset (R25)."""
    orders = topo_orders(g)
    best = INF
    saved = (g.alpha, g.beta)
    if zero_comm:
        g.alpha = [0] * len(g.alpha)
        g.beta = [0] * len(g.beta)
    try:
        for place in itertools.product([d for d in range(g.G) if dset is None or d in dset], repeat=g.V):
            for o in orders:
                best = min(best, evaluate(g, place, o)[2])
    finally:
        g.alpha, g.beta = saved
    return best


def count_topo_orders(g: G, cap=100000):
    return len(topo_orders(g, limit=cap))


def check_invariants(g: G, res, pin=None):
    """SURVEY P5 on an oracle result dict (feasible candidates only)."""
    V = g.V
    place = res["placement"][:V].tolist()
    start = res["start"][:V].tolist()
    order = [x for x in res["order"][:V].tolist() if x >= 0]
    fin = {i: start[i] + g.cost[i][place[i]] for i in range(V)}
    ms = res["makespan"]
    assert sorted(order) == list(range(V)), "each op exactly once"
    assert ms == max(fin.values()) if V else ms == 0
    if g.G == 1:
        assert ms == sum(g.cost[i][0] for i in range(V)), "G=1 -> makespan = sum of costs"
    # makespan >= longest path with min-over-allowed costs and zero comm
    lp = [0] * V
    for i in reversed(range(V)):  # ids are not topo in general: do a proper DP
        pass
    memo = {}

    def longest(i):
        if i in memo:
            return memo[i]
        c = g.cost[i][pin[i]] if pin and i in pin else min(g.cost[i])
        v = c + max([longest(j) for (j, _) in g.succ[i]] or [0])
        memo[i] = v
        return v

    import sys
    sys.setrecursionlimit(100000)
    assert ms >= max([longest(i) for i in range(V)] or [0]), "makespan >= critical path"
    busy = sum(g.cost[i][place[i]] for i in range(V))
    assert ms * g.G >= busy, "makespan >= total work / G"
    assert ms * g.G >= sum(min(r) for r in g.cost), "makespan >= sum min cost / G"
    for (s, d), (b, p) in g.edges.items():
        assert start[d] >= fin[s] + g.comm(b, place[s], place[d]), "edge precedence + transfer"
    for dev in range(g.G):
        iv = sorted((start[i], fin[i], i) for i in range(V) if place[i] == dev)
        for a, b in zip(iv, iv[1:]):
            assert b[0] >= a[1], "no overlap on a device"
        used = sum(g.mem[i] for i in range(V) if place[i] == dev)
        assert used == int(res["peak_mem"][dev])
        assert used <= g.cap[dev], "memory cap"
    pos = {op: k for k, op in enumerate(order)}
    for (s, d) in g.edges:
        assert pos[s] < pos[d], "order A is topological"
    if pin:
        for i, d in pin.items():
            assert place[i] == d


def est_insert(ops, r, w):
    """INSERT (R1i) by brute force over time.  ops = [(ST, FT)] of
    the ops already on the device (zero-length included).  t is feasible iff
    t is at or after the end of every op (the open-ended slot), or the op
    [t, t+w] conflicts with none of them (w > 0: no overlap with any [s, f),
    a zero-length op p counting as an obstacle when t < p < t+w; w = 0: t not
    strictly inside any op) and, for w = 0, the device is idle just before or
    just after t (t touches an idle slot of positive length; zero-length ops
    at t do not count).  The earliest feasible t is r or the end of some op."""
    last = max([f for (_, f) in ops] + [0])
    for t in sorted({r} | {f for (_, f) in ops if f >= r}):
        if t >= last:
            return t
        if w > 0:
            if not any(s < t + w and t < f for (s, f) in ops):
                return t
            continue
        if any(s < t < f for (s, f) in ops):
            continue
        left_idle = t > 0 and not any(s < t <= f for (s, f) in ops)
        right_idle = not any(s <= t < f for (s, f) in ops)
        if left_idle or right_idle:
            return t
    raise AssertionError("unreachable: the open-ended slot always fits")


def live_usage(g: G, done, place, d):
    """Liveness memory (R24) by its definition, before the next step: the
    parameters of every op already dequeued on d, plus the output
    (mem - param) of every such op that still has a consumer not dequeued."""
    tot = 0
    for j in done:
        if place[j] != d:
            continue
        tot += g.param[j]
        if any(c not in done for (c, _) in g.succ[j]):
            tot += g.mem[j] - g.param[j]
    return tot


def live_peaks(g: G, res):
    """R24 peak per device by definition: the largest, over the steps t of the
    dequeue sequence, of the memory held on the device while step t's op is
    placed: parameters of every op dequeued at or before t, outputs of ops
    dequeued at or before t whose last consumer is dequeued at t or later,
    and the output of step t's op itself."""
    V = g.V
    deq = [x for x in res["dequeue"][:V].tolist() if x >= 0]
    place = res["placement"][:V].tolist()
    dq = {op: t for t, op in enumerate(deq)}
    peak = [0] * g.G
    for t, i in enumerate(deq):
        d = place[i]
        tot = 0
        for j in deq[: t + 1]:
            if place[j] != d:
                continue
            tot += g.param[j]
            last = max([dq[c] for (c, _) in g.succ[j]] or [dq[j]])
            if j == i or last >= t:
                tot += g.mem[j] - g.param[j]
        peak[d] = max(peak[d], tot)
    return peak


def check_greedy_steps(g: G, res, rank, cp_dev=None, insert=False, live=False, dset=None):
    """every dequeued op is the max-(rank, -id) ready op and every
    free op sits on a device of minimum EFT (ties: lowest id) among the
    memory-feasible ones, given the partial schedule.  insert=True: EST by
    est_insert (busy intervals of the ops placed so far) instead of APPEND.
    live=True: memory feasibility with the liveness usage of R24 (by
    definition, live_usage).  dset: the candidate's device subset (R25)."""
    V = g.V
    deq = [x for x in res["dequeue"][:V].tolist() if x >= 0]
    place = res["placement"][:V].tolist()
    start = res["start"][:V].tolist()
    devs = [d for d in range(g.G) if dset is None or d in dset]
    done = set()
    avail = [0] * g.G
    used = [0] * g.G
    reserved = [0] * g.G
    if cp_dev:
        for i, d in cp_dev.items():
            reserved[d] += g.mem[i]
    FT = {}
    busy = [[] for _ in range(g.G)]

    def est_on(i, d):
        r = max([0 if insert else avail[d]] + [FT[p] + g.comm(b, place[p], d) for (p, b) in g.pred[i]])
        return est_insert(busy[d], r, g.cost[i][d]) if insert else r

    for i in deq:
        ready = [j for j in range(V) if j not in done and all(p in done for (p, _) in g.pred[j])]
        best = max(ready, key=lambda j: (rank[j], -j))
        assert i == best, "dequeued op is the highest-priority ready op"
        if cp_dev and i in cp_dev:
            d = cp_dev[i]
            reserved[d] -= g.mem[i]
            est = est_on(i, d)
        else:
            effs = []
            for d in devs:
                u = live_usage(g, done, place, d) if live else used[d]
                if u + reserved[d] + g.mem[i] > g.cap[d]:
                    continue
                est = est_on(i, d)
                effs.append((est + g.cost[i][d], d, est))
            eft, d, est = min(effs)
            assert place[i] == d, "device of minimum EFT (lowest id on ties)"
        assert start[i] == est
        FT[i] = est + g.cost[i][d]
        avail[d] = FT[i]
        busy[d].append((est, FT[i]))
        used[d] += g.mem[i]
        done.add(i)
    assert len(done) == V
