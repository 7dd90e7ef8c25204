"""Pins of the CPU oracle against things other than itself:
hand-derived examples (tests/golden), brute force, closed forms, invariants,
an independent greedy-step replay checker, Theorem 1 and published PRNG
outputs.  CPU only."""
import json
import os

import numpy as np
import pytest

import oracle as O
import refcheck as RC
from paper_conf_middleware_0001lmwlwyl20_b200 import synth

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def gold(name):
    with open(os.path.join(GOLD, name)) as f:
        return json.load(f)


def mk(V, G, edges, cost, mem=None, cap=None, smask=None, link=(0, 1_000_000), eparam=None, copy_fs=0):
    cost = np.asarray(cost, np.int64)
    if cost.ndim == 1:
        cost = np.repeat(cost[:, None], G, axis=1)
    src = [e[0] for e in edges]
    dst = [e[1] for e in edges]
    byt = [e[2] for e in edges]
    return synth._finish("t", G, src, dst, byt, eparam or [0] * len(edges), cost, mem or [0] * V, [0] * V,
                         smask or [0] * V, cap=cap, link=link, copy_fs=copy_fs)


# ------------------------------------------------------------ golden (P1-P3)

def test_a1_diamond_golden():
    gd = gold("a1_diamond.json")
    desc = synth.diamond()
    g = O.OracleGraph(desc)
    assert g.rank()[:4].tolist() == gd["rank"]
    assert g.critical_path().tolist() == gd["critical_path"]
    r = g.schedule(flags=O.F_CP_PIN)
    assert r["makespan"] == gd["cp_pin"]["makespan"]
    assert r["placement"][:4].tolist() == gd["cp_pin"]["placement"]
    assert r["start"][:4].tolist() == gd["cp_pin"]["start"]
    assert r["order"][:4].tolist() == gd["cp_pin"]["order"]
    r = g.schedule(flags=0)
    assert r["makespan"] == gd["pure_eft"]["makespan"]
    assert r["placement"][:4].tolist() == gd["pure_eft"]["placement"]
    assert r["start"][:4].tolist() == gd["pure_eft"]["start"]
    # independent re-derivation: path enumeration and brute force
    rg = RC.G(desc)
    assert RC.rank_by_paths(rg) == gd["rank"]
    assert RC.brute_force_opt(rg) == gd["brute_force_opt"]
    assert RC.brute_force_opt(rg, zero_comm=True) == gd["theorem1"]["opt_nocomm"]


def test_a2_split_chain_golden():
    gd = gold("a2_split_chain.json")
    g = O.OracleGraph(synth.split_chain())
    assert g.schedule(flags=O.F_CP_PIN)["makespan"] == gd["base_makespan"]
    s = gd["split"]
    c = O.make_cand(O.KIND_SPLIT, split=(s["op"], s["dim"], s["n"]))
    for flags in (0, O.F_CP_PIN):
        r = g.schedule(c, flags=flags)
        assert r["makespan"] == s["makespan"]
    r = g.schedule(c, flags=O.F_CP_PIN)
    V = s["V"]
    assert r["rank"][:V].tolist() == s["rank"]
    assert r["placement"][:V].tolist() == s["placement"]
    assert r["start"][:V].tolist() == s["start"]
    ss = g.split_search(flags=O.F_CP_PIN)
    assert [list(x) for x in ss["sp"]] == gd["split_search"]["sp"]
    assert ss["makespan"] == gd["split_search"]["makespan"]
    # closed form 1 + ceil(100/n) + 1 for both n (G=2 only allows n=2)
    assert s["makespan"] == 1 + -(-100 // 2) + 1


def test_a3_append_golden():
    gd = gold("a3_append_vs_insert.json")
    g = O.OracleGraph(synth.append_vs_insert())
    c = O.make_cand(O.KIND_PIN, pins=[(1, 1)])
    r = g.schedule(c, flags=O.F_CP_PIN)
    assert g.rank(c)[:3].tolist() == gd["rank"]
    assert r["makespan"] == gd["append"]["makespan"]
    assert r["placement"][:3].tolist() == gd["append"]["placement"]
    assert r["start"][:3].tolist() == gd["append"]["start"]


def test_a3_insert_golden():
    gd = gold("a3_append_vs_insert.json")
    g = O.OracleGraph(synth.append_vs_insert())
    c = O.make_cand(O.KIND_PIN, pins=[(1, 1)])
    r = g.schedule(c, flags=O.F_CP_PIN | O.F_POLICY_INSERT)
    assert r["makespan"] == gd["insert"]["makespan"]
    assert r["placement"][:3].tolist() == gd["insert"]["placement"]
    assert r["start"][:3].tolist() == gd["insert"]["start"]


# -------------------------------------------------------- closed forms (P3)

@pytest.mark.parametrize("flags", [0, O.F_CP_PIN, O.F_POLICY_INSERT, O.F_CP_PIN | O.F_POLICY_INSERT])
def test_single_device_is_sum_of_costs(flags):
    for seed in range(20):
        d = synth.random_dag(seed, G=1, caps="none")
        r = O.OracleGraph(d).schedule(flags=flags)
        assert r["makespan"] == int(d.cost[:, 0].sum())


@pytest.mark.parametrize("flags", [0, O.F_CP_PIN])
def test_independent_identical_ops_round_robin(flags):
    for V, G, c in [(7, 3, 5), (16, 4, 9), (5, 8, 3), (33, 8, 2)]:
        d = mk(V, G, [], [c] * V)
        r = O.OracleGraph(d).schedule(flags=flags)
        assert r["makespan"] == -(-V // G) * c
        if flags == 0:
            assert r["placement"][:V].tolist() == [i % G for i in range(V)]


@pytest.mark.parametrize("flags", [0, O.F_CP_PIN])
def test_chain_with_comm_stays_on_device0(flags):
    V = 12
    d = mk(V, 4, [(i, i + 1, 100 + i) for i in range(V - 1)], list(range(1, V + 1)))
    r = O.OracleGraph(d).schedule(flags=flags)
    assert r["makespan"] == sum(range(1, V + 1))
    assert set(r["placement"][:V].tolist()) == {0}


def test_cp_memory_handoff_prefix_first():
    """P2: a CP whose memory exceeds cap[0] spans two devices, prefix first."""
    V = 4
    d = mk(V, 2, [(i, i + 1, 1) for i in range(V - 1)], [10] * V, mem=[10] * V, cap=[25, 100])
    r = O.OracleGraph(d).schedule(flags=O.F_CP_PIN)
    assert r["placement"][:V].tolist() == [0, 0, 1, 1]
    assert r["peak_mem"].tolist() == [20, 20]


def test_cp_device_heterogeneous_average():
    """P2: the CP device is the one with the smallest average CP cost."""
    V = 3
    cost = np.array([[10, 6], [10, 6], [10, 6]], np.int64)
    d = mk(V, 2, [(0, 1, 1000), (1, 2, 1000)], cost)
    r = O.OracleGraph(d).schedule(flags=O.F_CP_PIN)
    assert r["placement"][:V].tolist() == [1, 1, 1]
    assert r["makespan"] == 18


# --------------------------------------------------- brute force (P1, P3, P4)

def _small_dags(n, maxV=7, maxG=3):
    out = []
    seed = 1000
    while len(out) < n:
        seed += 1
        rng = np.random.default_rng(seed)
        V = int(rng.integers(1, maxV + 1))
        G = int(rng.integers(1, maxG + 1))
        d = synth.random_dag(seed, V=V, G=G, max_in=2, caps="none")
        rg = RC.G(d)
        if RC.count_topo_orders(rg, cap=400) * G ** V > 60000:
            continue
        out.append((d, rg))
    return out


SMALL = _small_dags(40)


@pytest.mark.parametrize("k", range(len(SMALL)))
def test_small_dag_vs_brute_force(k):
    d, rg = SMALL[k]
    g = O.OracleGraph(d)
    assert g.rank()[: d.n_ops].tolist() == RC.rank_by_paths(rg)
    opt = RC.brute_force_opt(rg)
    for flags in (0, O.F_CP_PIN):
        r = g.schedule(flags=flags)
        assert r["status"] == O.CAND_OK
        # (i) the independent evaluator replays (placement, order A) exactly
        order = [x for x in r["order"][: d.n_ops].tolist() if x >= 0]
        ST, FT, ms = RC.evaluate(rg, r["placement"][: d.n_ops].tolist(), order)
        assert ms == r["makespan"]
        assert [ST[i] for i in range(d.n_ops)] == r["start"][: d.n_ops].tolist()
        # (ii) the heuristic never beats the optimum of its schedule space
        assert opt <= r["makespan"]
        RC.check_invariants(rg, r)
    RC.check_greedy_steps(rg, g.schedule(flags=0), RC.rank_by_paths(rg))


@pytest.mark.parametrize("k", range(len(SMALL)))
def test_small_dag_insert_vs_brute_force(k):
    """INSERT (R1i): the schedule is valid (invariants), never beats the
    optimum over all placements x orders, and every step is the brute-force
    greedy choice (EST by exhaustive search over time, refcheck.est_insert)."""
    d, rg = SMALL[k]
    g = O.OracleGraph(d)
    opt = RC.brute_force_opt(rg)
    for flags in (O.F_POLICY_INSERT, O.F_POLICY_INSERT | O.F_CP_PIN):
        r = g.schedule(flags=flags)
        assert r["status"] == O.CAND_OK
        assert opt <= r["makespan"]
        RC.check_invariants(rg, r)
    RC.check_greedy_steps(rg, g.schedule(flags=O.F_POLICY_INSERT), RC.rank_by_paths(rg), insert=True)


@pytest.mark.parametrize("k", range(0, len(SMALL), 3))
def test_small_dag_pinned_ranks(k):
    d, rg = SMALL[k]
    if d.n_devices < 2:
        return
    rng = np.random.default_rng(k)
    g = O.OracleGraph(d)
    for _ in range(5):
        npin = int(rng.integers(1, min(4, d.n_ops) + 1))
        ops = rng.choice(d.n_ops, npin, replace=False).tolist()
        pins = [(o, int(rng.integers(0, d.n_devices))) for o in ops]
        c = O.make_cand(O.KIND_PIN, pins=pins)
        pin = dict(pins)
        assert g.rank(c)[: d.n_ops].tolist() == RC.rank_by_paths(rg, pin)
        r = g.schedule(c, flags=0)
        RC.check_invariants(rg, r, pin)


def test_theorem1_bound():
    """P10 / Theorem 1: makespan <= 2*OPT_nocomm + C_max with
    sufficient memory, CP pinning off and homogeneous costs (R20)."""
    checked = 0
    seed = 5000
    while checked < 25:
        seed += 1
        rng = np.random.default_rng(seed)
        V = int(rng.integers(2, 7))
        G = int(rng.integers(2, 4))
        d = synth.random_dag(seed, V=V, G=G, max_in=2, caps="none", homogeneous=True, K=1)
        rg = RC.G(d)
        if RC.count_topo_orders(rg, cap=400) * G ** V > 40000:
            continue
        ms = O.OracleGraph(d).schedule(flags=0)["makespan"]
        opt0 = RC.brute_force_opt(rg, zero_comm=True)
        memo = {}

        def cmax(i):
            if i not in memo:
                memo[i] = max([rg.c(i, j, b) + cmax(j) for (j, b) in rg.succ[i]] or [0])
            return memo[i]

        c_max = max(cmax(i) for i in range(V))
        assert ms <= 2 * opt0 + c_max
        checked += 1


# ---------------------------------------------- invariants at medium size (P5, P6)

@pytest.mark.parametrize("seed", range(30))
def test_random_dag_invariants_and_greedy_replay(seed):
    d = synth.random_dag(seed + 77)
    g = O.OracleGraph(d)
    rg = RC.G(d)
    rng = np.random.default_rng(seed)
    for flags in (0, O.F_CP_PIN):
        r = g.schedule(flags=flags)
        if r["status"] == O.CAND_OK:
            RC.check_invariants(rg, r)
        else:
            assert r["makespan"] == O.INF and (r["peak_mem"] == -1).all()
    r = g.schedule(flags=0)
    if r["status"] == O.CAND_OK:
        RC.check_greedy_steps(rg, r, g.rank()[: d.n_ops].tolist())
    # INSERT policy (R1i): same checks, EST by brute force over time
    r = g.schedule(flags=O.F_POLICY_INSERT)
    if r["status"] == O.CAND_OK:
        RC.check_invariants(rg, r)
        RC.check_greedy_steps(rg, r, g.rank()[: d.n_ops].tolist(), insert=True)
    if d.n_devices > 1 and d.n_ops > 0:
        for _ in range(3):
            npin = int(rng.integers(1, min(4, d.n_ops) + 1))
            ops = rng.choice(d.n_ops, npin, replace=False).tolist()
            pins = [(o, int(rng.integers(0, d.n_devices))) for o in ops]
            r = g.schedule(O.make_cand(O.KIND_PIN, pins=pins), flags=O.F_CP_PIN)
            if r["status"] == O.CAND_OK:
                RC.check_invariants(rg, r, dict(pins))


# ------------------------------------------------------------ splits (P7, P8)

@pytest.mark.parametrize("seed", range(12))
def test_split_operation_properties(seed):
    d = synth.random_dag(seed + 300, caps="none")
    if d.n_devices < 2:
        return
    g = O.OracleGraph(d)
    rg = RC.G(d)
    ops = [i for i in range(d.n_ops) if d.split_mask[i]]
    for op in ops[:4]:
        for dim in (0, 1):
            if not d.split_mask[op] & (1 << dim):
                continue
            n = d.n_devices
            x = g.split_export(op, dim, n)
            P, S = len(rg.pred[op]), len(rg.succ[op])
            V2 = x["V"]
            assert V2 == d.n_ops + P + n + S
            assert int(x["alive"].sum()) == d.n_ops - 1 + P + n + S
            assert not x["alive"][op]
            src, dst, byt = x["src"], x["dst"], x["bytes"]
            assert not ((src == op) | (dst == op)).any()
            sp = list(range(d.n_ops, d.n_ops + P))
            subs = list(range(d.n_ops + P, d.n_ops + P + n))
            cons = list(range(d.n_ops + P + n, V2))
            for a, (pre, b) in enumerate(rg.pred[op]):          # pred order, full bytes in
                into = byt[(dst == sp[a])]
                assert src[dst == sp[a]].tolist() == [pre] and into.tolist() == [b]
                outs = byt[src == sp[a]]
                assert len(outs) == n
                assert int(outs.sum()) in (b, n * b)             # cut (sum = b) or replicated
            for a, (suc, b) in enumerate(rg.succ[op]):
                ins = byt[dst == cons[a]]
                assert len(ins) == n and int(ins.sum()) == b     # partitions sum to the tensor
                assert src[src == cons[a]].size == 1 and dst[src == cons[a]].tolist() == [suc]
            for k, s in enumerate(subs):
                c = x["cost"][s]
                assert (c * n >= d.cost[op]).all() and (c * n < d.cost[op] + n).all()
            act = int(d.mem[op] - d.param[op])
            assert int(x["mem"][subs].sum()) == act + (n * int(d.param[op]) if dim == 0 else int(d.param[op]))
            assert int(x["param"][subs].sum()) == (n * int(d.param[op]) if dim == 0 else int(d.param[op]))
            # the split graph is a DAG: loading it back into the oracle succeeds
            sd = synth._finish("s", d.n_devices, src, dst, byt, x["eparam"], x["cost"], x["mem"], x["param"],
                               np.zeros(V2, np.uint8), cap=None, classes=(d.link_class, d.alpha, d.beta))
            O.OracleGraph(sd)


def _placed_cp(d, place):
    """The placement-aware critical path of R15 (Alg. 2 lines 4-5), recomputed
    here independently of the oracle: longest cost+comm path under `place`,
    ties to the lower id."""
    rg = RC.G(d)
    memo = {}

    def rk(i):
        if i not in memo:
            memo[i] = d.cost[i][place[i]] + max([rg.comm(b, place[i], place[j]) + rk(j) for (j, b) in rg.succ[i]]
                                                or [0])
        return memo[i]

    srcs = [i for i in range(d.n_ops) if not rg.pred[i]]
    cur = max(srcs, key=lambda i: (rk(i), -i))
    cp = [cur]
    while rg.succ[cur]:
        cur = max([j for (j, _) in rg.succ[cur]], key=lambda j: (rk(j), -j))
        cp.append(cur)
    return cp


@pytest.mark.parametrize("seed", range(8))
def test_split_search_monotone(seed):
    d = synth.random_dag(seed + 900, V=60, G=4, caps="none")
    g = O.OracleGraph(d)
    base = g.schedule(flags=O.F_CP_PIN)
    ss = g.split_search(flags=O.F_CP_PIN)
    assert ss["makespan"] <= base["makespan"]
    if ss["sp"]:
        assert ss["makespan"] < base["makespan"]
    # SP ops come from the placement-aware CP of the initial DPOS (R15)
    cp = _placed_cp(d, base["placement"][: d.n_ops].tolist())
    for (op, dim, n) in ss["sp"]:
        assert op in cp and d.split_mask[op] & (1 << dim) and 2 <= n <= d.n_devices


# ------------------------------------- best-improvement split search (NEXT N2)

def test_split_search_best_a2_golden():
    """A.2: X is the only splittable op and G=2 allows only n=2, so both
    searches accept exactly that split (golden a2 "split_search")."""
    gd = gold("a2_split_chain.json")
    ss = O.OracleGraph(synth.split_chain()).split_search(flags=O.F_CP_PIN, best_improvement=True)
    assert [list(x) for x in ss["sp"]] == gd["split_search"]["sp"]
    assert ss["makespan"] == gd["split_search"]["makespan"]


# seeds where the best-improvement search differs from Alg. 2 or splits twice
BI_SEEDS = [4, 13, 21, 32, 34, 39, 116, 122, 214, 1, 3]


@pytest.mark.parametrize("seed", BI_SEEDS)
def test_split_search_best_first_round_is_brute_force_min(seed):
    """Round 1 of the best-improvement search is the minimum over every single
    split of every split-eligible CP op of G0 (brute force through SPLIT
    candidates); later rounds only lower the makespan; no op is split twice;
    the emitted schedule respects every surviving original edge."""
    d = synth.random_dag(seed, V=40, G=4, caps="none", max_in=2)
    g = O.OracleGraph(d)
    rg = RC.G(d)
    base = g.schedule(flags=O.F_CP_PIN)
    bi = g.split_search(flags=O.F_CP_PIN, best_improvement=True)
    cp = _placed_cp(d, base["placement"][: d.n_ops].tolist())
    singles = {}
    for op in cp:
        for dim in (0, 1):
            if d.split_mask[op] & (1 << dim):
                for n in range(2, d.n_devices + 1):
                    r = g.schedule(O.make_cand(O.KIND_SPLIT, split=(op, dim, n)), flags=O.F_CP_PIN)
                    if r["status"] == O.CAND_OK:
                        singles[(op, dim, n)] = r["makespan"]
    m1 = min(singles.values(), default=None)
    if m1 is not None and m1 < base["makespan"]:
        assert bi["sp"] and singles[tuple(bi["sp"][0])] == m1
        assert bi["makespan"] <= m1 < base["makespan"]
    else:
        assert bi["sp"] == [] and bi["makespan"] == base["makespan"]
    ops = [x[0] for x in bi["sp"]]
    assert len(set(ops)) == len(ops) and set(ops) <= set(cp)
    split = set(ops)
    place, start = bi["placement"], bi["start"]
    for i in range(d.n_ops):
        if i in split:
            assert place[i] == 0xFF and start[i] == -1
            continue
        fi = start[i] + d.cost[i][place[i]]
        assert 0 <= start[i] and fi <= bi["makespan"]
        for (j, b) in rg.succ[i]:
            if j not in split:
                assert start[j] >= fi + rg.comm(b, place[i], place[j])


# ------------------------------------------------------ memory / statuses

def test_infeasible_and_badspec():
    d = mk(3, 2, [(0, 1, 1), (1, 2, 1)], [5, 5, 5], mem=[10, 10, 10], cap=[25, 15])
    g = O.OracleGraph(d)
    r = g.schedule(flags=0)
    # op2 no longer fits next to ops 0,1 on device 0 (R8) and moves to device 1
    assert r["status"] == O.CAND_OK and r["peak_mem"].tolist() == [20, 10]
    assert r["placement"][:3].tolist() == [0, 0, 1] and r["makespan"] == 5 + 5 + 1 + 5
    d2 = mk(3, 2, [(0, 1, 1), (1, 2, 1)], [5, 5, 5], mem=[10, 10, 10], cap=[12, 12])
    r = O.OracleGraph(d2).schedule(flags=0)
    assert r["status"] == O.CAND_INFEASIBLE and r["makespan"] == O.INF
    r = g.schedule(O.make_cand(O.KIND_PIN, pins=[(0, 1), (1, 1)]), flags=0)
    assert r["status"] == O.CAND_INFEASIBLE
    for c in [O.make_cand(O.KIND_PIN, pins=[(0, 2)]), O.make_cand(O.KIND_PIN, pins=[(0, 1), (0, 0)]),
              O.make_cand(O.KIND_PIN, pins=[(7, 0)]), O.make_cand(O.KIND_SPLIT, split=(1, 0, 2)),
              O.make_cand(7)]:
        r = g.schedule(c, flags=0)
        assert r["status"] == O.CAND_BADSPEC and r["makespan"] == O.INF


def test_load_errors_and_empty_graph():
    with pytest.raises(O.OracleError) as e:
        O.OracleGraph(mk(3, 2, [(0, 1, 1), (1, 2, 1), (2, 0, 1)], [1, 1, 1]))
    assert e.value.code == -2
    with pytest.raises(O.OracleError) as e:
        O.OracleGraph(mk(2, 2, [(0, 0, 1)], [1, 1]))
    assert e.value.code == -2
    with pytest.raises(O.OracleError) as e:
        O.OracleGraph(mk(2, 2, [(0, 1, 1)], [1, -1]))
    assert e.value.code == -1
    # bytes * split_copy_fs_per_byte (R13) and merged parallel-edge bytes (R11) must stay in int64
    with pytest.raises(O.OracleError) as e:
        O.OracleGraph(mk(2, 2, [(0, 1, 1 << 40)], [1, 1], link=(0, 0), copy_fs=1 << 22))
    assert e.value.code == -5
    with pytest.raises(O.OracleError) as e:
        O.OracleGraph(mk(2, 2, [(0, 1, 1 << 61), (0, 1, 1 << 61)], [1, 1], link=(0, 0)))
    assert e.value.code == -5
    r = O.OracleGraph(mk(0, 2, [], np.zeros((0, 2), np.int64))).schedule(flags=O.F_CP_PIN)
    assert r["makespan"] == 0 and r["status"] == O.CAND_OK


def test_parallel_edges_merge():
    """R11: parallel edges behave as one edge carrying the summed bytes."""
    a = mk(3, 2, [(0, 1, 30), (0, 1, 20), (1, 2, 5), (0, 2, 1)], [5, 5, 5])
    b = mk(3, 2, [(0, 1, 50), (1, 2, 5), (0, 2, 1)], [5, 5, 5])
    for flags in (0, 1):
        ra, rb = O.OracleGraph(a).schedule(flags=flags), O.OracleGraph(b).schedule(flags=flags)
        assert ra["makespan"] == rb["makespan"]
        assert (ra["start"] == rb["start"]).all()


# ------------------------------------------------------- generator (R21, P11)

def test_splitmix64_published_outputs():
    """splitmix64 (Steele, Lea, Flood 2014; Vigna's reference splitmix64.c):
    from state 0 the first outputs are 0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4."""
    v1, s = O.splitmix64_next(0)
    v2, s = O.splitmix64_next(s)
    assert v1 == 0xE220A8397B1DCDAF and v2 == 0x6E789E6AA1B965F4


def test_candidate_stream_properties():
    d = synth.config("C1")
    g = O.OracleGraph(d)
    n_split, base_place = g.stream_info(flags=O.F_CP_PIN)
    base = g.schedule(flags=O.F_CP_PIN)
    assert (base_place == base["placement"][: d.n_ops]).all()
    cs = g.generate(seed=123, first=0, n=n_split + 500, kmin=1, kmax=4, flags=O.F_CP_PIN)
    assert cs[0]["kind"] == O.KIND_BASE
    sp = cs[1 : n_split + 1]
    assert (sp["kind"] == O.KIND_SPLIT).all()
    keys = [(int(c["split_op"]), int(c["split_dim"]), int(c["split_n"])) for c in sp]
    assert len(set(keys)) == len(keys)
    for c in cs[n_split + 1 :]:
        assert c["kind"] == O.KIND_PIN and 1 <= c["n_pins"] <= 4
        ops = c["pin_op"][: c["n_pins"]].tolist()
        assert len(set(ops)) == len(ops)
        for o, dv in zip(ops, c["pin_dev"][: c["n_pins"]].tolist()):
            assert dv != base_place[o] and 0 <= dv < d.n_devices
    # index-addressable: a window equals the same slice of a longer run
    w = g.generate(seed=123, first=n_split + 100, n=50, flags=O.F_CP_PIN)
    assert w.tobytes() == cs[n_split + 100 : n_split + 150].tobytes()
    # the sweep's best equals the argmin over per-candidate makespans
    sw = g.sweep(seed=123, first=0, n=400, flags=O.F_CP_PIN, per_candidate=True)
    m = sw["makespans"]
    assert sw["makespan"] == m.min() and sw["index"] == int(np.argmin(m))
