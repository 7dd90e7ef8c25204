"""Pins of the oracle's NEXT-row N3 features against things
other than itself.  CPU only.

* R24 liveness memory (FASTT_F_MEM_LIVE): a hand-derived chain, the chain's
  closed form, peaks re-derived from the live-set definition on random DAGs
  (refcheck.live_peaks), the greedy-step replay with liveness feasibility,
  the reduction to the static model when every op's memory is parameters,
  and "no caps -> the schedule is the static one".
* R25 device subsets (dev_mask): a one-device subset is the
  G = 1 closed form on that device; a subset M reduces exactly to the full
  oracle on the graph restricted to M; ranks by path enumeration with the
  subset as the allowed set; brute force over placements inside M; the
  greedy-step replay restricted to M; validation (BADSPEC) and the stream's
  subset block.
"""
import numpy as np
import pytest

import oracle as O
import refcheck as RC
from paper_conf_middleware_0001lmwlwyl20_b200 import synth

INT64_MAX = np.iinfo(np.int64).max


def chain(mem, param, cost=None, G=1, cap=None):
    V = len(mem)
    cost = cost or [10] * V
    edges = [(i, i + 1, 8) for i in range(V - 1)]
    return synth._finish("chain", G, [e[0] for e in edges], [e[1] for e in edges], [e[2] for e in edges],
                         [0] * len(edges), np.repeat(np.asarray(cost, np.int64)[:, None], G, axis=1), mem, param,
                         [0] * V, cap=cap)


# ------------------------------------------------------------- R24 liveness

def test_live_hand_chain():
    """A -> B -> C on one device, mem (10, 20, 30), param (0, 5, 0), by hand:
    step A: live 10; step B: 10 + 20 = 30, then A's output (10) is freed -> 20;
    step C: 20 + 30 = 50, then B's output (15) -> 35, C is a sink -> 5.
    Peak 50 (the static model holds 60)."""
    g = O.OracleGraph(chain([10, 20, 30], [0, 5, 0]))
    assert g.schedule(flags=O.F_MEM_LIVE)["peak_mem"].tolist() == [50]
    assert g.schedule(flags=0)["peak_mem"].tolist() == [60]
    # a cap of 50 fits only under liveness
    g = O.OracleGraph(chain([10, 20, 30], [0, 5, 0], cap=[50]))
    assert g.schedule(flags=O.F_MEM_LIVE)["status"] == O.CAND_OK
    assert g.schedule(flags=0)["status"] == O.CAND_INFEASIBLE
    g = O.OracleGraph(chain([10, 20, 30], [0, 5, 0], cap=[49]))
    assert g.schedule(flags=O.F_MEM_LIVE)["status"] == O.CAND_INFEASIBLE


@pytest.mark.parametrize("seed", range(8))
def test_live_chain_closed_form(seed):
    """Chain on one device: at step i the device holds the parameters of ops
    0..i plus the outputs of ops i-1 and i, so the peak is
    max_i (sum_{j<=i} param_j + act_{i-1} + act_i)."""
    rng = np.random.default_rng(seed)
    V = int(rng.integers(1, 30))
    mem = rng.integers(0, 1000, V)
    param = (mem * rng.random(V)).astype(np.int64) * (rng.random(V) < 0.4)
    act = mem - param
    g = O.OracleGraph(chain(mem.tolist(), param.tolist()))
    want = max(int(param[: i + 1].sum()) + (int(act[i - 1]) if i else 0) + int(act[i]) for i in range(V))
    r = g.schedule(flags=O.F_MEM_LIVE)
    assert r["peak_mem"].tolist() == [want]


@pytest.mark.parametrize("seed", range(40))
def test_live_peaks_and_replay_random(seed):
    """Random DAGs (random caps, some infeasible): peaks equal the live-set
    definition; every step is the greedy choice with liveness feasibility;
    an infeasible result is infeasible in the replay too."""
    desc = synth.random_dag(5000 + seed, V=int(np.random.default_rng(seed).integers(2, 40)))
    g = O.OracleGraph(desc)
    rg = RC.G(desc)
    for flags in (O.F_MEM_LIVE, O.F_MEM_LIVE | O.F_CP_PIN):
        r = g.schedule(flags=flags)
        if r["status"] != O.CAND_OK:
            assert r["status"] == O.CAND_INFEASIBLE and r["makespan"] == INT64_MAX
            continue
        assert r["peak_mem"].tolist() == RC.live_peaks(rg, r)
        for d in range(desc.n_devices):
            assert r["peak_mem"][d] <= desc.cap[d]
        if not flags & O.F_CP_PIN:
            RC.check_greedy_steps(rg, r, g.rank().tolist(), live=True)


@pytest.mark.parametrize("seed", range(20))
def test_live_infeasible_replay(seed):
    """Where the liveness oracle reports INFEASIBLE (no CP pins), the greedy
    replay of the dequeue order reaches an op that fits on no device."""
    desc = synth.random_dag(7000 + seed, V=25, caps="none")
    tot = int(desc.mem.sum())
    desc.cap[:] = max(1, tot // (3 * desc.n_devices))
    g = O.OracleGraph(desc)
    r = g.schedule(flags=O.F_MEM_LIVE)
    if r["status"] == O.CAND_OK:
        RC.check_greedy_steps(RC.G(desc), r, g.rank().tolist(), live=True)
        return
    # replay with the live-set usage until no device fits
    rg = RC.G(desc)
    rank = g.rank().tolist()
    done, place, avail, FT = set(), {}, [0] * rg.G, {}
    while len(done) < rg.V:
        ready = [j for j in range(rg.V) if j not in done and all(p in done for (p, _) in rg.pred[j])]
        i = max(ready, key=lambda j: (rank[j], -j))
        effs = []
        for d in range(rg.G):
            if RC.live_usage(rg, done, place, d) + rg.mem[i] > rg.cap[d]:
                continue
            est = max([avail[d]] + [FT[p] + rg.comm(b, place[p], d) for (p, b) in rg.pred[i]])
            effs.append((est + rg.cost[i][d], d))
        if not effs:
            return  # infeasible here, as the oracle says
        eft, d = min(effs)
        place[i], FT[i], avail[d] = d, eft, eft
        done.add(i)
    raise AssertionError("the replay found a feasible schedule the oracle called infeasible")


@pytest.mark.parametrize("seed", range(15))
def test_live_reduces_to_static_when_all_parameters(seed):
    """mem == param for every op: nothing is ever freed, so the liveness model
    is the static model R8 (same status, makespan, placement, peaks)."""
    desc = synth.random_dag(9000 + seed, V=60)
    desc.param[:] = desc.mem
    g = O.OracleGraph(desc)
    for flags in (0, O.F_CP_PIN):
        a = g.schedule(flags=flags)
        b = g.schedule(flags=flags | O.F_MEM_LIVE)
        assert a["status"] == b["status"] and a["makespan"] == b["makespan"]
        assert (a["peak_mem"] == b["peak_mem"]).all()
        assert (a["placement"] == b["placement"]).all()


@pytest.mark.parametrize("seed", range(15))
def test_live_without_caps_keeps_the_schedule(seed):
    """Unlimited memory: feasibility never binds, so the schedule is the
    static model's and only the peaks change (live peak <= static peak)."""
    desc = synth.random_dag(11000 + seed, V=80, caps="none")
    g = O.OracleGraph(desc)
    for flags in (0, O.F_CP_PIN, O.F_POLICY_INSERT):
        a = g.schedule(flags=flags)
        b = g.schedule(flags=flags | O.F_MEM_LIVE)
        assert a["makespan"] == b["makespan"]
        assert (a["placement"] == b["placement"]).all() and (a["start"] == b["start"]).all()
        assert (b["peak_mem"] <= a["peak_mem"]).all()


# -------------------------------------------------------------- R25 subsets

def restrict(desc, devs):
    """The same problem on the devices `devs` only (order kept)."""
    devs = list(devs)
    G2 = len(devs)
    lc = desc.link_class[np.ix_(devs, devs)]
    return synth._finish("restricted", G2, desc.src, desc.dst, desc.bytes, desc.eparam, desc.cost[:, devs],
                         desc.mem, desc.param, desc.split_mask, cap=desc.cap[devs],
                         classes=(lc, desc.alpha, desc.beta), copy_fs=desc.copy_fs)


def mask_of(devs):
    return int(sum(1 << d for d in devs))


@pytest.mark.parametrize("seed", range(30))
def test_subset_reduces_to_restricted_graph(seed):
    """A candidate restricted to devices M schedules exactly like the full
    oracle on the graph that only has the devices of M (ranks, CP devices and
    the EFT argmin all range over M in the same order)."""
    rng = np.random.default_rng(seed)
    desc = synth.random_dag(13000 + seed, G=int(rng.integers(2, 7)))
    G = desc.n_devices
    k = int(rng.integers(1, G + 1))
    devs = sorted(rng.choice(G, size=k, replace=False).tolist())
    g = O.OracleGraph(desc)
    h = O.OracleGraph(restrict(desc, devs))
    V = desc.n_ops
    pins = []
    if V >= 2 and rng.random() < 0.5:
        pins = [(int(rng.integers(0, V)), int(rng.choice(devs)))]
    for flags in (0, O.F_CP_PIN, O.F_POLICY_INSERT, O.F_MEM_LIVE):
        c = O.make_cand(O.KIND_PIN if pins else O.KIND_BASE, pins=pins, dev_mask=mask_of(devs))
        c2 = O.make_cand(O.KIND_PIN if pins else O.KIND_BASE, pins=[(o, devs.index(d)) for o, d in pins])
        a = g.schedule(c, flags=flags)
        b = h.schedule(c2, flags=flags)
        assert a["status"] == b["status"] and a["makespan"] == b["makespan"]
        if a["status"] != O.CAND_OK:
            continue
        pl = a["placement"][:V]
        assert all(int(x) in devs for x in pl)
        assert [devs.index(int(x)) for x in pl] == b["placement"][:V].tolist()
        assert (a["start"][:V] == b["start"][:V]).all() and (a["order"][:V] == b["order"][:V]).all()
        assert a["peak_mem"][devs].tolist() == b["peak_mem"].tolist()
        assert all(a["peak_mem"][d] == 0 for d in range(G) if d not in devs)


@pytest.mark.parametrize("seed", range(10))
def test_subset_single_device_closed_form(seed):
    """M = {d}: every op on d, makespan = sum of cost[i][d] (no transfers)."""
    desc = synth.random_dag(15000 + seed, caps="none")
    g = O.OracleGraph(desc)
    for d in range(desc.n_devices):
        r = g.schedule(O.make_cand(dev_mask=1 << d), flags=O.F_CP_PIN)
        assert r["makespan"] == int(desc.cost[:, d].sum())
        assert (r["placement"][: desc.n_ops] == d).all()


@pytest.mark.parametrize("seed", range(25))
def test_subset_rank_paths_bruteforce_replay(seed):
    """Small DAGs: ranks with the subset as the allowed set by explicit path
    enumeration; OPT over placements inside M <= oracle; greedy replay."""
    rng = np.random.default_rng(seed)
    desc = synth.random_dag(17000 + seed, V=int(rng.integers(2, 7)), G=3, caps="none")
    devs = sorted(rng.choice(3, size=int(rng.integers(1, 3)), replace=False).tolist())
    g = O.OracleGraph(desc)
    rg = RC.G(desc)
    c = O.make_cand(dev_mask=mask_of(devs))
    rank = g.rank(c)[: desc.n_ops].tolist()
    assert rank == RC.rank_by_paths(rg, dset=set(devs))
    r = g.schedule(c, flags=0)
    assert RC.brute_force_opt(rg, dset=set(devs)) <= r["makespan"]
    RC.check_greedy_steps(rg, r, rank, dset=set(devs))


def test_subset_validation():
    desc = synth.random_dag(19000, V=20, G=4)
    g = O.OracleGraph(desc)
    assert g.schedule(O.make_cand(dev_mask=1 << 4))["status"] == O.CAND_BADSPEC  # device 4 does not exist
    assert g.schedule(O.make_cand(O.KIND_PIN, pins=[(3, 2)], dev_mask=0b0011))["status"] == O.CAND_BADSPEC
    assert g.schedule(O.make_cand(O.KIND_PIN, pins=[(3, 1)], dev_mask=0b0011))["status"] != O.CAND_BADSPEC
    full = g.schedule(O.make_cand(dev_mask=0b1111), flags=O.F_CP_PIN)
    zero = g.schedule(O.make_cand(dev_mask=0), flags=O.F_CP_PIN)
    assert full["makespan"] == zero["makespan"] and (full["placement"] == zero["placement"]).all()


def test_stream_subset_block():
    """With the subset block on, indices n_split+1 .. n_split+G-1 are BASE on
    devices {0..k-1}, k = 1..G-1; every other index is unchanged."""
    desc = synth.config("C1")
    g = O.OracleGraph(desc)
    G = desc.n_devices
    ns, _ = g.stream_info(flags=O.F_CP_PIN)
    a = g.generate(0xABC, 0, ns + 40, flags=O.F_CP_PIN)
    b = g.generate(0xABC, 0, ns + 40, flags=O.F_CP_PIN, subsets=True)
    assert a[: ns + 1].tobytes() == b[: ns + 1].tobytes()
    for k in range(1, G):
        c = b[ns + k]
        assert c["kind"] == O.KIND_BASE and c["dev_mask"] == (1 << k) - 1
    assert a[ns + G:].tobytes() == b[ns + G:].tobytes()
    sw = g.sweep(0xABC, 0, ns + 40, flags=O.F_CP_PIN, subsets=True, per_candidate=True)
    for k in range(1, G):
        r = g.schedule(b[ns + k], flags=O.F_CP_PIN)
        assert sw["makespans"][ns + k] == r["makespan"]
