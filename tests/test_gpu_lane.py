"""GPU parity of the lane-per-candidate position-order kernel (k_sim_lane.cu):
bit-exact against the CPU oracle and against the group-per-candidate kernels
(FASTT_NO_LANE=1 / FASTT_NO_TOPO=1 A/B), on graphs whose priority order is
topological (all op costs > 0, so rank_u strictly decreases along edges, R2).

Coverage: device counts 1..32 (every lane-group width), one and several link
classes (the single-class arrival shortcut and the per-pair path), 32- and
64-bit time, hetero costs (CP devices that move when CP ops are pinned, so
prefix sharing is refused), sweeps against the group kernel."""
import dataclasses
import os

import numpy as np
import pytest

import oracle as O
from paper_conf_middleware_0001lmwlwyl20_b200 import synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_middleware_0001lmwlwyl20_b200 import build as B  # noqa: E402

B.build()
from paper_conf_middleware_0001lmwlwyl20_b200 import fastt as F  # noqa: E402

LANE, GROUP = 2, 1


def _graph_env(desc, **env):
    old = {k: os.environ.get(k) for k in env}
    os.environ.update(env)
    try:
        return F.Graph(desc)
    finally:
        for k, v in old.items():
            if v is None:
                del os.environ[k]
            else:
                os.environ[k] = v


def topo_dag(seed, V, G, K=1, homogeneous=False, scale=1, caps="none"):
    """random DAG with every op cost > 0 (topological priority order)"""
    d = synth.random_dag(seed, V=V, G=G, K=K, zero_frac=0.0, caps=caps, homogeneous=homogeneous)
    cost = np.maximum(d.cost, 1) * scale
    return dataclasses.replace(d, cost=cost)


def pin_cands(desc, rng, n, kmax=4):
    V, G = desc.n_ops, desc.n_devices
    out = np.zeros(n, F.CANDIDATE_DTYPE)
    for k in range(n):
        if k == 0 or V == 0:
            out[k] = F.make_candidate()
            continue
        npin = int(rng.integers(1, min(kmax, V) + 1))
        ops = rng.choice(V, npin, replace=False)
        out[k] = F.make_candidate(F.KIND_PIN, pins=[(int(o), int(rng.integers(0, G))) for o in ops])
    return out


def check(desc, cands, flags, expect_kernel=LANE, oracle_every=1, peak=False):
    gl = _graph_env(desc, FASTT_LANE_INS="1") if flags & F.F_POLICY_INSERT else F.Graph(desc)
    gg = _graph_env(desc, FASTT_NO_LANE="1")
    r = gl.schedule_batch(cands, flags=flags, peak=peak)
    assert gl.last_timing()["topo"] == expect_kernel
    r0 = gg.schedule_batch(cands, flags=flags, peak=peak)
    assert gg.last_timing()["topo"] in (0, GROUP)
    assert (r["makespan"] == r0["makespan"]).all() and (r["status"] == r0["status"]).all()
    if peak:
        assert (r["peak_mem"] == r0["peak_mem"]).all()
    og = O.OracleGraph(desc)
    for k in range(0, len(cands), oracle_every):
        o = og.schedule(cands[k], flags=flags, outputs=False)
        assert int(r["makespan"][k]) == o["makespan"] and int(r["status"][k]) == o["status"], (desc.name, k, flags)
        if peak:
            assert (r["peak_mem"][k] == o["peak_mem"]).all(), (desc.name, k, flags)
    return r


@pytest.mark.parametrize("G", [1, 2, 3, 4, 5, 8, 13, 16, 32])
def test_lane_device_counts(G):
    desc = topo_dag(4000 + G, V=150, G=G, K=1, homogeneous=bool(G % 2))
    cands = pin_cands(desc, np.random.default_rng(G), 160)
    for flags in (0, F.F_CP_PIN):
        check(desc, cands, flags)


@pytest.mark.parametrize("seed", range(6))
def test_lane_link_classes(seed):
    """several link classes: per (pred, device) comm terms (CM = 2)"""
    desc = topo_dag(4100 + seed, V=120, G=int(3 + seed % 6), K=3)
    cands = pin_cands(desc, np.random.default_rng(seed), 128)
    check(desc, cands, F.F_CP_PIN)


@pytest.mark.parametrize("seed", range(4))
def test_lane_64bit_time(seed):
    desc = topo_dag(4200 + seed, V=100, G=int(2 + 2 * seed), K=1 + seed % 2, scale=50_000_000)
    assert F.Graph(desc).time_bits == 64
    cands = pin_cands(desc, np.random.default_rng(seed), 96)
    check(desc, cands, F.F_CP_PIN)


@pytest.mark.parametrize("seed", range(8))
def test_cp_pins_refuse_sharing(seed):
    """Hetero costs: pinning critical-path ops moves the CP device (R9), so
    those candidates cannot start from the recorded BASE prefix; every CP op
    pinned to every device, both position-order kernels against the oracle."""
    desc = topo_dag(4300 + seed, V=80, G=3 + seed % 3, K=1)
    og = O.OracleGraph(desc)
    base = og.schedule(F.make_candidate(), flags=F.F_CP_PIN)
    cands = [F.make_candidate()]
    for o in range(desc.n_ops):
        for dv in range(desc.n_devices):
            cands.append(F.make_candidate(F.KIND_PIN, pins=[(o, dv)]))
    cands = np.array(cands)
    r = check(desc, cands, F.F_CP_PIN)
    assert int(r["makespan"][0]) == base["makespan"]
    # the group position-order kernel on the same list (t0 of refused candidates)
    gg = _graph_env(desc, FASTT_NO_LANE="1")
    r1 = gg.schedule_batch(cands, flags=F.F_CP_PIN, peak=False)
    assert gg.last_timing()["topo"] == GROUP
    assert (r1["makespan"] == r["makespan"]).all()


@pytest.mark.parametrize("name", ["C2", "C5"])
def test_lane_sweep_configs(name):
    desc = synth.config(name)
    gl, gg = F.Graph(desc), _graph_env(desc, FASTT_NO_LANE="1")
    gen = F.gen_params(seed=0xFA57)
    ns = gl.stream_info(gen, flags=F.F_CP_PIN)
    n = ns + 3000
    b1 = gl.sweep_best(gen, 0, n, flags=F.F_CP_PIN)
    assert gl.last_timing()["topo"] == LANE
    b0 = gg.sweep_best(gen, 0, n, flags=F.F_CP_PIN)
    assert b1 == b0
    c = gl.generate_candidates(gen, ns + 1, 700, flags=F.F_CP_PIN)
    r = gl.schedule_batch(c, flags=F.F_CP_PIN, peak=False)
    assert gl.last_timing()["topo"] == LANE
    r0 = gg.schedule_batch(c, flags=F.F_CP_PIN, peak=False)
    assert (r["makespan"] == r0["makespan"]).all()
    og = O.OracleGraph(desc)
    for k in range(0, len(c), 233):
        assert int(r["makespan"][k]) == og.schedule(c[k], flags=F.F_CP_PIN, outputs=False)["makespan"], (name, k)


def test_lane_small_batches_no_sharing():
    """fewer than 64 candidates: no snapshot, every candidate from step 0"""
    desc = topo_dag(4400, V=200, G=8, K=1)
    cands = pin_cands(desc, np.random.default_rng(1), 40)
    check(desc, cands, F.F_CP_PIN)
    check(desc, cands, 0)


def test_lane_ragged_and_invalid():
    """a batch that is not a multiple of 32, bad specs and splits mixed in"""
    desc = topo_dag(4500, V=90, G=4, K=1)
    desc = dataclasses.replace(desc, split_mask=np.full(desc.n_ops, 3, np.uint8))
    rng = np.random.default_rng(2)
    cands = list(pin_cands(desc, rng, 101))
    cands[7] = F.make_candidate(F.KIND_PIN, pins=[(3, desc.n_devices)])         # device out of range
    cands[40] = F.make_candidate(F.KIND_SPLIT, split=(10, 0, 2))                 # deferred (prep pipeline)
    cands[41] = F.make_candidate(F.KIND_PIN, pins=[(5, 1), (5, 2)])              # duplicate op
    cands[77] = F.make_candidate(dev_mask=0b0011)                                # device subset (deferred)
    check(desc, np.array(cands), F.F_CP_PIN)


# ------------------------------------------- packed device keys (PK variant)

@pytest.mark.parametrize("G", [1, 2, 3, 5, 8, 16, 32])
def test_pk_ab_device_counts(G):
    """the packed-key lane kernel (default for 32-bit time, one link class)
    against the unpacked lane kernel (FASTT_NO_PK=1) and the oracle"""
    desc = topo_dag(4600 + G, V=140, G=G, K=1, homogeneous=bool(G % 2))
    cands = pin_cands(desc, np.random.default_rng(100 + G), 200)
    gp = F.Graph(desc)
    gu = _graph_env(desc, FASTT_NO_PK="1")
    for flags in (0, F.F_CP_PIN):
        r = check(desc, cands, flags)
        r0 = gu.schedule_batch(cands, flags=flags, peak=False)
        assert gu.last_timing()["topo"] == LANE
        assert (r["makespan"] == r0["makespan"]).all()
        if G > 1:  # (G = 1: the stream has no PIN candidates)
            assert gp.sweep_best(F.gen_params(seed=G), 0, 3000, flags=flags) == \
                gu.sweep_best(F.gen_params(seed=G), 0, 3000, flags=flags)


@pytest.mark.parametrize("lim_q", [0.0, 0.3, 0.7])
def test_pk_deferral_path(lim_q):
    """candidates whose makespan reaches the packed-key bound are deferred to
    the preparation pipeline and re-run unpacked: FASTT_PK_LIM lowers the bound
    to a quantile of the makespans so part (or all) of a batch takes that path"""
    desc = topo_dag(4700, V=180, G=8, K=1)
    cands = pin_cands(desc, np.random.default_rng(7), 256)
    ms = F.Graph(desc).schedule_batch(cands, flags=F.F_CP_PIN, peak=False)["makespan"]
    lim = max(1, int(np.quantile(ms, lim_q)))
    gl = _graph_env(desc, FASTT_PK_LIM=str(lim))
    r = gl.schedule_batch(cands, flags=F.F_CP_PIN, peak=False)
    t = gl.last_timing()
    assert t["topo"] == LANE and t["deferred"] >= int((ms >= lim).sum()) > 0
    assert (r["makespan"] == ms).all()
    og = O.OracleGraph(desc)
    for k in range(0, len(cands), 5):
        assert int(r["makespan"][k]) == og.schedule(cands[k], flags=F.F_CP_PIN, outputs=False)["makespan"]
    # the sweep: deferred candidates still compete for the argmin
    gen = F.gen_params(seed=3)
    assert gl.sweep_best(gen, 0, 2000, flags=F.F_CP_PIN) == F.Graph(desc).sweep_best(gen, 0, 2000, flags=F.F_CP_PIN)


def test_pk_large_makespans():
    """makespans above 2^29 ns with 32-bit time at G = 8: the natural
    packed-key bound defers them (no key may wrap), results stay exact"""
    d0 = topo_dag(4800, V=120, G=8, K=1)
    V = d0.n_ops
    # a chain through all ops on top of the random edges: makespan ~ sum of costs
    src = np.concatenate([np.asarray(d0.src), np.arange(V - 1)]).astype(np.asarray(d0.src).dtype)
    dst = np.concatenate([np.asarray(d0.dst), np.arange(1, V)]).astype(np.asarray(d0.dst).dtype)
    nb = np.concatenate([np.asarray(d0.bytes), np.full(V - 1, 1024)]).astype(np.asarray(d0.bytes).dtype)
    ep = np.concatenate([np.asarray(d0.eparam), np.zeros(V - 1)]).astype(np.asarray(d0.eparam).dtype)
    scale = max(1, int(1.5e9 / float(d0.cost.reshape(V, -1).max(axis=1).sum())))
    desc = dataclasses.replace(d0, src=src, dst=dst, bytes=nb, eparam=ep, cost=d0.cost * scale)
    g = F.Graph(desc)
    assert g.time_bits == 32
    cands = pin_cands(desc, np.random.default_rng(9), 96)
    r = check(desc, cands, F.F_CP_PIN)
    assert int(r["makespan"].max()) >= (1 << 29)
    g.schedule_batch(cands, flags=F.F_CP_PIN, peak=False)
    assert g.last_timing()["deferred"] >= int((r["makespan"] >= (1 << 29)).sum()) > 0


# ------------------------------------------- memory on the lane kernel (MM)

@pytest.mark.parametrize("G", [1, 2, 3, 5, 8, 13, 32])
def test_lane_peak_memory(G):
    """per-device peak memory (R8: the static total per device) requested
    without caps: the lane kernel's MM 1 variant, against the group kernel
    and the oracle, with and without prefix sharing"""
    desc = topo_dag(5000 + G, V=150, G=G, K=1 + G % 2, homogeneous=bool(G % 2))
    cands = pin_cands(desc, np.random.default_rng(G), 160)
    for flags in (0, F.F_CP_PIN):
        check(desc, cands, flags, peak=True)
    gn = _graph_env(desc, FASTT_NO_SHARE="1")
    r0 = gn.schedule_batch(cands, flags=F.F_CP_PIN, peak=True)
    r1 = F.Graph(desc).schedule_batch(cands, flags=F.F_CP_PIN, peak=True)
    assert (r0["peak_mem"] == r1["peak_mem"]).all() and (r0["makespan"] == r1["makespan"]).all()


@pytest.mark.parametrize("seed", range(12))
def test_lane_memory_caps(seed):
    """finite per-device caps (Alg. 1 line 13, R8, R9: multi-round CP devices
    with reservations, infeasible candidates): the lane kernel's MM 2 variant
    on 32- and 64-bit time, one and several link classes"""
    G = [2, 3, 4, 5, 8, 16][seed % 6]
    desc = topo_dag(5100 + seed, V=130, G=G, K=1 + (seed % 3 == 2) * 2, caps="random",
                    scale=(50_000_000 if seed % 4 == 3 else 1))
    cands = pin_cands(desc, np.random.default_rng(seed), 192)
    for flags in (0, F.F_CP_PIN):
        r = check(desc, cands, flags, peak=True)
        r2 = F.Graph(desc).schedule_batch(cands, flags=flags, peak=False)
        assert (r2["makespan"] == r["makespan"]).all() and (r2["status"] == r["status"]).all()


@pytest.mark.parametrize("seed", range(6))
def test_lane_caps_tight_and_sweep(seed):
    """caps just above the average load (many infeasible candidates, CP
    rounds that span several devices), the sweep argmin and prefix sharing
    (A/B against FASTT_NO_SHARE=1 and the group kernel)"""
    d0 = topo_dag(5200 + seed, V=160, G=4 + seed % 5, K=1)
    cap = np.full(d0.n_devices, int(d0.mem.sum() * (1.1 + 0.1 * (seed % 3)) / d0.n_devices), np.int64)
    desc = dataclasses.replace(d0, cap=cap)
    cands = pin_cands(desc, np.random.default_rng(seed), 200)
    r = check(desc, cands, F.F_CP_PIN, peak=True)
    gn = _graph_env(desc, FASTT_NO_SHARE="1")
    r0 = gn.schedule_batch(cands, flags=F.F_CP_PIN, peak=True)
    assert (r0["makespan"] == r["makespan"]).all() and (r0["peak_mem"] == r["peak_mem"]).all()
    gen = F.gen_params(seed=seed)
    gl, gg = F.Graph(desc), _graph_env(desc, FASTT_NO_LANE="1")
    b1 = gl.sweep_best(gen, 0, 2500, flags=F.F_CP_PIN)
    assert gl.last_timing()["topo"] == LANE
    assert b1 == gg.sweep_best(gen, 0, 2500, flags=F.F_CP_PIN)


def test_lane_memory_configs():
    """C4 (VGG-19, caps, 64-bit time) and C5 (peak requested) stay on the
    lane kernel; sampled against the oracle"""
    for name, peak in (("C4", True), ("C5", True)):
        desc = synth.config(name)
        gl = F.Graph(desc)
        gen = F.gen_params(seed=0xFA57, n_pow2_only=name == "C4")
        ns = gl.stream_info(gen, flags=F.F_CP_PIN)
        c = gl.generate_candidates(gen, ns + 1, 600, flags=F.F_CP_PIN)
        r = gl.schedule_batch(c, flags=F.F_CP_PIN, peak=peak)
        assert gl.last_timing()["topo"] == LANE, name
        og = O.OracleGraph(desc)
        for k in range(0, len(c), 50):
            o = og.schedule(c[k], flags=F.F_CP_PIN, outputs=False)
            assert (int(r["makespan"][k]), int(r["status"][k])) == (o["makespan"], o["status"]), (name, k)
            assert (r["peak_mem"][k] == o["peak_mem"]).all(), (name, k)


# ------------------------------------------- INSERT on the lane kernel (R1i)

INS = F.F_POLICY_INSERT


@pytest.mark.parametrize("G", [1, 2, 3, 5, 8, 16])
def test_lane_insert(G):
    """INSERT (R1i) on the lane kernel (FASTT_LANE_INS=1: opt-in,
    the group kernel is faster on C5): per-lane idle-slot arrays, binary
    search + scan, slot split/shrink/removal -- against the group kernel
    (FASTT_NO_LANE=1) and the oracle, with and without CP pins, one and
    several link classes, 32- and 64-bit time"""
    for K, scale in ((1, 1), (3, 1), (1, 50_000_000)):
        desc = topo_dag(5300 + G + 7 * K, V=140, G=G, K=K, homogeneous=bool(G % 2), scale=scale)
        cands = pin_cands(desc, np.random.default_rng(G + K), 128)
        for flags in (INS, INS | F.F_CP_PIN):
            check(desc, cands, flags)


def test_lane_insert_capacity_deferral():
    """a device needing more idle slots than the lane kernel's capacity
    (FASTT_INS_CAP) defers the candidate to the group kernel: same results"""
    desc = topo_dag(5400, V=200, G=4, K=1)
    cands = pin_cands(desc, np.random.default_rng(3), 96)
    ref = F.Graph(desc).schedule_batch(cands, flags=INS | F.F_CP_PIN, peak=False)
    for cap in ("1", "3"):
        g = _graph_env(desc, FASTT_INS_CAP=cap, FASTT_LANE_INS="1")
        r = g.schedule_batch(cands, flags=INS | F.F_CP_PIN, peak=False)
        assert g.last_timing()["topo"] == LANE and g.last_timing()["deferred"] > 0
        assert (r["makespan"] == ref["makespan"]).all() and (r["status"] == ref["status"]).all()
    og = O.OracleGraph(desc)
    for k in range(0, len(cands), 7):
        assert int(ref["makespan"][k]) == og.schedule(cands[k], flags=INS | F.F_CP_PIN, outputs=False)["makespan"]


@pytest.mark.parametrize("name", ["C2", "C5"])
def test_lane_insert_sweep_configs(name):
    """the INSERT sweep on paper-shaped configs: lane kernel == group kernel,
    winner == the oracle's makespan at that index"""
    desc = synth.config(name)
    gl, gg = _graph_env(desc, FASTT_LANE_INS="1"), F.Graph(desc)
    flags = INS | F.F_CP_PIN
    gen = F.gen_params(seed=0xFA57)
    ns = gl.stream_info(gen, flags=flags)
    n = ns + 1500
    b1 = gl.sweep_best(gen, 0, n, flags=flags)
    assert gl.last_timing()["topo"] == LANE
    assert b1 == gg.sweep_best(gen, 0, n, flags=flags)
    c = gl.generate_candidates(gen, b1[1], 1, flags=flags)
    assert O.OracleGraph(desc).schedule(c[0], flags=flags, outputs=False)["makespan"] == b1[0]
