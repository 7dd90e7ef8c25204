"""GPU parity: the CUDA path (through the C-ABI) against the CPU oracle,
element by element, bit-exact (all arithmetic is integer, R18)."""
import json
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

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def compare(desc, cands, flags, outputs=True, gg=None, og=None):
    gg = gg or F.Graph(desc)
    og = og or O.OracleGraph(desc)
    res = gg.schedule_batch(cands, flags=flags, placement=outputs, order=outputs, start=outputs)
    for k, c in enumerate(cands):
        r = og.schedule(c, flags=flags)
        ctx = (desc.name, k, int(c["kind"]), flags)
        assert int(res["makespan"][k]) == r["makespan"], ctx
        assert int(res["status"][k]) == r["status"], ctx
        assert (res["peak_mem"][k] == r["peak_mem"]).all(), ctx
        if outputs:
            assert (res["placement"][k] == r["placement"]).all(), ctx
            assert (res["start"][k] == r["start"]).all(), ctx
            assert (res["order"][k] == r["order"]).all(), ctx
    return res


def random_cands(desc, rng, n, split_frac=0.2, bad_frac=0.05):
    V, G = desc.n_ops, desc.n_devices
    out = np.zeros(n, F.CANDIDATE_DTYPE)
    smask = desc.split_mask
    splittable = [i for i in range(V) if smask[i]]
    for k in range(n):
        c = F.make_candidate()
        u = rng.random()
        if k == 0 or V == 0:
            pass
        elif u < split_frac and splittable and G >= 2:
            o = int(rng.choice(splittable))
            dims = [d for d in (0, 1) if smask[o] & (1 << d)]
            c = F.make_candidate(F.KIND_SPLIT, split=(o, int(rng.choice(dims)), int(rng.integers(2, G + 1))))
        elif u < split_frac + bad_frac:
            c = F.make_candidate(F.KIND_PIN, pins=[(int(rng.integers(0, V)), G)])  # device out of range
        else:
            npin = int(rng.integers(1, min(4, V) + 1))
            ops = rng.choice(V, npin, replace=False)
            c = F.make_candidate(F.KIND_PIN, pins=[(int(o), int(rng.integers(0, G))) for o in ops])
        out[k] = c
    return out


# ------------------------------------------------------------- hand cases

def test_appendix_golden_on_gpu():
    a1 = json.load(open(os.path.join(GOLD, "a1_diamond.json")))
    g = F.Graph(synth.diamond())
    assert g.rank()[:4].tolist() == a1["rank"]
    base = np.array([F.make_candidate()])
    r = g.schedule_batch(base, flags=F.F_CP_PIN, placement=True, order=True, start=True)
    assert int(r["makespan"][0]) == a1["cp_pin"]["makespan"]
    assert r["placement"][0][:4].tolist() == a1["cp_pin"]["placement"]
    assert r["start"][0][:4].tolist() == a1["cp_pin"]["start"]
    r = g.schedule_batch(base, flags=0, placement=True, start=True)
    assert int(r["makespan"][0]) == a1["pure_eft"]["makespan"]
    assert r["placement"][0][:4].tolist() == a1["pure_eft"]["placement"]
    a2 = json.load(open(os.path.join(GOLD, "a2_split_chain.json")))
    g = F.Graph(synth.split_chain())
    s = a2["split"]
    c = np.array([F.make_candidate(F.KIND_SPLIT, split=(s["op"], s["dim"], s["n"]))])
    r = g.schedule_batch(c, flags=F.F_CP_PIN, placement=True, start=True)
    assert int(r["makespan"][0]) == s["makespan"]
    assert r["placement"][0][: s["V"]].tolist() == s["placement"]
    assert r["start"][0][: s["V"]].tolist() == s["start"]
    assert g.rank(c[0])[: s["V"]].tolist() == s["rank"]
    ss = g.split_search(flags=F.F_CP_PIN)
    assert [list(x) for x in ss["sp"]] == a2["split_search"]["sp"] and ss["makespan"] == a2["split_search"]["makespan"]
    a3 = json.load(open(os.path.join(GOLD, "a3_append_vs_insert.json")))
    g = F.Graph(synth.append_vs_insert())
    c = np.array([F.make_candidate(F.KIND_PIN, pins=[(1, 1)])])
    r = g.schedule_batch(c, flags=F.F_CP_PIN, placement=True, start=True)
    assert int(r["makespan"][0]) == a3["append"]["makespan"]
    assert r["placement"][0][:3].tolist() == a3["append"]["placement"]


# ------------------------------------------------------------- fuzz parity

@pytest.mark.parametrize("seed", range(60))
def test_fuzz_random_dags(seed):
    desc = synth.random_dag(seed)
    rng = np.random.default_rng(seed + 1)
    cands = random_cands(desc, rng, 24)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for flags in (0, F.F_CP_PIN):
        compare(desc, cands, flags, gg=gg, og=og)


@pytest.mark.parametrize("seed", range(12))
def test_fuzz_ranks(seed):
    desc = synth.random_dag(seed + 400)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    assert (gg.rank()[: og.v_max] == og.rank()).all()
    rng = np.random.default_rng(seed)
    for c in random_cands(desc, rng, 10, bad_frac=0.1):
        try:
            want = og.rank(c)
        except O.OracleError:
            with pytest.raises(F.FasttError):
                gg.rank(c)
            continue
        assert (gg.rank(c)[: og.v_max] == want).all()


@pytest.mark.parametrize("V", [1, 2, 31, 32, 33, 63, 64, 65, 1023, 1024, 1025, 2049, 4097])
def test_ragged_sizes(V):
    """bitmap word / summary boundaries and tails"""
    desc = synth.random_dag(V * 7 + 3, V=V, G=4, caps="none", max_in=3)
    rng = np.random.default_rng(V)
    cands = random_cands(desc, rng, 8)
    compare(desc, cands, F.F_CP_PIN)


def test_degenerate_graphs():
    # empty graph
    d0 = synth._finish("empty", 2, [], [], [], [], np.zeros((0, 2), np.int64), [], [], [])
    g = F.Graph(d0)
    r = g.schedule_batch(np.array([F.make_candidate()]), flags=F.F_CP_PIN)
    assert int(r["makespan"][0]) == 0 and int(r["status"][0]) == 0
    # single device, no edges, all-zero costs
    for d in [synth.random_dag(5, G=1, caps="none"), synth.random_dag(6, V=50, zero_frac=1.0, caps="none")]:
        compare(d, random_cands(d, np.random.default_rng(1), 6), F.F_CP_PIN)
    # 32 devices (a full warp of devices) and many link classes
    d = synth.random_dag(77, V=120, G=32, K=5, caps="none")
    compare(d, random_cands(d, np.random.default_rng(2), 10), F.F_CP_PIN)
    # high fan-in / fan-out beyond the inline card entries
    V = 60
    srcs = [0] * 40 + list(range(1, 41))
    dsts = list(range(1, 41)) + [59] * 40
    cost = np.full((V, 3), 7, np.int64)
    d = synth._finish("fan", 3, srcs, dsts, [100] * 80, [0] * 80, cost, [1] * V, [0] * V, [3] * V)
    compare(d, random_cands(d, np.random.default_rng(3), 12), F.F_CP_PIN)
    compare(d, random_cands(d, np.random.default_rng(4), 12), 0)


def test_infeasible_memory_caps():
    for seed in range(10):
        d = synth.random_dag(seed + 50, V=150, G=3, caps=[20000, 20000, 20000])
        compare(d, random_cands(d, np.random.default_rng(seed), 10), F.F_CP_PIN)


# ------------------------------------------------------------- configs

@pytest.mark.parametrize("name", ["C1", "C4"])
def test_config_stream_exhaustive(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    gen = F.gen_params(seed=0xC0FFEE, n_pow2_only=(name == "C4"))
    n_split = gg.stream_info(gen, flags=F.F_CP_PIN)
    n_o, _ = og.stream_info(flags=O.F_CP_PIN, pow2_only=(name == "C4"))
    assert n_split == n_o
    n = n_split + (400 if name == "C1" else 150)
    c = gg.generate_candidates(gen, 0, n, flags=F.F_CP_PIN)
    oc = og.generate(0xC0FFEE, 0, n, flags=O.F_CP_PIN, pow2_only=(name == "C4"))
    assert c.tobytes() == oc.tobytes()
    compare(desc, c, F.F_CP_PIN, gg=gg, og=og, outputs=(name == "C1"))


@pytest.mark.parametrize("name", ["C2", "C3", "C5"])
def test_config_sampled(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    gen = F.gen_params(seed=0xFA57)
    n_split = gg.stream_info(gen, flags=F.F_CP_PIN)
    assert n_split == og.stream_info(flags=O.F_CP_PIN)[0]
    # BASE, a few SPLITs, and PINs far into the stream
    idx = [0] + list(range(1, min(n_split, 3) + 1)) + [n_split + 1 + 7919 * k for k in range(6)]
    cands = np.concatenate([gg.generate_candidates(gen, i, 1, flags=F.F_CP_PIN) for i in idx])
    ocands = np.concatenate([og.generate(0xFA57, i, 1, flags=O.F_CP_PIN) for i in idx])
    assert cands.tobytes() == ocands.tobytes()
    compare(desc, cands, F.F_CP_PIN, gg=gg, og=og, outputs=True)


def test_c4_tight_caps_infeasible():
    desc = synth.vgg19(cap_frac=1.05)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    gen = F.gen_params(seed=11, n_pow2_only=True)
    ns = gg.stream_info(gen, flags=F.F_CP_PIN)
    c = gg.generate_candidates(gen, 0, ns + 60, flags=F.F_CP_PIN)
    res = compare(desc, c, F.F_CP_PIN, gg=gg, og=og, outputs=False)
    n_inf = sum(1 for x in c if og.schedule(x, flags=O.F_CP_PIN, outputs=False)["status"] == 1)
    assert n_inf > 0, "1.05x caps should make some candidates infeasible"
    assert int((res["status"] == 1).sum()) == n_inf


# ------------------------------------------------------------- sweep + argmin

@pytest.mark.parametrize("name", ["C1", "C4"])
def test_sweep_argmin_and_shards(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    pow2 = name == "C4"
    gen = F.gen_params(seed=99, n_pow2_only=pow2)
    n = 600
    best = gg.sweep_best(gen, 0, n, flags=F.F_CP_PIN)
    ob = og.sweep(99, 0, n, flags=O.F_CP_PIN, pow2_only=pow2)
    assert best == (ob["makespan"], ob["index"])
    # W shards (c = r mod W) combined by the lexicographic min == single sweep (P9)
    for W in (2, 4, 8):
        parts = [gg.sweep_best(gen, r, (n - r + W - 1) // W, stride=W, flags=F.F_CP_PIN) for r in range(W)]
        feas = [p for p in parts if p[1] >= 0]
        comb = min(feas) if feas else (F.INT64_MAX, -1)
        assert comb == best


def test_sweep_device_output():
    desc = synth.config("C1")
    gg = F.Graph(desc)
    gen = F.gen_params(seed=5)
    out = torch.zeros(2, dtype=torch.int64, device="cuda")
    gg.sweep_best(gen, 0, 300, flags=F.F_CP_PIN, out=out)
    assert tuple(out.cpu().tolist()) == gg.sweep_best(gen, 0, 300, flags=F.F_CP_PIN)


# ------------------------------------------------------------- split search

@pytest.mark.parametrize("seed", range(10))
def test_split_search_random(seed):
    desc = synth.random_dag(seed + 900, V=80, G=4, caps="none")
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for flags in (0, F.F_CP_PIN):
        a, b = gg.split_search(flags=flags), og.split_search(flags=flags)
        assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"] and a["n_ops_final"] == b["n_ops_final"]
        assert (a["placement"] == b["placement"]).all()
        assert (a["start"] == b["start"]).all()
        assert (a["order"] == b["order"]).all()


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C4", "C5"])
def test_split_search_configs(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    a = gg.split_search(flags=F.F_CP_PIN, n_pow2_only=(name == "C4"))
    b = og.split_search(flags=O.F_CP_PIN, pow2_only=(name == "C4"))
    assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"]
    assert (a["placement"] == b["placement"]).all() and (a["order"] == b["order"]).all()


@pytest.mark.parametrize("seed", [4, 13, 21, 32, 34, 39, 116, 122, 214, 1, 3])
def test_split_search_best_random(seed):
    desc = synth.random_dag(seed, V=40, G=4, caps="none", max_in=2)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for flags in (0, F.F_CP_PIN):
        a = gg.split_search(flags=flags, best_improvement=True)
        b = og.split_search(flags=flags, best_improvement=True)
        assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"] and a["n_ops_final"] == b["n_ops_final"]
        assert (a["placement"] == b["placement"]).all()
        assert (a["start"] == b["start"]).all()
        assert (a["order"] == b["order"]).all()


@pytest.mark.parametrize("name", ["C1", "C2", "C4"])
def test_split_search_best_configs(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    a = gg.split_search(flags=F.F_CP_PIN, n_pow2_only=(name == "C4"), best_improvement=True)
    b = og.split_search(flags=O.F_CP_PIN, pow2_only=(name == "C4"), best_improvement=True)
    assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"]
    assert (a["placement"] == b["placement"]).all() and (a["order"] == b["order"]).all()


# seeds whose multi-split search (R27) accepts a C_j with j >= 2 in some round
# (tests/test_oracle_alg2.py BI_DAGS: random_dag(s, V=40, G=4, max_in=2))
MULTI_SEEDS = [4, 13, 21, 32, 34, 39, 116, 122, 214, 1, 3] + list(range(8))


@pytest.mark.parametrize("seed", MULTI_SEEDS)
def test_split_search_multi_random(seed):
    """NEXT N2 multi-split candidates (R27): the GPU's rounds (C_j
    materialised split after split, DPOS of each) equal the oracle's SP list,
    makespan and per-op outputs"""
    desc = synth.random_dag(seed, V=40, G=4, caps="none", max_in=2)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for flags in (0, F.F_CP_PIN):
        a = gg.split_search(flags=flags, multi=True)
        b = og.split_search(flags=flags, multi=True)
        assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"] and a["n_ops_final"] == b["n_ops_final"]
        assert (a["placement"] == b["placement"]).all()
        assert (a["start"] == b["start"]).all()
        assert (a["order"] == b["order"]).all()


@pytest.mark.parametrize("name", ["C1", "C2", "C4"])
def test_split_search_multi_configs(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    a = gg.split_search(flags=F.F_CP_PIN, n_pow2_only=(name == "C4"), multi=True)
    b = og.split_search(flags=O.F_CP_PIN, pow2_only=(name == "C4"), multi=True)
    assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"]
    assert (a["placement"] == b["placement"]).all() and (a["order"] == b["order"]).all()


@pytest.mark.parametrize("name", ["C3", "C5"])
def test_split_search_best_large_properties(name):
    """C3/C5 best-improvement is minutes of oracle time, so check properties:
    the sweep stream's SPLIT block (R21) is exactly round 1's batch in the
    same enumeration order, so round 1 accepts its first argmin if it beats
    BASE; the result never exceeds BASE; no op is split twice."""
    desc = synth.config(name)
    gg = F.Graph(desc)
    a = gg.split_search(flags=F.F_CP_PIN, best_improvement=True)
    gen = F.gen_params(seed=0)
    n_split = gg.stream_info(gen, flags=F.F_CP_PIN)
    c = gg.generate_candidates(gen, 0, n_split + 1, flags=F.F_CP_PIN)
    r = gg.schedule_batch(c, flags=F.F_CP_PIN)
    base = int(r["makespan"][0])
    ms = np.where(r["status"][1:] == F.CAND_OK, r["makespan"][1:], F.INT64_MAX)
    ops = [x[0] for x in a["sp"]]
    assert len(set(ops)) == len(ops)
    if len(ms) and ms.min() < base:
        k = 1 + int(np.argmin(ms))
        assert a["sp"][0] == (int(c[k]["split_op"]), int(c[k]["split_dim"]), int(c[k]["split_n"]))
        assert a["makespan"] <= int(ms.min())
    else:
        assert a["sp"] == [] and a["makespan"] == base


# ------------------------------------------------------------- device buffers

def test_device_buffers_roundtrip():
    desc = synth.config("C1")
    gg = F.Graph(desc)
    gen = F.gen_params(seed=3)
    c = gg.generate_candidates(gen, 0, 200, flags=F.F_CP_PIN)
    host = gg.schedule_batch(c, flags=F.F_CP_PIN)
    dc = torch.from_numpy(c.view(np.uint8).reshape(-1, 32).copy()).cuda()
    out = {"makespan": torch.zeros(200, dtype=torch.int64, device="cuda"),
           "status": torch.zeros(200, dtype=torch.uint8, device="cuda"),
           "peak_mem": torch.zeros(200 * desc.n_devices, dtype=torch.int64, device="cuda")}
    gg.schedule_batch(dc, flags=F.F_CP_PIN, out=out)
    assert (out["makespan"].cpu().numpy() == host["makespan"]).all()
    assert (out["status"].cpu().numpy() == host["status"]).all()


def test_bench_config_c5_size_and_32bit():
    desc = synth.config("C5")
    gg = F.Graph(desc)
    assert gg.time_bits == 32, "C5 should run the 32-bit time path"


# ------------------------------------------------ BASE-schedule prefix sharing

def _graph_noshare(desc):
    os.environ["FASTT_NO_SHARE"] = "1"
    try:
        return F.Graph(desc)
    finally:
        del os.environ["FASTT_NO_SHARE"]


@pytest.mark.parametrize("seed", range(16))
def test_prefix_sharing_random(seed):
    """makespan-only batches take the prefix-sharing path (no caps, no
    outputs): they must equal the oracle and the non-sharing path."""
    desc = synth.random_dag(seed + 1300, V=int(np.random.default_rng(seed).integers(20, 400)), caps="none",
                            homogeneous=bool(seed % 2))
    gg, og, g0 = F.Graph(desc), O.OracleGraph(desc), _graph_noshare(desc)
    cands = random_cands(desc, np.random.default_rng(seed), 96, split_frac=0.1, bad_frac=0.02)
    for flags in (0, F.F_CP_PIN):
        r = gg.schedule_batch(cands, flags=flags, peak=False)
        r0 = g0.schedule_batch(cands, flags=flags, peak=False)
        assert (r["makespan"] == r0["makespan"]).all() and (r["status"] == r0["status"]).all()
        for k, c in enumerate(cands):
            o = og.schedule(c, flags=flags, outputs=False)
            assert int(r["makespan"][k]) == o["makespan"] and int(r["status"][k]) == o["status"], (seed, k, flags)


@pytest.mark.parametrize("name", ["C1", "C2", "C3", "C5"])
def test_prefix_sharing_configs(name):
    desc = synth.config(name)
    gg, og, g0 = F.Graph(desc), O.OracleGraph(desc), _graph_noshare(desc)
    gen = F.gen_params(seed=0xFA57)
    ns = gg.stream_info(gen, flags=F.F_CP_PIN)
    n = 2000 if name in ("C1",) else 600
    c = gg.generate_candidates(gen, 0, ns + n, flags=F.F_CP_PIN)
    r = gg.schedule_batch(c, flags=F.F_CP_PIN, peak=False)
    r0 = g0.schedule_batch(c, flags=F.F_CP_PIN, peak=False)
    assert (r["makespan"] == r0["makespan"]).all()
    step = 1 if name == "C1" else 97
    for k in list(range(0, len(c), step)) + [0, len(c) - 1]:
        assert int(r["makespan"][k]) == og.schedule(c[k], flags=F.F_CP_PIN, outputs=False)["makespan"], (name, k)
    assert gg.sweep_best(gen, 0, ns + n, flags=F.F_CP_PIN) == g0.sweep_best(gen, 0, ns + n, flags=F.F_CP_PIN)


# ------------------------------------------------ INSERT policy (R1i, NEXT N1)

INS = F.F_POLICY_INSERT


def test_a3_insert_golden_on_gpu():
    a3 = json.load(open(os.path.join(GOLD, "a3_append_vs_insert.json")))
    g = F.Graph(synth.append_vs_insert())
    c = np.array([F.make_candidate(F.KIND_PIN, pins=[(1, 1)])])
    r = g.schedule_batch(c, flags=F.F_CP_PIN | INS, placement=True, start=True)
    assert int(r["makespan"][0]) == a3["insert"]["makespan"]
    assert r["placement"][0][:3].tolist() == a3["insert"]["placement"]
    assert r["start"][0][:3].tolist() == a3["insert"]["start"]


@pytest.mark.parametrize("seed", range(40))
def test_insert_fuzz_random_dags(seed):
    desc = synth.random_dag(seed + 3000)
    rng = np.random.default_rng(seed + 7)
    cands = random_cands(desc, rng, 24)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for flags in (INS, INS | F.F_CP_PIN):
        compare(desc, cands, flags, gg=gg, og=og)


@pytest.mark.parametrize("seed", range(6))
def test_insert_zero_cost_heavy(seed):
    """Many zero-cost ops: zero-length slots and ops splitting idle slots."""
    desc = synth.random_dag(seed + 3100, V=120, G=3, zero_frac=0.5, caps="none")
    rng = np.random.default_rng(seed)
    compare(desc, random_cands(desc, rng, 16), INS | F.F_CP_PIN)


@pytest.mark.parametrize("name", ["C1", "C2", "C4", "C5"])
def test_insert_configs_sampled(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    pow2 = name == "C4"
    flags = F.F_CP_PIN | INS
    gen = F.gen_params(seed=0xFA57, n_pow2_only=pow2)
    n_split = gg.stream_info(gen, flags=flags)
    assert n_split == og.stream_info(flags=flags, pow2_only=pow2)[0]
    idx = [0] + list(range(1, min(n_split, 2) + 1)) + [n_split + 1 + 7919 * k for k in range(3 if name == "C5" else 8)]
    cands = np.concatenate([gg.generate_candidates(gen, i, 1, flags=flags) for i in idx])
    ocands = np.concatenate([og.generate(0xFA57, i, 1, flags=flags, pow2_only=pow2) for i in idx])
    assert cands.tobytes() == ocands.tobytes()
    compare(desc, cands, flags, gg=gg, og=og, outputs=(name != "C5"))


@pytest.mark.parametrize("name", ["C1", "C4"])
def test_insert_sweep(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    pow2 = name == "C4"
    flags = F.F_CP_PIN | INS
    gen = F.gen_params(seed=21, n_pow2_only=pow2)
    n = 300
    assert gg.sweep_best(gen, 0, n, flags=flags) == tuple(
        (lambda o: (o["makespan"], o["index"]))(og.sweep(21, 0, n, flags=flags, pow2_only=pow2)))


@pytest.mark.parametrize("seed", range(6))
def test_insert_split_search(seed):
    desc = synth.random_dag(seed + 950, V=50, G=4, caps="none", max_in=2)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for best in (False, True):
        a = gg.split_search(flags=INS | F.F_CP_PIN, best_improvement=best)
        b = og.split_search(flags=INS | F.F_CP_PIN, best_improvement=best)
        assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"]
        assert (a["placement"] == b["placement"]).all() and (a["start"] == b["start"]).all()


# ------------------------------------------------- TOPO path (dequeue = position order)

def _graph(desc, no_topo):
    old = os.environ.get("FASTT_NO_TOPO")
    os.environ["FASTT_NO_TOPO"] = "1" if no_topo else "0"
    try:
        return F.Graph(desc)
    finally:
        if old is None:
            del os.environ["FASTT_NO_TOPO"]
        else:
            os.environ["FASTT_NO_TOPO"] = old


@pytest.mark.parametrize("name", ["C2", "C3", "C4", "C5"])
def test_topo_path_used_and_equal_to_ready_set_path(name):
    """The paper-shaped configs have c_ij > 0 on every edge (alpha > 0), so
    ranks fall strictly along edges and the priority order is topological:
    the sweep runs the TOPO kernel.  Its per-candidate results equal the
    ready-set kernel's (FASTT_NO_TOPO=1) and the oracle's on a sample."""
    desc = synth.config(name)
    pow2 = name == "C4"
    gen = F.gen_params(seed=0xFA57, n_pow2_only=pow2)
    a, b = _graph(desc, False), _graph(desc, True)
    ns = a.stream_info(gen, flags=F.F_CP_PIN)
    n = 3000 if name == "C5" else 6000
    first = ns + 1
    ca = a.generate_candidates(gen, first, n, flags=F.F_CP_PIN)
    ra = a.schedule_batch(ca, flags=F.F_CP_PIN, peak=False)
    # every paper-shaped config runs the lane kernel (C4: its memory-cap variant)
    assert a.last_timing()["topo"] == 2
    rb = b.schedule_batch(ca, flags=F.F_CP_PIN, peak=False)
    assert b.last_timing()["topo"] == 0
    assert (ra["makespan"] == rb["makespan"]).all() and (ra["status"] == rb["status"]).all()
    assert a.sweep_best(gen, 0, ns + 1 + n, flags=F.F_CP_PIN) == b.sweep_best(gen, 0, ns + 1 + n, flags=F.F_CP_PIN)
    og = O.OracleGraph(desc)
    for k in range(0, n, n // 12):
        assert int(ra["makespan"][k]) == og.schedule(ca[k], flags=O.F_CP_PIN)["makespan"]


@pytest.mark.parametrize("seed", range(12))
def test_topo_vs_ready_set_random(seed):
    """Random DAGs (some with alpha = 0 classes and zero costs, where the
    priority order is not topological and the ready-set kernel must run):
    both paths agree with the oracle on every output."""
    desc = synth.random_dag(seed + 6000)
    rng = np.random.default_rng(seed)
    cands = random_cands(desc, rng, 30)
    og = O.OracleGraph(desc)
    for g in (_graph(desc, False), _graph(desc, True)):
        for flags in (0, F.F_CP_PIN):
            compare(desc, cands, flags, gg=g, og=og)


# ------------------------------------------ SPLIT slots reuse the base ranks

@pytest.mark.parametrize("name", ["C2", "C3", "C5"])
def test_split_rank_reuse_ab(name):
    """SPLIT slots copy the base ranks below the split op's height (no path to
    the split op): every split candidate of the stream against the slots that
    recompute all ranks (FASTT_NO_RANK_REUSE=1), a sample against the oracle"""
    desc = synth.config(name)
    gg = F.Graph(desc)
    os.environ["FASTT_NO_RANK_REUSE"] = "1"
    try:
        g0 = F.Graph(desc)
    finally:
        del os.environ["FASTT_NO_RANK_REUSE"]
    gen = F.gen_params(seed=0xFA57)
    ns = gg.stream_info(gen, flags=F.F_CP_PIN)
    c = gg.generate_candidates(gen, 1, min(ns, 600), flags=F.F_CP_PIN)
    a = gg.schedule_batch(c, flags=F.F_CP_PIN, peak=False)
    b = g0.schedule_batch(c, flags=F.F_CP_PIN, peak=False)
    assert (a["makespan"] == b["makespan"]).all() and (a["status"] == b["status"]).all()
    og = O.OracleGraph(desc)
    for k in range(0, len(c), max(1, len(c) // 6)):
        assert int(a["makespan"][k]) == og.schedule(c[k], flags=O.F_CP_PIN, outputs=False)["makespan"], (name, k)
