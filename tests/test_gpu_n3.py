"""GPU parity of the NEXT-row N3 features through the C-ABI:
liveness memory (R24, FASTT_F_MEM_LIVE) and device-subset candidates (R25,
dev_mask), bit-exact against the CPU oracle (all arithmetic is integer)."""
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

LIVE = F.F_MEM_LIVE
INS = F.F_POLICY_INSERT


def compare(desc, cands, flags, gg, og, outputs=True):
    res = gg.schedule_batch(cands, flags=flags, placement=outputs, order=outputs, start=outputs)
    for k, c in enumerate(cands):
        r = og.schedule(c, flags=flags)
        ctx = (desc.name, k, int(c["kind"]), int(c["dev_mask"]), flags)
        assert int(res["makespan"][k]) == r["makespan"], ctx
        assert int(res["status"][k]) == r["status"], ctx
        assert (res["peak_mem"][k] == r["peak_mem"]).all(), ctx
        if outputs:
            assert (res["placement"][k] == r["placement"]).all(), ctx
            assert (res["start"][k] == r["start"]).all(), ctx
            assert (res["order"][k] == r["order"]).all(), ctx
    return res


def subset_cands(desc, rng, n):
    """BASE / PIN / SPLIT candidates, most with a random device subset (some
    invalid: pins outside the subset, bits >= G)."""
    V, G = desc.n_ops, desc.n_devices
    full = (1 << G) - 1
    splittable = [i for i in range(V) if desc.split_mask[i]]
    out = np.zeros(n, F.CANDIDATE_DTYPE)
    for k in range(n):
        m = int(rng.integers(1, full + 1)) if rng.random() < 0.8 else 0
        if rng.random() < 0.04:
            m |= 1 << G  # not a device
        devs = [d for d in range(G) if (m or full) >> d & 1] or [0]
        u = rng.random()
        if u < 0.3 or V == 0:
            c = F.make_candidate(dev_mask=m)
        elif u < 0.45 and splittable and G >= 2:
            o = int(rng.choice(splittable))
            dims = [d for d in (0, 1) if desc.split_mask[o] & (1 << d)]
            c = F.make_candidate(F.KIND_SPLIT, split=(o, int(rng.choice(dims)), int(rng.integers(2, G + 1))), dev_mask=m)
        else:
            npin = int(rng.integers(1, min(4, V) + 1))
            ops = rng.choice(V, npin, replace=False)
            pool = devs if rng.random() < 0.9 else list(range(G))
            c = F.make_candidate(F.KIND_PIN, pins=[(int(o), int(rng.choice(pool))) for o in ops], dev_mask=m)
        out[k] = c
    return out


# ------------------------------------------------------------ R24 liveness

@pytest.mark.parametrize("seed", range(40))
def test_live_fuzz_random_dags(seed):
    desc = synth.random_dag(seed + 3000)
    rng = np.random.default_rng(seed)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    cands = subset_cands(desc, rng, 20)
    cands["dev_mask"][rng.random(len(cands)) < 0.6] = 0
    for flags in (LIVE, LIVE | F.F_CP_PIN, LIVE | F.F_CP_PIN | INS):
        compare(desc, cands, flags, gg, og)


@pytest.mark.parametrize("seed", range(10))
def test_live_tight_caps(seed):
    """Caps between the live peak and the static total: the two models
    disagree on feasibility; the GPU follows the oracle in both."""
    desc = synth.random_dag(seed + 3100, V=120, caps="none")
    tot = int(desc.mem.sum())
    desc.cap[:] = tot // desc.n_devices // 2 + 1
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    cands = subset_cands(desc, np.random.default_rng(seed), 24)
    cands["dev_mask"] = 0
    for flags in (0, LIVE, LIVE | F.F_CP_PIN):
        compare(desc, cands, flags, gg, og, outputs=False)


@pytest.mark.parametrize("name", ["C1", "C4", "C2"])
def test_live_configs_sampled(name):
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    pow2 = name == "C4"
    flags = F.F_CP_PIN | LIVE
    gen = F.gen_params(seed=0xFA57, n_pow2_only=pow2)
    n_split = gg.stream_info(gen, flags=flags)
    assert n_split == og.stream_info(flags=flags, pow2_only=pow2)[0]
    idx = [0] + list(range(1, min(n_split, 3) + 1)) + [n_split + 1 + 7919 * k for k in range(8)]
    cands = np.concatenate([gg.generate_candidates(gen, i, 1, flags=flags) for i in idx])
    ocands = np.concatenate([og.generate(0xFA57, i, 1, flags=flags, pow2_only=pow2) for i in idx])
    assert cands.tobytes() == ocands.tobytes()
    compare(desc, cands, flags, gg, og, outputs=(name != "C2"))


def test_live_c4_tight_sweep():
    """VGG-19 with caps at 1.05 x the even share: the sweep's argmin under
    liveness memory equals the oracle's."""
    desc = synth.vgg19(cap_frac=1.05)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    flags = F.F_CP_PIN | LIVE
    gen = F.gen_params(seed=11, n_pow2_only=True)
    n = 200
    ob = og.sweep(11, 0, n, flags=flags, pow2_only=True)
    assert gg.sweep_best(gen, 0, n, flags=flags) == (ob["makespan"], ob["index"])


@pytest.mark.parametrize("seed", range(5))
def test_live_split_search(seed):
    desc = synth.random_dag(seed + 3200, V=60, G=4, max_in=2)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for best in (False, True):
        a = gg.split_search(flags=LIVE | F.F_CP_PIN, best_improvement=best)
        b = og.split_search(flags=LIVE | F.F_CP_PIN, best_improvement=best)
        assert a["sp"] == b["sp"] and a["makespan"] == b["makespan"]
        if b["status"] == 0:
            assert (a["placement"] == b["placement"]).all() and (a["start"] == b["start"]).all()


# ------------------------------------------------------------- R25 subsets

@pytest.mark.parametrize("seed", range(40))
def test_subset_fuzz_random_dags(seed):
    desc = synth.random_dag(seed + 3300)
    rng = np.random.default_rng(seed + 7)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    cands = subset_cands(desc, rng, 24)
    for flags in (0, F.F_CP_PIN, F.F_CP_PIN | INS):
        compare(desc, cands, flags, gg, og)


@pytest.mark.parametrize("seed", range(10))
def test_subset_ranks(seed):
    desc = synth.random_dag(seed + 3400)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    for c in subset_cands(desc, np.random.default_rng(seed), 12):
        try:
            want = og.rank(c)
        except O.OracleError:
            with pytest.raises(F.FasttError):
                gg.rank(c)
            continue
        assert (gg.rank(c)[: og.v_max] == want).all()


@pytest.mark.parametrize("name", ["C1", "C3"])
def test_subset_stream_and_sweep(name):
    """The stream's subset block (R25) and a sweep over it, against the oracle."""
    desc = synth.config(name)
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    G = desc.n_devices
    gen = F.gen_params(seed=0x5B, subset_prefixes=True)
    ns = gg.stream_info(gen, flags=F.F_CP_PIN)
    n = ns + G + 40
    c = gg.generate_candidates(gen, 0, n, flags=F.F_CP_PIN)
    oc = og.generate(0x5B, 0, n, flags=O.F_CP_PIN, subsets=True)
    assert c.tobytes() == oc.tobytes()
    sub = c[ns + 1: ns + G]
    assert [int(x) for x in sub["dev_mask"]] == [(1 << k) - 1 for k in range(1, G)]
    compare(desc, sub, F.F_CP_PIN, gg, og, outputs=(name == "C1"))
    if name == "C1":
        ob = og.sweep(0x5B, 0, n, flags=O.F_CP_PIN, subsets=True)
        assert gg.sweep_best(gen, 0, n, flags=F.F_CP_PIN) == (ob["makespan"], ob["index"])
