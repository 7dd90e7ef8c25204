"""GPU parity of the communication cost-model fit (reading
R26) through the C-ABI (fastt_fit_comm) against the exact-rational oracle
(oracle/commfit.py): bit-exact integers on every pair."""
import numpy as np
import pytest

import oracle as O
from oracle import commfit as CF
from paper_conf_middleware_0001lmwlwyl20_b200 import synth

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

from paper_conf_middleware_0001lmwlwyl20_b200 import build as B  # noqa: E402

B.build()
from paper_conf_middleware_0001lmwlwyl20_b200 import costmodel as CM  # noqa: E402
from paper_conf_middleware_0001lmwlwyl20_b200 import fastt as F  # noqa: E402


def samples(rng, G, n, kind):
    s = rng.integers(0, G, n)
    d = (s + rng.integers(1, G, n)) % G if G > 1 else s
    if kind == "linear":
        b = rng.integers(0, 1 << 30, n)
        t = 10_000 + (b * rng.uniform(0.001, 0.1)).astype(np.int64) + rng.integers(0, 5000, n)
    elif kind == "falling":
        b = rng.integers(0, 1 << 20, n)
        t = np.maximum(5_000_000 - b * 3 + rng.integers(0, 100000, n), 0)
    elif kind == "origin":
        b = rng.integers(0, 1 << 20, n)
        t = np.maximum(b * 7 - 2_000_000 + rng.integers(0, 1000, n), 0)
    elif kind == "huge":  # near the envelope: bytes, time < 2^40
        b = rng.integers((1 << 40) - (1 << 36), 1 << 40, n)
        t = rng.integers((1 << 40) - (1 << 38), 1 << 40, n)
    elif kind == "tiny":
        b = rng.integers(0, 4, n)
        t = rng.integers(0, 4, n)
    else:  # one size per pair (no spread)
        b = np.full(n, 4096)
        t = rng.integers(0, 1 << 30, n)
    return s.astype(np.uint8), d.astype(np.uint8), b.astype(np.int64), t.astype(np.int64)


@pytest.mark.parametrize("kind", ["linear", "falling", "origin", "huge", "tiny", "flat"])
@pytest.mark.parametrize("seed", range(4))
def test_fit_matches_oracle(kind, seed):
    rng = np.random.default_rng(seed)
    G = int(rng.integers(2, 9))
    n = int(rng.integers(1, 3000))
    s, d, b, t = samples(rng, G, n, kind)
    a, bb, c = F.fit_comm(G, s, d, b, t)
    oa, ob, oc = CF.fit_comm(G, s, d, b, t)
    assert a.tolist() == oa and bb.tolist() == ob and c.tolist() == oc


def test_fit_large_and_all_pairs():
    """1e6 samples over all 32 x 31 pairs of G = 32 (sums across many blocks)."""
    rng = np.random.default_rng(7)
    G, n = 32, 1_000_000
    s, d, b, t = samples(rng, G, n, "linear")
    a, bb, c = F.fit_comm(G, s, d, b, t)
    oa, ob, oc = CF.fit_comm(G, s, d, b, t)
    assert a.tolist() == oa and bb.tolist() == ob and c.tolist() == oc
    assert int(c.sum()) == n


def test_fit_rejects_bad_samples():
    for s, d, b, t in [([0], [0], [1], [1]), ([0], [2], [1], [1]), ([0], [1], [-1], [1]),
                       ([0], [1], [1 << 40], [1]), ([0], [1], [1], [1 << 40])]:
        with pytest.raises(F.FasttError) as e:
            F.fit_comm(2, s, d, b, t)
        assert e.value.code == F.EINVAL
    a, bb, c = F.fit_comm(3, [], [], [], [])
    assert not a.any() and not bb.any() and not c.any()


def test_fitted_model_schedules_like_the_oracle():
    """Trace -> GPU fit -> link classes -> a graph whose schedules the GPU and
    the oracle compute identically (the fitted model feeds R10)."""
    rng = np.random.default_rng(3)
    G = 4
    ev = []
    for _ in range(400):
        s_ = int(rng.integers(0, G))
        d_ = int((s_ + rng.integers(1, G)) % G)
        nvl = (s_ // 2) == (d_ // 2)  # two "NVLink islands"
        byt = int(rng.integers(1 << 10, 1 << 26))
        us = (5 if nvl else 20) + byt * (0.0011 if nvl else 0.04) / 1000
        ev.append({"ph": "X", "cat": "gpu_memcpy", "dur": round(us, 3),
                   "args": {"src_device": s_, "dst_device": d_, "bytes": byt}})
    m = CM.fit_link_model(ev, G)
    assert len(m["alpha"]) <= 16 and m["count"].sum() == 400
    base = synth.random_dag(77, V=150, G=G, caps="none")
    desc = synth._finish("fitted", G, base.src, base.dst, base.bytes, base.eparam, base.cost, base.mem, base.param,
                         base.split_mask, cap=base.cap, classes=(m["link_class"], m["alpha"], m["beta"]))
    gg, og = F.Graph(desc), O.OracleGraph(desc)
    gen = F.gen_params(seed=5)
    ns = gg.stream_info(gen, flags=F.F_CP_PIN)
    c = gg.generate_candidates(gen, 0, ns + 30, flags=F.F_CP_PIN)
    res = gg.schedule_batch(c, flags=F.F_CP_PIN, placement=True, start=True)
    for k, cand in enumerate(c):
        r = og.schedule(cand, flags=O.F_CP_PIN)
        assert int(res["makespan"][k]) == r["makespan"]
        assert (res["placement"][k] == r["placement"]).all() and (res["start"][k] == r["start"]).all()


# ------------------------------------------------ computation cost table (N4)

@pytest.mark.parametrize("seed", range(6))
def test_cost_table_matches_oracle(seed):
    """fastt_cost_table (GPU integer sums) equals the exact-rational mean of
    every (op, device) group, halves up; groups without a sample are 0"""
    rng = np.random.default_rng(seed)
    V, G = int(rng.integers(1, 300)), int(rng.integers(1, 33))
    n = int(rng.integers(0, 20_000))
    op = rng.integers(0, V, n)
    dv = rng.integers(0, G, n)
    t = rng.integers(0, 1 << (10 + 5 * (seed % 7)), n)
    if seed == 5:
        t[:] = (1 << 40) - 1  # the envelope's edge: sums near 2^64
    got = F.cost_table(V, G, op, dv, t)
    assert got.tolist() == CF.cost_table(V, G, zip(op, dv, t))


def test_cost_table_rounding_and_envelope():
    got = F.cost_table(2, 2, [0, 0, 1], [1, 1, 0], [1, 2, 7])  # mean 1.5 -> 2
    assert got.tolist() == [[0, 2], [7, 0]]
    for bad in (([2], [0], [1]), ([0], [2], [1]), ([0], [0], [-1]), ([0], [0], [1 << 40]), ([-1], [0], [1])):
        with pytest.raises(F.FasttError) as e:
            F.cost_table(2, 2, *bad)
        assert e.value.code == F.EINVAL


def test_trace_cost_table_hand_trace():
    import json
    from test_costmodel import trace as hand_trace
    ev = CM.load_trace(json.dumps(hand_trace()))
    cost = CM.cost_table(ev, {"matmul": 0, "relu": 1, "softmax": 2}, 3, 2)
    # mean 11250 ns on device 0; 1.5 ns rounds half up to 2; unknown entries 0
    assert cost.tolist() == [[11250, 11000], [0, 2], [0, 0]]


def test_committed_b200_trace_to_cost_model():
    """the trimmed torch.profiler capture from a B200: GPU cost table and host
    link fit equal the oracle's exact computations on the same samples"""
    import json
    import os
    path = os.path.join(os.path.dirname(__file__), "golden", "trace_b200_mlp2.json")
    if not os.path.exists(path):
        pytest.skip("trace not captured yet")
    obj = json.load(open(path))
    ev = CM.load_trace(obj)
    names = obj["fastt_op_names"]
    idx = {n: i for i, n in enumerate(names)}
    cost = CM.cost_table(ev, idx, len(names), 1)
    assert cost.tolist() == CF.cost_table(len(names), 1, CM.compute_samples(ev, idx))
    assert (cost[:, 0] > 0).all()
    m = CM.fit_link_model(ev, 2, host_device=1)
    smp = CM.comm_samples(ev, host_device=1)
    for s, d in ((0, 1), (1, 0)):
        grp = [(b, t) for s_, d_, b, t in smp if (s_, d_) == (s, d)]
        a_q, b_q = CF.nnls_line([b for b, _ in grp], [t for _, t in grp])
        a_ref, b_ref = CF.round_half_up(a_q), CF.round_half_up(b_q * 10**6)
        assert (int(m["pair_alpha"][s][d]), int(m["pair_beta"][s][d])) == (a_ref, b_ref)
        assert b_ref > 0  # bytes cost time over the host link
