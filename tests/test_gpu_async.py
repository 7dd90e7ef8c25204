"""The asynchronous ABI (include/fastt.h "Synchronisation"; SURVEY 8(b):
calls are asynchronous on cuda_stream, the caller synchronizes).

With FASTT_F_ASYNC, fastt_sweep_best / fastt_schedule_batch /
fastt_generate_candidates return once enqueued: the preparation rounds a
batch needs (the classified tail past the arena, the deferral queue) run as
a CUDA-graph WHILE loop whose condition is set on the device.  These tests
check that the asynchronous results equal the blocking ones (and the
oracle's), that the call returns before the device work ends, that a
multi-round loop (tail several times the arena) is exact, and that calls on
one graph issued on different streams are ordered while calls on different
graphs overlap."""
import time

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

SEED = 0xFA57


def _dev_cands(c):
    return torch.from_numpy(np.ascontiguousarray(c).view(np.uint8).reshape(len(c), 32)).cuda()


def test_async_sweep_equals_blocking_and_returns_before_the_device():
    g = F.Graph(synth.config("C5"))
    gen = F.gen_params(seed=SEED)
    n = 200_000
    ref = g.sweep_best(gen, 0, n, flags=F.F_CP_PIN)  # (also the one-time setup)
    s = torch.cuda.Stream()
    out = torch.empty(2, dtype=torch.int64, device="cuda")
    g.sweep_best(gen, 0, n, flags=F.F_CP_PIN | F.F_ASYNC, stream=s, out=out)  # builds the loop graph
    g.sync(stream=s)
    assert tuple(out.tolist()) == ref
    out.fill_(-7)
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    g.sweep_best(gen, 0, n, flags=F.F_CP_PIN | F.F_ASYNC, stream=s, out=out)
    t_enq = time.perf_counter() - t0
    g.sync(stream=s)
    t_all = time.perf_counter() - t0
    assert tuple(out.tolist()) == ref
    # nothing on the steady-state path waits for the device
    assert t_enq < 0.5 * t_all, (t_enq, t_all)
    t = g.last_timing()
    assert t["deferred"] > 0 and t["candidates"] == n


def _split_heavy_list(desc, gen, reps, n_pin):
    """the SPLIT block of the stream repeated `reps` times, then PINs: every
    SPLIT goes through the preparation pipeline"""
    og = O.OracleGraph(desc)
    gg = F.Graph(desc)
    ns = gg.stream_info(gen, flags=F.F_CP_PIN)
    sp = gg.generate_candidates(gen, 1, ns, flags=F.F_CP_PIN)
    pins = gg.generate_candidates(gen, ns + 1, n_pin, flags=F.F_CP_PIN)
    cands = np.concatenate([np.tile(sp, reps), pins])
    rng = np.random.default_rng(5)
    rng.shuffle(cands)
    want = np.array([og.schedule(c, flags=O.F_CP_PIN, outputs=False)["makespan"] for c in cands], np.int64)
    return cands, want, ns


@pytest.mark.parametrize("cfg", ["C1", "C4"])
def test_multi_round_deferral_loop(cfg):
    """more deferred candidates than the first call's arena (256 slots): the
    WHILE loop runs several rounds, blocking and asynchronous alike"""
    desc = synth.config(cfg)
    gen = F.gen_params(seed=SEED, n_pow2_only=(cfg == "C4"))
    reps = 1 + 1200 // max(1, F.Graph(desc).stream_info(gen, flags=F.F_CP_PIN))
    cands, want, ns = _split_heavy_list(desc, gen, reps, 700)
    n_split = int((cands["kind"] == F.KIND_SPLIT).sum())
    assert n_split > 2 * 256
    g = F.Graph(desc)  # fresh graph: arena sized from the default hint
    res = g.schedule_batch(cands, flags=F.F_CP_PIN, peak=False)
    assert (res["makespan"] == want).all()
    assert g.last_timing()["deferred"] >= n_split
    # the same list, asynchronous, device in/out, on a side stream
    s = torch.cuda.Stream()
    dc = _dev_cands(cands)
    out = {"makespan": torch.empty(len(cands), dtype=torch.int64, device="cuda"),
           "status": torch.empty(len(cands), dtype=torch.uint8, device="cuda")}
    g2 = F.Graph(desc)
    g2.schedule_batch(dc, flags=F.F_CP_PIN | F.F_ASYNC, stream=s, peak=False, out=out)
    g2.sync(stream=s)
    assert (out["makespan"].cpu().numpy() == want).all()
    assert g2.last_timing()["deferred"] >= n_split


def test_async_host_outputs_after_sync():
    """FASTT_F_ASYNC with numpy (pageable) outputs: valid after fastt_sync"""
    desc = synth.config("C2")
    gen = F.gen_params(seed=SEED)
    g = F.Graph(desc)
    ns = g.stream_info(gen, flags=F.F_CP_PIN)
    cands = g.generate_candidates(gen, 0, ns + 3000, flags=F.F_CP_PIN)
    ref = g.schedule_batch(cands, flags=F.F_CP_PIN)
    res = g.schedule_batch(cands, flags=F.F_CP_PIN | F.F_ASYNC)
    g.sync()
    for k in ("makespan", "status", "peak_mem"):
        assert (res[k] == ref[k]).all(), k


def test_async_generate_candidates_device():
    desc = synth.config("C3")
    gen = F.gen_params(seed=SEED)
    g = F.Graph(desc)
    host = g.generate_candidates(gen, 17, 5000, flags=F.F_CP_PIN)
    s = torch.cuda.Stream()
    out = torch.empty((5000, 32), dtype=torch.uint8, device="cuda")
    g.generate_candidates(gen, 17, 5000, flags=F.F_CP_PIN | F.F_ASYNC, stream=s, out=out)
    g.sync(stream=s)
    assert out.cpu().numpy().tobytes() == host.tobytes()


def test_same_graph_two_streams_are_ordered():
    """a sweep on stream A and a batch on stream B of the same graph share its
    scratch: the library orders them, both results are exact"""
    desc = synth.config("C3")
    gen = F.gen_params(seed=SEED)
    g = F.Graph(desc)
    ns = g.stream_info(gen, flags=F.F_CP_PIN)
    ref_best = g.sweep_best(gen, 0, 60_000, flags=F.F_CP_PIN)
    cands = g.generate_candidates(gen, 0, ns + 4000, flags=F.F_CP_PIN)
    ref = g.schedule_batch(cands, flags=F.F_CP_PIN, peak=False)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    best = torch.empty(2, dtype=torch.int64, device="cuda")
    out = {"makespan": torch.empty(len(cands), dtype=torch.int64, device="cuda"),
           "status": torch.empty(len(cands), dtype=torch.uint8, device="cuda")}
    dc = _dev_cands(cands)
    for _ in range(3):
        g.sweep_best(gen, 0, 60_000, flags=F.F_CP_PIN | F.F_ASYNC, stream=sa, out=best)
        g.schedule_batch(dc, flags=F.F_CP_PIN | F.F_ASYNC, stream=sb, peak=False, out=out)
    g.sync(stream=sa)
    g.sync(stream=sb)
    assert tuple(best.tolist()) == ref_best
    assert (out["makespan"].cpu().numpy() == ref["makespan"]).all()


def test_two_graphs_overlap_on_two_streams():
    """independent graphs on independent streams: both asynchronous sweeps in
    flight at once, each equal to its blocking result"""
    gen = F.gen_params(seed=SEED)
    ga, gb = F.Graph(synth.config("C2")), F.Graph(synth.config("C3"))
    ra = ga.sweep_best(gen, 0, 100_000, flags=F.F_CP_PIN)
    rb = gb.sweep_best(gen, 0, 50_000, flags=F.F_CP_PIN)
    sa, sb = torch.cuda.Stream(), torch.cuda.Stream()
    oa = torch.empty(2, dtype=torch.int64, device="cuda")
    ob = torch.empty(2, dtype=torch.int64, device="cuda")
    for _ in range(2):
        ga.sweep_best(gen, 0, 100_000, flags=F.F_CP_PIN | F.F_ASYNC, stream=sa, out=oa)
        gb.sweep_best(gen, 0, 50_000, flags=F.F_CP_PIN | F.F_ASYNC, stream=sb, out=ob)
    torch.cuda.synchronize()
    ga.sync(stream=sa)
    gb.sync(stream=sb)
    assert tuple(oa.tolist()) == ra and tuple(ob.tolist()) == rb


@pytest.mark.parametrize("cfg,extra,n", [("C4", "insert", 3000), ("C2", "live", 3000), ("C1", "insert", 20000)])
def test_async_other_paths(cfg, extra, n):
    """the sequential (non-overlapped) evaluations -- INSERT (R1i), liveness
    memory (R24): unsorted stream deferrals (source 2 of the loop) -- are
    asynchronous too and equal their blocking results"""
    desc = synth.config(cfg)
    gen = F.gen_params(seed=SEED, n_pow2_only=(cfg == "C4"))
    fl = F.F_CP_PIN | (F.F_POLICY_INSERT if extra == "insert" else F.F_MEM_LIVE)
    g = F.Graph(desc)
    ref = g.sweep_best(gen, 0, n, flags=fl)
    s = torch.cuda.Stream()
    out = torch.empty(2, dtype=torch.int64, device="cuda")
    for _ in range(2):
        g.sweep_best(gen, 0, n, flags=fl | F.F_ASYNC, stream=s, out=out)
    g.sync(stream=s)
    assert tuple(out.tolist()) == ref


def test_async_per_op_outputs():
    """placement / start / order outputs (an unsorted candidate list: source
    1 of the loop, and the order sort's stream-ordered scratch) on a device
    stream equal the blocking host-buffer results and the oracle's"""
    desc = synth.config("C1")
    gen = F.gen_params(seed=SEED)
    g = F.Graph(desc)
    ns = g.stream_info(gen, flags=F.F_CP_PIN)
    cands = g.generate_candidates(gen, 0, ns + 300, flags=F.F_CP_PIN)
    ref = g.schedule_batch(cands, flags=F.F_CP_PIN, placement=True, order=True, start=True)
    n, vm = len(cands), g.v_max
    out = {"makespan": torch.empty(n, dtype=torch.int64, device="cuda"),
           "status": torch.empty(n, dtype=torch.uint8, device="cuda"),
           "peak_mem": torch.empty(n * g.G, dtype=torch.int64, device="cuda"),
           "placement": torch.empty(n * vm, dtype=torch.uint8, device="cuda"),
           "order": torch.empty(n * vm, dtype=torch.int32, device="cuda"),
           "start": torch.empty(n * vm, dtype=torch.int64, device="cuda")}
    s = torch.cuda.Stream()
    g.schedule_batch(_dev_cands(cands), flags=F.F_CP_PIN | F.F_ASYNC, stream=s, out=out)
    g.sync(stream=s)
    assert (out["makespan"].cpu().numpy() == ref["makespan"]).all()
    assert (out["placement"].cpu().numpy().reshape(n, vm) == ref["placement"]).all()
    assert (out["order"].cpu().numpy().reshape(n, vm) == ref["order"]).all()
    assert (out["start"].cpu().numpy().reshape(n, vm) == ref["start"]).all()
    og = O.OracleGraph(desc)
    for k in range(0, n, 37):
        r = og.schedule(cands[k], flags=O.F_CP_PIN)
        assert int(ref["makespan"][k]) == r["makespan"]
        if r["status"] == 0:
            assert (ref["order"][k] == r["order"]).all()
