"""Host side of the cost-model ingestion: trace parsing, the
computation cost table, fastt_link_model (host-only C-ABI call) and the
fit's argument validation.  CPU only."""
import json

import numpy as np
import pytest

from paper_conf_middleware_0001lmwlwyl20_b200 import build as B

B.build()
from paper_conf_middleware_0001lmwlwyl20_b200 import costmodel as CM  # noqa: E402
from paper_conf_middleware_0001lmwlwyl20_b200 import fastt as F  # noqa: E402


def trace():
    ev = [
        {"ph": "X", "cat": "kernel", "name": "matmul", "dur": 10.0, "args": {"device": 0}},
        {"ph": "X", "cat": "kernel", "name": "matmul", "dur": 12.5, "args": {"device": 0}},
        {"ph": "X", "cat": "kernel", "name": "matmul", "dur": 11.0, "args": {"device": 1}},
        {"ph": "X", "cat": "kernel", "name": "relu", "dur": 0.0015, "args": {"device": 1}},
        {"ph": "X", "cat": "kernel", "name": "not_in_graph", "dur": 99.0, "args": {"device": 0}},
        {"ph": "i", "cat": "kernel", "name": "matmul", "args": {"device": 0}},
        {"ph": "X", "cat": "gpu_memcpy", "name": "Memcpy PtoP", "dur": 3.0,
         "args": {"src_device": 0, "dst_device": 1, "bytes": 4096}},
        {"ph": "X", "cat": "gpu_memcpy", "name": "Memcpy PtoP", "dur": 5.0,
         "args": {"device": 1, "dst_device": 0, "bytes": 1 << 20}},
        {"ph": "X", "cat": "gpu_memcpy", "name": "Memcpy DtoD", "dur": 1.0,
         "args": {"src_device": 1, "dst_device": 1, "bytes": 64}},
    ]
    return {"traceEvents": ev}


def test_trace_parsing_and_cost_table():
    ev = CM.load_trace(json.dumps(trace()))
    idx = {"matmul": 0, "relu": 1, "softmax": 2}
    assert sorted(CM.compute_samples(ev, idx)) == [(0, 0, 10000), (0, 0, 12500), (0, 1, 11000), (1, 1, 2)]
    assert CM.comm_samples(ev) == [(0, 1, 4096, 3000), (1, 0, 1 << 20, 5000)]
    # (the averaging itself runs in the library: tests/test_gpu_fit.py)


def test_kineto_copy_kinds():
    """torch.profiler (Kineto) memcpy events carry the copy kind in the name
    and the GPU in args.device: HtoD / DtoH are transfers over the host link
    when the host has a device index, same-device copies never are"""
    ev = [{"ph": "X", "cat": "gpu_memcpy", "name": "Memcpy HtoD (Pinned -> Device)", "dur": 2.5,
           "args": {"device": 0, "bytes": 1 << 16}},
          {"ph": "X", "cat": "gpu_memcpy", "name": "Memcpy DtoH (Device -> Pinned)", "dur": 3.0,
           "args": {"device": 0, "bytes": 1 << 17}},
          {"ph": "X", "cat": "gpu_memcpy", "name": "Memcpy DtoD (Device -> Device)", "dur": 1.0,
           "args": {"device": 0, "bytes": 64}},
          {"ph": "X", "cat": "gpu_memset", "name": "Memset (Device)", "dur": 1.0, "args": {"device": 0, "bytes": 64}}]
    assert CM.comm_samples(ev) == []
    assert CM.comm_samples(ev, host_device=1) == [(1, 0, 1 << 16, 2500), (0, 1, 1 << 17, 3000)]


def test_committed_b200_trace_parses():
    """the trimmed torch.profiler capture from a B200 (tests/golden/
    trace_b200_mlp2.json, tools/capture_trace.py): every op of the C1 graph
    has GPU-side samples under its record_function name, and the host link
    has transfer samples of several sizes in both directions"""
    import os
    from paper_conf_middleware_0001lmwlwyl20_b200 import synth
    path = os.path.join(os.path.dirname(__file__), "golden", "trace_b200_mlp2.json")
    if not os.path.exists(path):
        pytest.skip("trace not captured yet")
    obj = json.load(open(path))
    ev = CM.load_trace(obj)
    desc = synth.config("C1")
    idx = {n: i for i, n in enumerate(obj["fastt_op_names"])}
    assert len(idx) == desc.n_ops
    smp = CM.compute_samples(ev, idx)
    assert {op for op, _, _ in smp} == set(range(desc.n_ops))
    assert all(d == 0 and t >= 0 for _, d, t in smp)
    cs = CM.comm_samples(ev, host_device=1)
    assert {(s, d) for s, d, _, _ in cs} == {(0, 1), (1, 0)}
    assert len({b for _, _, b, _ in cs}) >= 4


def test_link_model_groups_pairs():
    a = np.array([[0, 5, 5, 9], [5, 0, 5, 9], [5, 5, 0, 9], [9, 9, 9, 0]])
    b = np.array([[0, 1, 1, 7], [1, 0, 1, 7], [1, 1, 0, 7], [7, 7, 7, 0]])
    lc, ka, kb = F.link_model(a, b)
    assert ka.tolist() == [5, 9] and kb.tolist() == [1, 7]
    assert lc.tolist() == [[0, 0, 0, 1], [0, 0, 0, 1], [0, 0, 0, 1], [1, 1, 1, 0]]
    lc, ka, kb = F.link_model(np.zeros((1, 1)), np.zeros((1, 1)))
    assert lc.tolist() == [[0]] and ka.tolist() == [0] and kb.tolist() == [0]
    # 17 distinct pairs exceed K <= 16
    G = 5
    a = np.arange(G * G).reshape(G, G)
    with pytest.raises(F.FasttError) as e:
        F.link_model(a, np.zeros((G, G)))
    assert e.value.code == F.EUNSUP
    with pytest.raises(F.FasttError):
        F.link_model(-np.ones((2, 2)), np.zeros((2, 2)))


def test_fit_comm_argument_checks():
    with pytest.raises(F.FasttError) as e:
        F.fit_comm(0, [], [], [], [])
    assert e.value.code == F.EINVAL
    with pytest.raises(F.FasttError):
        F.fit_comm(33, [], [], [], [])
    with pytest.raises(ValueError):
        F.fit_comm(2, [0], [1, 1], [1], [1])
