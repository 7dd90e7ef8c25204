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
    cost = CM.cost_table(ev, idx, 3, 2)
    # mean 11250 ns on device 0; 1.5 ns rounds half up to 2; unknown entries 0
    assert cost.tolist() == [[11250, 11000], [0, 2], [0, 0]]
    assert CM.comm_samples(ev) == [(0, 1, 4096, 3000), (1, 0, 1 << 20, 5000)]


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
