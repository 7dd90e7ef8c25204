"""CPU-side checks of the C-ABI library: it builds for sm_100a, loads, exports
every symbol include/fastt.h declares, and its host-side validation rejects
malformed graphs (no compute call needs a GPU for these paths)."""
import os
import re

import numpy as np
import pytest

from paper_conf_middleware_0001lmwlwyl20_b200 import build as B
from paper_conf_middleware_0001lmwlwyl20_b200 import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def F():
    B.build()
    from paper_conf_middleware_0001lmwlwyl20_b200 import fastt
    return fastt


def declared_symbols():
    txt = open(os.path.join(ROOT, "include", "fastt.h")).read()
    return sorted(set(re.findall(r"\b(fastt_[a-z_]+)\s*\(", txt)))


def test_header_declares_the_boundary():
    syms = declared_symbols()
    for s in ["fastt_load_graph", "fastt_rank", "fastt_schedule_batch", "fastt_split_search", "fastt_sweep_best"]:
        assert s in syms


def test_library_exports_every_declared_symbol(F):
    L = F.lib()
    for s in declared_symbols():
        assert hasattr(L, s), s
    assert set(F.SYMBOLS) == set(declared_symbols())
    assert "sm_100a" in F.version()


def test_sass_is_sm100a(F):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "-lelf", F.LIB_PATH], capture_output=True, text=True).stdout
    assert "sm_100a" in out


def _mk(V, G, edges, cost):
    return synth._finish("t", G, [e[0] for e in edges], [e[1] for e in edges], [1] * len(edges), [0] * len(edges),
                         np.asarray(cost, np.int64).reshape(V, G), [0] * V, [0] * V, [0] * V)


def test_load_validation_errors(F):
    with pytest.raises(F.FasttError) as e:
        F.Graph(_mk(3, 2, [(0, 1), (1, 2), (2, 0)], np.ones((3, 2))))
    assert e.value.code == F.ECYCLE
    with pytest.raises(F.FasttError) as e:
        F.Graph(_mk(2, 2, [(0, 0)], np.ones((2, 2))))
    assert e.value.code == F.ECYCLE
    with pytest.raises(F.FasttError) as e:
        F.Graph(_mk(2, 2, [(0, 1)], [[1, 1], [1, -1]]))
    assert e.value.code == F.EINVAL
    d = _mk(2, 2, [(0, 1)], np.ones((2, 2)))
    d.n_devices = 33
    with pytest.raises(F.FasttError) as e:
        F.Graph(d)
    assert e.value.code == F.EINVAL
    d = _mk(2, 2, [(0, 1)], np.ones((2, 2)))
    d.link_class = np.full((2, 2), 3, np.uint8)
    with pytest.raises(F.FasttError) as e:
        F.Graph(d)
    assert e.value.code == F.EINVAL
    d = _mk(2, 2, [(0, 1)], np.ones((2, 2)))
    d.cost = np.full((2, 2), 1 << 60, np.int64)
    with pytest.raises(F.FasttError) as e:
        F.Graph(d)
    assert e.value.code == F.ERANGE
    # bytes * split_copy_fs_per_byte (R13 split/concat node cost) must stay in int64
    d = _mk(2, 2, [(0, 1)], np.ones((2, 2)))
    d.bytes = np.array([1 << 40], np.int64)
    d.beta = np.array([0], np.int64)
    d.copy_fs = 1 << 22
    with pytest.raises(F.FasttError) as e:
        F.Graph(d)
    assert e.value.code == F.ERANGE


def test_no_cpu_fallback_without_device(F):
    """A valid graph needs a device; without one the call fails loudly."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    with pytest.raises(F.FasttError) as e:
        F.Graph(synth.diamond())
    assert e.value.code == F.ECUDA
