"""Launch-shape A/B of the sweep's main kernel (k_lane_pk.cuh): one or two
candidates per lane (FASTT_PK_CPL), the overlap of the main launch with the
preparation pipeline (FASTT_OVL_MODE 0/1/2, persistent or non-persistent
main launch) -- every shape must give bit-identical per-candidate makespans
and the same sweep winner, and the winner must be the oracle's makespan at
that index."""
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

SHAPES = [
    {"FASTT_PK_CPL": "1"},
    {"FASTT_PK_CPL": "2"},
    {"FASTT_PK_CPL": "2", "FASTT_OVL_MODE": "0", "FASTT_LANE_BATCHES": "1"},
    {"FASTT_PK_CPL": "2", "FASTT_OVL_MODE": "0", "FASTT_LANE_BATCHES": "3"},
    {"FASTT_PK_CPL": "2", "FASTT_OVL_MODE": "2", "FASTT_LANE_BATCHES": "0", "FASTT_MAIN_BPS": "1"},
    {"FASTT_PK_CPL": "1", "FASTT_OVL_MODE": "2", "FASTT_LANE_BATCHES": "0", "FASTT_MAIN_BPS": "2"},
    {"FASTT_PK_CPL": "2", "FASTT_NO_OVERLAP": "1"},
    {"FASTT_PK_CPL": "2", "FASTT_PK_CPL_PEAK": "0"},
    {"FASTT_PK_CPL": "2", "FASTT_PK_WPB": "1"},
    {"FASTT_PK_CPL": "4"},
    {"FASTT_NO_COST_HOLE": "1"},
    {"FASTT_NO_LVLREC": "1"},
    {"FASTT_PK_CPL": "4", "FASTT_PK_WPB": "2", "FASTT_OVL_MODE": "0", "FASTT_LANE_BATCHES": "1"},
    {"FASTT_PK_CPL": "2", "FASTT_PK_WPB": "4", "FASTT_OVL_MODE": "0", "FASTT_LANE_BATCHES": "2"},
]
KEYS = ("FASTT_PK_CPL", "FASTT_OVL_MODE", "FASTT_LANE_BATCHES", "FASTT_MAIN_BPS", "FASTT_NO_OVERLAP", "FASTT_PK_CPL_PEAK",
        "FASTT_PK_WPB", "FASTT_NO_COST_HOLE", "FASTT_NO_LVLREC")


def _graph(desc, env):
    old = {k: os.environ.get(k) for k in KEYS}
    for k in KEYS:
        os.environ.pop(k, None)
    os.environ.update(env)
    try:
        return F.Graph(desc)
    finally:
        for k, v in old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


@pytest.mark.parametrize("cfg,n", [("C5", 120_000), ("C3", 60_000), ("C1", 30_000)])
def test_shapes_agree(cfg, n):
    desc = synth.config(cfg)
    gen = F.gen_params(seed=0xFA57)
    ref_best = ref_ms = ref_peak = None
    for env in SHAPES:
        g = _graph(desc, env)
        ns = g.stream_info(gen, flags=F.F_CP_PIN)
        best = g.sweep_best(gen, 0, n, flags=F.F_CP_PIN)
        cands = g.generate_candidates(gen, 0, min(n, ns + 20_000), flags=F.F_CP_PIN)
        ms = g.schedule_batch(cands, flags=F.F_CP_PIN, peak=False)["makespan"]
        rp = g.schedule_batch(cands, flags=F.F_CP_PIN, peak=True)  # (memory mode 1 of the lane kernel)
        assert np.array_equal(rp["makespan"], ms), env
        if ref_best is None:
            ref_best, ref_ms, ref_peak = best, ms, rp["peak_mem"]
            c = g.generate_candidates(gen, best[1], 1, flags=F.F_CP_PIN)
            assert O.OracleGraph(desc).schedule(c[0], flags=O.F_CP_PIN, outputs=False)["makespan"] == best[0]
        assert best == ref_best, env
        assert np.array_equal(ms, ref_ms), env
        assert np.array_equal(rp["peak_mem"], ref_peak), env
