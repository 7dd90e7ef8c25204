"""Multi-rank sweep through bench.py's own N > 1 path:
torchrun starts 2 ranks (FASTT_DIST_BACKEND=gloo so both ranks share the one
GPU of the test box), rank r sweeps the global indices c = r (mod 2) of
[0, 2S) with fastt_sweep_best, and the all_reduce(MIN) pair of combine_best
picks the winner.  It must equal the single-GPU sweep over the same window,
and both must equal the oracle's makespan at that index."""
import json
import os
import socket
import subprocess
import sys

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

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_bench_two_ranks_equals_single_sweep():
    S = 20_000  # candidates per rank
    env = dict(os.environ, FASTT_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"), "--gpus", "2", "--steps", "1",
           "--warmup", "3", "--candidates", str(S), "--no-e2e", "--no-cpu", "--no-configs"]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [ln for ln in out.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, out.stdout[-2000:]  # rank 0 alone prints
    line = json.loads(lines[0])
    assert line["n_gpus"] == 2 and line["scaling"] == "weak"
    best = (line["best"]["makespan_ns"], line["best"]["index"])
    desc = synth.config("C5")
    g = F.Graph(desc)
    gen = F.gen_params(seed=0xFA57, pin_k_min=1, pin_k_max=4)
    assert g.sweep_best(gen, 0, 2 * S, flags=F.F_CP_PIN) == best
    c = g.generate_candidates(gen, best[1], 1, flags=F.F_CP_PIN)
    assert O.OracleGraph(desc).schedule(c[0], flags=O.F_CP_PIN, outputs=False)["makespan"] == best[0]
