"""Per-call wall time of the bench's e2e batch (host pinned buffers, makespan +
status + per-device peak memory): variance check."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
g = F.Graph(synth.config("C5"))
gen = F.gen_params(seed=0xFA57)
g.stream_info(gen, flags=F.F_CP_PIN)
for _ in range(3):
    g.sweep_best(gen, 0, 1_000_000, flags=F.F_CP_PIN)
c = g.generate_candidates(gen, 0, 1_000_000, flags=F.F_CP_PIN)
hc = torch.from_numpy(c.view(np.uint8).reshape(-1, 32).copy()).pin_memory()
n = len(c)
out = {"makespan": torch.empty(n, dtype=torch.int64).pin_memory(), "status": torch.empty(n, dtype=torch.uint8).pin_memory(),
       "peak_mem": torch.empty((n, 8), dtype=torch.int64).pin_memory()}
hcn = hc.numpy().view(F.CANDIDATE_DTYPE).reshape(-1)
outn = {k: v.numpy() for k, v in out.items()}
for k in range(8):
    torch.cuda.synchronize(); t = time.perf_counter()
    g.schedule_batch(hcn, flags=F.F_CP_PIN | F.F_TIMING, out=outn)
    el = time.perf_counter() - t
    tm = g.last_timing()
    print("call %d: %.1f ms wall, device total %.1f ms, main %.1f ms" % (k, 1e3 * el, tm["ms_total"], tm["ms_sim"]), flush=True)
