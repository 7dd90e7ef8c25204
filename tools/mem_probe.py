"""C5R8 sweeps with and without a resident C5 graph (the bench's order):
per-sweep device time, launches, deferred, and free device memory."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
def run(name, n, reps=3):
    g = F.Graph(synth.config(name))
    gen = F.gen_params(seed=0xFA57)
    g.stream_info(gen, flags=F.F_CP_PIN)
    for _ in range(reps):
        g.sweep_best(gen, 0, n, flags=F.F_CP_PIN | F.F_TIMING)
        t = g.last_timing()
        print(name, "total %.1f ms sim %.1f prep %.1f launches %d deferred %d free %.1f GB" % (
            t["ms_total"], t["ms_sim"], t["ms_prep"], t["launches"], t["deferred"],
            torch.cuda.mem_get_info()[0] / 1e9), flush=True)
    return g
run("C5R8", 200_000)
g5 = run("C5", 1_000_000)
run("C5R8", 200_000)
