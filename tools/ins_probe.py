"""wall vs device time of repeated C5 INSERT sweeps (R1i), 100k candidates."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
g = F.Graph(synth.config(sys.argv[1] if len(sys.argv) > 1 else "C5"))
gen = F.gen_params(seed=0xFA57)
fl = F.F_CP_PIN | F.F_POLICY_INSERT
g.stream_info(gen, flags=fl)
for k in range(4):
    t = time.perf_counter(); g.sweep_best(gen, 0, 100_000, flags=fl | F.F_TIMING); el = time.perf_counter() - t
    tm = g.last_timing()
    print(k, "wall %.1f ms device %.1f ms sim %.1f prep %.1f launches %d deferred %d" % (1e3 * el, tm["ms_total"], tm["ms_sim"], tm["ms_prep"], tm["launches"], tm["deferred"]), flush=True)
