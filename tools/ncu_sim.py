"""ncu target: one main-sweep k_sim launch on C5 over PIN candidates only.
k_sim launch #0 = the BASE run of stream_info, #1 = the sweep (use -s 1 -c 1)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
n = int(sys.argv[1]) if len(sys.argv) > 1 else 20000
cfg = sys.argv[2] if len(sys.argv) > 2 else "C5"
g = F.Graph(synth.config(cfg))
gen = F.gen_params(seed=0xFA57)
ns = g.stream_info(gen, flags=F.F_CP_PIN)
print(g.sweep_best(gen, ns + 1, n, flags=F.F_CP_PIN | F.F_TIMING), g.last_timing())
