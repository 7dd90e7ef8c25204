"""Throughput of the per-candidate preparation path: heterogeneous device
costs make every PIN candidate change ranks (hetero_ppm jitter)."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
name = sys.argv[1] if len(sys.argv) > 1 else "C5"
n = int(sys.argv[2]) if len(sys.argv) > 2 else 20000
d = synth.config(name, hetero_ppm=20000)
g = F.Graph(d)
gen = F.gen_params(seed=0xFA57)
ns = g.stream_info(gen, flags=F.F_CP_PIN)
g.sweep_best(gen, 0, 2000, flags=F.F_CP_PIN)
t = time.time(); b = g.sweep_best(gen, 0, n, flags=F.F_CP_PIN | F.F_TIMING); el = time.time() - t
print(name, "hetero n", n, "best", b, "wall %.3f s" % el, "cand/s %.0f" % (n / el), g.last_timing())
