"""ncu target: fastt_schedule_batch over C5 PIN candidates (the e2e path's main
launch; peak=1 requests per-device peak memory, the lane kernel's MM 1).
usage: ncu_batch.py <n> <peak 0|1>"""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
n = int(sys.argv[1]) if len(sys.argv) > 1 else 300000
peak = len(sys.argv) > 2 and sys.argv[2] == "1"
g = F.Graph(synth.config("C5"))
gen = F.gen_params(seed=0xFA57)
ns = g.stream_info(gen, flags=F.F_CP_PIN)
c = g.generate_candidates(gen, ns + 1, n, flags=F.F_CP_PIN)
r = g.schedule_batch(c, flags=F.F_CP_PIN | F.F_TIMING, peak=peak)
print(int(r["makespan"].min()), g.last_timing())
