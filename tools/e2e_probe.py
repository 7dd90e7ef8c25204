"""e2e probe: fastt_schedule_batch over the C5 stream window with host
buffers (makespan, status, peak), timed per call, with last_timing."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
n = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
g = F.Graph(synth.config("C5"))
gen = F.gen_params(seed=0xFA57, pin_k_min=1, pin_k_max=4)
g.stream_info(gen, flags=F.F_CP_PIN)
c = g.generate_candidates(gen, 0, n, flags=F.F_CP_PIN)
for peak in (False, True):
    for k in range(3):
        t = time.time()
        r = g.schedule_batch(c, flags=F.F_CP_PIN | F.F_TIMING, peak=peak)
        el = time.time() - t
        print("peak", peak, "call %.1f ms" % (1000 * el), g.last_timing())
