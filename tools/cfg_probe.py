import os, sys, time
sys.path.insert(0, "/root/repo")
import torch
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
GEN = 0xFA57
st = torch.cuda.current_stream()
g5 = F.Graph(synth.config("C5")); gen = F.gen_params(seed=GEN); g5.stream_info(gen, flags=F.F_CP_PIN)
for _ in range(3): g5.sweep_best(gen, 0, 1_000_000, flags=F.F_CP_PIN, stream=st)
for name, n in (("C1", 1_000_000), ("C2", 300_000), ("C3", 200_000), ("C4", 300_000), ("C5R8", 200_000)):
    g2 = F.Graph(synth.config(name)); gen2 = F.gen_params(seed=GEN, n_pow2_only=(name == "C4"))
    g2.stream_info(gen2, flags=F.F_CP_PIN, stream=st)
    for k in range(4):
        torch.cuda.synchronize(); t = time.perf_counter()
        g2.sweep_best(gen2, 0, n, flags=F.F_CP_PIN | F.F_TIMING, stream=st)
        el = time.perf_counter() - t; tm = g2.last_timing()
        print(name, k, "wall %.1f ms device %.1f ms launches %d" % (1e3 * el, tm["ms_total"], tm["launches"]), flush=True)
    del g2
