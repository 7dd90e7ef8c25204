"""FASTT_HOST_TRACE=1 checkpoints of repeated sweeps on one config (where a
blocking call spends host time). usage: host_probe.py <config> <n>"""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
name, n = sys.argv[1], int(sys.argv[2])
g = F.Graph(synth.config(name)); gen = F.gen_params(seed=0xFA57, n_pow2_only=(name == "C4"))
g.stream_info(gen, flags=F.F_CP_PIN)
for k in range(3):
    print("---- call", k, file=sys.stderr, flush=True)
    t = time.perf_counter(); g.sweep_best(gen, 0, n, flags=F.F_CP_PIN); print("wall %.1f ms" % (1e3 * (time.perf_counter() - t)), file=sys.stderr, flush=True)
