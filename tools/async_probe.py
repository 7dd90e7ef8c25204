"""Host-side timing of an asynchronous C5 sweep (FASTT_HOST_TRACE=1 prints
the library's checkpoints): how long the call takes to enqueue vs the work."""
import os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
n = int(sys.argv[1]) if len(sys.argv) > 1 else 200_000
g = F.Graph(synth.config(sys.argv[2] if len(sys.argv) > 2 else "C5"))
gen = F.gen_params(seed=0xFA57)
ref = g.sweep_best(gen, 0, n, flags=F.F_CP_PIN)
s = torch.cuda.Stream()
out = torch.empty(2, dtype=torch.int64, device="cuda")
for it in range(3):
    torch.cuda.synchronize()
    print("---- call", it, file=sys.stderr, flush=True)
    t0 = time.perf_counter()
    g.sweep_best(gen, 0, n, flags=F.F_CP_PIN | F.F_ASYNC, stream=s, out=out)
    t1 = time.perf_counter()
    g.sync(stream=s)
    t2 = time.perf_counter()
    print("enqueue %.3f ms, total %.3f ms, ok %s" % (1e3 * (t1 - t0), 1e3 * (t2 - t0), tuple(out.tolist()) == ref),
          flush=True)
