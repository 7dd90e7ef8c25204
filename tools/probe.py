"""Quick throughput probe (not the bench): sweep_best timing per config."""
import sys, time, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
from paper_conf_middleware_0001lmwlwyl20_b200 import build as B, synth
B.build()
from paper_conf_middleware_0001lmwlwyl20_b200 import fastt as F
args = [a for a in sys.argv[1:] if not a.startswith("--")]
cfgs = args[0].split(",") if len(args) > 0 else ["C5"]
ns = [int(x) for x in args[1].split(",")] if len(args) > 1 else [20000, 100000]
FL = F.F_CP_PIN | (F.F_POLICY_INSERT if "--insert" in sys.argv else 0)
for name in cfgs:
    d = synth.config(name)
    t = time.time(); g = F.Graph(d); tl = time.time() - t
    gen = F.gen_params(seed=0xFA57, n_pow2_only=(name == "C4"))
    t = time.time(); nsp = g.stream_info(gen, flags=FL); ts = time.time() - t
    print(f"{name}: V={g.V} vmax={g.v_max} cp={g.cp_len} tbits={g.time_bits} n_split={nsp} load={tl:.2f}s stream={ts:.2f}s", flush=True)
    for n in ns:
        g.sweep_best(gen, 0, min(n, 2000), flags=FL)
        t = time.time(); best = g.sweep_best(gen, 0, n, flags=FL | F.F_TIMING); el = time.time() - t
        tm = g.last_timing()
        fast = n - tm["deferred"]
        print(f"  n={n} best={best} wall={el:.3f}s cand/s={n/el:.0f} sim={tm['ms_sim']:.1f}ms ({fast/(tm['ms_sim']/1e3+1e-9):.0f} fast cand/s) prep={tm['ms_prep']:.1f}ms deferred={tm['deferred']} launches={tm['launches']} total={tm['ms_total']:.1f}ms", flush=True)
