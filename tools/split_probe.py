"""Time fastt_split_search (GPU) vs the oracle's OS-DPOS on the configs."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
for name in (sys.argv[1].split(",") if len(sys.argv) > 1 else ["C1", "C2", "C3", "C4", "C5"]):
    d = synth.config(name)
    pow2 = name == "C4"
    g, og = F.Graph(d), O.OracleGraph(d)
    g.split_search(flags=F.F_CP_PIN, n_pow2_only=pow2)  # warm-up (stream/arena)
    t = time.time(); a = g.split_search(flags=F.F_CP_PIN, n_pow2_only=pow2); tg = time.time() - t
    t = time.time(); b = og.split_search(flags=O.F_CP_PIN, pow2_only=pow2); to = time.time() - t
    ok = a["sp"] == b["sp"] and a["makespan"] == b["makespan"] and (a["placement"] == b["placement"]).all() and (a["order"] == b["order"]).all()
    print(f"{name}: splits={len(a['sp'])} makespan={a['makespan']} gpu={tg:.3f}s oracle={to:.3f}s parity={ok}", flush=True)
