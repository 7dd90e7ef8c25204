"""Time fastt_split_search (GPU) vs the oracle on the configs.

usage: split_probe.py [C1,C2,...] [--best] [--no-oracle]
  --best       best-improvement variant (FASTT_F_SPLIT_BEST, NEXT N2)
  --no-oracle  GPU timing only (C3/C5 best-improvement oracle takes minutes)
"""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle as O
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
args = [a for a in sys.argv[1:] if not a.startswith("--")]
best = "--best" in sys.argv
use_oracle = "--no-oracle" not in sys.argv
for name in (args[0].split(",") if args else ["C1", "C2", "C3", "C4", "C5"]):
    d = synth.config(name)
    pow2 = name == "C4"
    g = F.Graph(d)
    g.split_search(flags=F.F_CP_PIN, n_pow2_only=pow2)  # warm-up (stream/arena)
    t = time.time(); a = g.split_search(flags=F.F_CP_PIN, n_pow2_only=pow2, best_improvement=best); tg = time.time() - t
    line = f"{name}{' BI' if best else ''}: splits={a['sp']} makespan={a['makespan']} gpu={tg:.3f}s"
    if use_oracle:
        og = O.OracleGraph(d)
        t = time.time(); b = og.split_search(flags=O.F_CP_PIN, pow2_only=pow2, best_improvement=best); to = time.time() - t
        ok = a["sp"] == b["sp"] and a["makespan"] == b["makespan"] and (a["placement"] == b["placement"]).all() and (a["order"] == b["order"]).all()
        line += f" oracle={to:.3f}s parity={ok}"
    print(line, flush=True)
