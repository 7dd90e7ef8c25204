"""Diff one fuzz candidate GPU vs oracle (debug aid)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np
import oracle as O
from paper_conf_middleware_0001lmwlwyl20_b200 import synth, fastt as F
seed, k, flags = int(sys.argv[1]), int(sys.argv[2]), int(sys.argv[3])
src = open(os.path.join(os.path.dirname(__file__), "..", "tests", "test_gpu_parity.py")).read()
ns = {}
exec(src[src.index("def random_cands"):src.index("# ------------------------------------------------------------- hand cases")], {"np": np, "F": F}, ns)
desc = synth.random_dag(seed)
print("V", desc.n_ops, "G", desc.n_devices, "K", len(desc.alpha), "caps", desc.cap.tolist())
cands = ns["random_cands"](desc, np.random.default_rng(seed + 1), 24)
print("cand", cands[k])
gg, og = F.Graph(desc), O.OracleGraph(desc)
print("time_bits", gg.time_bits)
for sub in ([k], list(range(len(cands)))):
    res = gg.schedule_batch(cands[sub], flags=flags, placement=True, order=True, start=True)
    j = sub.index(k)
    r = og.schedule(cands[k], flags=flags)
    print("batch", len(sub), "gpu", int(res["makespan"][j]), "oracle", r["makespan"])
    V = desc.n_ops
    deq = [x for x in r["dequeue"][:V] if x >= 0]
    for t, op in enumerate(deq):
        if res["placement"][j][op] != r["placement"][op] or res["start"][j][op] != r["start"][op]:
            print(" first diff at dequeue step", t, "op", op, "gpu", res["placement"][j][op], res["start"][j][op],
                  "oracle", r["placement"][op], r["start"][op], "npred", len([1 for s, dd in zip(desc.src, desc.dst) if dd == op]))
            break
