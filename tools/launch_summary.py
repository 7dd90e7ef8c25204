"""Aggregate an `ncu --metrics gpu__time_duration.sum --csv` launch list per kernel.
usage: launch_summary.py <launches.csv> <command string> > summary.json"""
import csv, json, re, sys
rows = [r for r in csv.reader(l for l in open(sys.argv[1]) if l.startswith('"'))]
h = rows[0]
agg = {}
for r in rows[1:]:
    d = dict(zip(h, r))
    if d.get("Metric Name") != "gpu__time_duration.sum":
        continue
    k = re.sub(r"\(.*$", "", d["Kernel Name"]).replace("void ", "")
    t = float(d["Metric Value"]) * {"ns": 1e-6, "us": 1e-3, "ms": 1.0}.get(d["Metric Unit"], 1e-6)
    a = agg.setdefault(k, [0, 0.0])
    a[0] += 1
    a[1] += t
tot = sum(v[1] for v in agg.values())
ks = sorted(agg.items(), key=lambda kv: -kv[1][1])
print(json.dumps({"command": sys.argv[2] if len(sys.argv) > 2 else "",
                  "note": "cold-cache, serialised launches under ncu: compare shares, not absolute times",
                  "kernels": [{"kernel": k, "launches": v[0], "total_ms": round(v[1], 3), "share": round(v[1] / tot, 4)}
                              for k, v in ks]}, indent=1))
