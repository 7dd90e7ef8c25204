"""Hot SASS lines of an ncu source page (--page source --csv --print-source sass):
instructions with the most warp-stall samples, and the hot loop's size.
usage: sass_hot.py <source.csv> [top]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
h = next(r for r in rows if r and r[0] == "Address")
data, seen = [], set()
for r in rows:
    if len(r) == len(h) and r[0].startswith("0x") and r[0] not in seen:
        seen.add(r[0])
        data.append(dict(zip(h, r)))
ie = lambda r: int(r["Instructions Executed"] or 0)
S = lambda r: int(r["Warp Stall Sampling (All Samples)"] or 0)
tot, smp = sum(ie(r) for r in data), sum(S(r) for r in data)
mx = max(ie(r) for r in data)
loop = [r for r in data if ie(r) >= 0.5 * mx]
print("instructions executed %d, stall samples %d, hot-loop instructions (>= half max count) %d" % (tot, smp, len(loop)))
for i, r in sorted(enumerate(data), key=lambda x: -S(x[1]))[:top]:
    print("%5d %6.2f%% exec %11d  %s" % (i, 100.0 * S(r) / smp, ie(r), r["Source"].strip()[:100]))
