"""Summarise an ncu launch list of scripts/loopback_profile.py: kernel time per virtual rank by family."""
import csv
import sys
from collections import OrderedDict, defaultdict

rows = list(csv.reader(open(sys.argv[1])))
W = int(sys.argv[2]) if len(sys.argv) > 2 else 8
h, L = None, OrderedDict()
for r in rows:
    if r and r[0] == "ID":
        h = r
        continue
    if h and len(r) == len(h):
        d = dict(zip(h, r))
        e = L.setdefault(d["ID"], {"name": d["Kernel Name"].split("(")[0].replace("void ", "")[:44]})
        e[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
agg = defaultdict(lambda: [0, 0.0])
for it in L.values():
    if it["name"].startswith(("k_c5", "gen")):
        continue
    agg[it["name"]][0] += 1
    agg[it["name"]][1] += it.get("gpu__time_duration.sum", 0) / 1e6
tot = sum(v[1] for v in agg.values())
print(f"kernel time, all {W} virtual ranks: {tot:.2f} ms; per rank {tot / W:.3f} ms")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
    if v[1] / W >= 0.005:
        print(f"  {k:46s} launches {v[0]:4d}  per rank {v[1] / W:7.3f} ms")
