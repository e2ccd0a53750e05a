"""Summarise an ncu launch list (gpu__time_duration.sum [+ dram bytes]) of `bench.py`: the LAST step (from the
last extents launch on), time per kernel family and its share of the step.  Cold-cache and serialised per launch:
compare shares, not absolute times, with the bench line."""
import csv
import sys
from collections import OrderedDict, defaultdict

rows = list(csv.reader(open(sys.argv[1])))
h, L = None, OrderedDict()
for r in rows:
    if r and r[0] == "ID":
        h = r
        continue
    if h and len(r) == len(h):
        d = dict(zip(h, r))
        e = L.setdefault(d["ID"], {"name": d["Kernel Name"].split("(")[0].replace("void ", "")})
        e[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
ls = list(L.values())
# a step starts at its first pass over the records: the record sample of the fused path, else the extents pass
starts = [i for i, x in enumerate(ls) if "presample_kernel" in x["name"]]
if not starts:
    starts = [i for i, x in enumerate(ls) if "extents2" in x["name"]]
last = max(starts)
step = ls[last:]
agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0])
for x in step:
    k = x["name"][:60]
    agg[k][0] += 1
    agg[k][1] += x.get("gpu__time_duration.sum", 0) / 1e6
    agg[k][2] += x.get("dram__bytes_read.sum", 0) / 1e9
    agg[k][3] += x.get("dram__bytes_write.sum", 0) / 1e9
tot = sum(v[1] for v in agg.values())
print(f"{sys.argv[1]}: last step, {len(step)} launches, {tot:.2f} ms of kernel time (ncu, serialised)")
print(f"{'kernel':62s} {'n':>3s} {'ms':>8s} {'share':>6s} {'DRAM R GB':>10s} {'W GB':>7s}")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1]):
    print(f"{k:62s} {v[0]:3d} {v[1]:8.3f} {v[1] / tot:6.3f} {v[2]:10.3f} {v[3]:7.3f}")
