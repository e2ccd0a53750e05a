"""Stall reasons by SASS region of an ncu source-page CSV: python scripts/sass_stalls.py file.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
reasons = [x for x in h if x.startswith("stall_") and "Not Issued" not in x]
ia, isrc = h.index("Address"), h.index("Source")
tot = {r: 0 for r in reasons}
lines = []
for r in rows[2:]:
    try:
        v = {k: int(r[h.index(k)] or 0) for k in reasons}
    except (ValueError, IndexError):
        continue
    for k in reasons:
        tot[k] += v[k]
    lines.append((sum(v.values()), r[ia][-5:], r[isrc].strip(), v))
T = sum(tot.values())
print("by reason:", ", ".join(f"{k[6:]}={100 * x / T:.1f}%" for k, x in sorted(tot.items(), key=lambda kv: -kv[1]) if x))
for s, a, src, v in sorted(lines, reverse=True)[: int(sys.argv[2]) if len(sys.argv) > 2 else 25]:
    top = ", ".join(f"{k[6:]}={x}" for k, x in sorted(v.items(), key=lambda kv: -kv[1])[:3] if x)
    print(f"{100 * s / T:5.1f}% {a} {src[:60]:60s} {top}")
