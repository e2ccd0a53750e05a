"""Top stall-sampled SASS lines of an ncu source-page CSV: python scripts/sass_hot.py file.csv [N]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
h = rows[1]
ia, isrc, iss = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)")
iex = h.index("Instructions Executed")
data = []
for r in rows[2:]:
    try:
        data.append((int(r[iss]), r[ia][-5:], r[isrc].strip(), int(r[iex] or 0)))
    except (ValueError, IndexError):
        pass
tot = sum(d[0] for d in data)
print("total samples", tot, "instructions", sum(d[3] for d in data))
for d in sorted(data, reverse=True)[: int(sys.argv[2]) if len(sys.argv) > 2 else 40]:
    print(f"{d[0]:8d} {100 * d[0] / tot:5.1f}% {d[1]} {d[2][:90]:90s} x{d[3]}")
