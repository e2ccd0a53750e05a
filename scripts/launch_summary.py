"""Summarise an ncu --metrics launch list (csv log): per-kernel launches, device time, DRAM bytes, and share.
usage: python scripts/launch_summary.py gpurun_out/launches_*.csv"""
import csv
import sys


def summarise(path):
    lines = [l for l in open(path) if not l.startswith("==")]
    rows = list(csv.reader(lines))
    h = rows[0]
    name, mn, mv, idc = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
    mu = h.index("Metric Unit")
    scale = {"nsecond": 1.0, "usecond": 1e3, "msecond": 1e6, "second": 1e9, "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6,
             "Gbyte": 1e9}
    per = {}
    for r in rows[1:]:
        if len(r) <= mv:
            continue
        per.setdefault((r[idc], r[name].split("(")[0].replace("void ", "")[:48]), {})[r[mn]] = \
            float(r[mv].replace(",", "")) * scale.get(r[mu], 1.0)
    tot = {}
    for (_, k), m in per.items():
        t = tot.setdefault(k, [0, 0.0, 0.0, 0.0])
        t[0] += 1
        t[1] += m.get("gpu__time_duration.sum", 0)  # ns
        t[2] += m.get("dram__bytes_read.sum", 0)
        t[3] += m.get("dram__bytes_write.sum", 0)
    alltime = sum(t[1] for t in tot.values())
    out = []
    for k, t in sorted(tot.items(), key=lambda x: -x[1][1]):
        out.append(f"{k:50s} {t[0]:4d} launches {t[1] / 1e6:9.3f} ms {100 * t[1] / alltime:5.1f}%  "
                   f"dram rd {t[2] / 1e9:7.2f} GB wr {t[3] / 1e9:7.2f} GB")
    return out


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print("==", p)
        print("\n".join(summarise(p)))
