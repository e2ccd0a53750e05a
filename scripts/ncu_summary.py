"""Summarise ncu reports: python scripts/ncu_summary.py gpurun_out/prof_*.ncu-rep"""
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem", "smsp__inst_executed.sum"]


def summary(path, extra=False):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    if len(rows) < 3:
        return {}
    h, units, v = rows[0], rows[1], rows[2]
    d = {k: f"{v[h.index(k)]} {units[h.index(k)]}".strip() for k in KEYS if k in h}
    d["kernel"] = v[h.index("Kernel Name")] if "Kernel Name" in h else "?"
    if extra:
        for i, name in enumerate(h):
            if ("pipe" in name and "inst_executed" in name and name.endswith("avg.pct_of_peak_sustained_active")) or \
                    (name.startswith("smsp__average_warps_issue_stalled") and name.endswith("per_issue_active.ratio")):
                try:
                    if float(v[i]) > 0.5:
                        d[name] = v[i]
                except ValueError:
                    pass
    return d


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print("==", p)
        for k, val in summary(p, extra=True).items():
            print(f"  {k}: {val}")
