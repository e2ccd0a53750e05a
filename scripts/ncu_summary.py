"""Key metrics of every kernel in an ncu --set full report (for profiles/): duration, DRAM bytes, instructions,
occupancy, registers, the top warp-stall reasons."""
import csv
import io
import subprocess
import sys

for rep in sys.argv[1:]:
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(raw)))
    h, units = r[0], dict(zip(r[0], r[1]))
    scale = {"ns": 1e-6, "us": 1e-3, "usecond": 1e-3, "msecond": 1.0, "ms": 1.0, "nsecond": 1e-6, "second": 1e3,
             "byte": 1e-9, "Kbyte": 1e-6, "Mbyte": 1e-3, "Gbyte": 1.0, "Tbyte": 1e3}
    print(f"== {rep}")
    for row in r[2:]:
        d = dict(zip(h, row))

        def f(k, norm=False):  # norm: ms for times, GB for bytes
            try:
                v = float(d.get(k, "nan").replace(",", ""))
            except ValueError:
                return float("nan")
            return v * scale.get(units.get(k, ""), 1.0) if norm else v
        print(f"  {d['Kernel Name'][:70]}")
        print(f"    duration {f('gpu__time_duration.sum', True):.3f} ms | DRAM read {f('dram__bytes_read.sum', True):.2f} GB"
              f" write {f('dram__bytes_write.sum', True):.2f} GB | warp instructions {f('smsp__inst_executed.sum') / 1e6:.0f} M"
              f" | regs {f('launch__registers_per_thread'):.0f} | warps active {f('sm__warps_active.avg.pct_of_peak_sustained_active'):.1f}%"
              f" | issue active {f('smsp__issue_active.avg.pct_of_peak_sustained_active'):.1f}%"
              f" | L2 tex read sectors {f('lts__t_sectors_srcunit_tex_op_read.sum') / 1e6:.0f} M")
        st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): f(k) for k in h
              if k.startswith("smsp__pcsamp_warps_issue_stalled") and not k.endswith("not_issued")}
        tot = sum(v for v in st.values() if v == v)
        top = sorted(((v, k) for k, v in st.items() if v == v), reverse=True)[:5]
        print("    stalls: " + ", ".join(f"{k} {v / tot:.0%}" for v, k in top))
