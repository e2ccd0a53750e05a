"""Summarise bench.py JSON lines: value, ms/step, roofline frac and per-kernel ms.  usage: python scripts/bsum.py f..."""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:  # noqa: BLE001
        print(f, "unreadable", e)
        continue
    ks = " ".join(f"{k}={v['ms_per_step']:.2f}" for k, v in sorted(d.get("kernels", {}).items(),
                                                                     key=lambda kv: -kv[1]["ms_per_step"]))
    r = d.get("roofline", {})
    print(f"{f}: {d.get('value', 0):.2f} {d.get('unit')} {d.get('ms_per_step', 0):.2f} ms frac={r.get('frac', 0):.3f} "
          f"clk={d.get('clocks', {}).get('sm_mhz')} | {ks}")
