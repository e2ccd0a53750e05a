# onesweep configuration sweep on C5 (SESA_SORT_CFG); usage: bash scripts/sort_sweep.sh "cfgs" "prof cfgs"
for c in $1; do
  SESA_SORT_CFG=$c timeout 300 python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu > gpurun_out/sw_$c.json 2> gpurun_out/sw_$c.log
  python - "$c" <<'PY'
import json, sys
c = sys.argv[1]
d = json.loads(open(f"gpurun_out/sw_{c}.json").read().strip().splitlines()[-1]); k = d["kernels"]["onesweep_pass"]
print("cfg", c, round(d["value"], 2), "Grec/s", round(d["ms_per_step"], 2), "ms; onesweep", round(k["ms_per_step"], 2), "ms",
      round(d["roofline"]["frac"], 3), d["clocks"]["sm_mhz"], d["clocks"]["reasons"])
PY
  grep -i "truth\|error" gpurun_out/sw_$c.log | head -2
done
for c in $2; do echo "prof cfg $c"; SESA_SORT_CFG=$c SESA_SORT_PROF=1 timeout 300 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu 2>&1 >/dev/null | grep sortprof | tail -2; done
