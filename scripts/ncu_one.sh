#!/bin/bash
# one ncu --set full capture of a kernel of a bench command; usage: bash scripts/ncu_one.sh <regex> <tag> [env] [config]
OUT=gpurun_out; mkdir -p $OUT
env $3 timeout 900 ncu --set full --clock-control none --import-source on -k regex:$1 -s 0 -c 1 -o $OUT/prof_$2 \
  python bench.py --config ${4:-c5} --steps 1 --warmup 0 --no-e2e --no-cpu > $OUT/ncu_$2.log 2>&1
ncu -i $OUT/prof_$2.ncu-rep --page raw --csv > $OUT/prof_$2.csv 2>/dev/null
python scripts/ncu_summary.py $OUT/prof_$2.ncu-rep 2>/dev/null | head -40
ncu -i $OUT/prof_$2.ncu-rep --page source --csv --print-source sass > $OUT/prof_$2_sass.csv 2>/dev/null
ls -la $OUT/prof_$2_sass.csv
