#!/bin/bash
# quick A/B under gpurun: usage: bash scripts/exp.sh "ENV=.. ENV2=..;ENV=.." [config] [tests]
OUT=gpurun_out; mkdir -p $OUT
CFG=${2:-c5}
if [ -n "$3" ]; then timeout 900 python -m pytest $3 -q -x > $OUT/exp_tests.log 2>&1; tail -3 $OUT/exp_tests.log; fi
IFS=';' read -ra VS <<< "$1"
i=0
for V in "${VS[@]}"; do
  env $V timeout 300 python bench.py --config $CFG --steps 5 --warmup 3 --no-e2e --no-cpu > $OUT/exp_$i.json 2> $OUT/exp_$i.log
  echo "[$V]"; python scripts/bsum.py $OUT/exp_$i.json; grep -i "error\|truth\|mismatch" $OUT/exp_$i.log | head -3
  i=$((i+1))
done
