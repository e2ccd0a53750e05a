#!/bin/bash
# ncu evidence for the bench: launch list (per-launch device times) + one --set full capture per hot kernel.
# usage (under gpurun): bash scripts/profile.sh <config> <n> <tag> [kernel regexes...]
set -u
CFG=${1:-c5}; N=${2:-100000000}; TAG=${3:-r1}; shift 3
KS=${@:-onesweep extract_1to1 compact_multi extents_kernel}
OUT=gpurun_out; mkdir -p $OUT
BENCH="python bench.py --config $CFG --records $N --steps 1 --warmup 1 --no-e2e --no-cpu"
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_${CFG}_${TAG}.csv $BENCH > /dev/null 2>&1
for K in $KS; do
  ncu --set full --clock-control none --import-source on -k regex:$K -s 0 -c 1 -o $OUT/prof_${CFG}_${TAG}_${K} $BENCH > /dev/null 2>&1
done
ls $OUT | grep $TAG
