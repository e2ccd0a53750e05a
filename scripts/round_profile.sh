#!/bin/bash
# Round evidence under gpurun: GPU tests, bench lines for C2..C5, the ncu launch list of the C5 bench command and
# one `ncu --set full` capture per hot kernel.  usage: bash scripts/round_profile.sh <tag>
TAG=${1:-r1}
OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_$TAG.log 2>&1; tail -2 $OUT/pytest_gpu_$TAG.log
for C in c5 c2 c3 c4; do
  timeout 600 python bench.py --config $C --steps 5 --warmup 3 > $OUT/bench_${C}_$TAG.json 2> $OUT/bench_${C}_$TAG.log
  tail -1 $OUT/bench_${C}_$TAG.json | cut -c1-200
done
BENCH="python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $OUT/launches_c5_$TAG.csv $BENCH > /dev/null 2>&1
for K in onesweep2 extents_kernel extract_1to1 compact_kernel; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 0 -c 1 -o $OUT/prof_c5_${TAG}_$K $BENCH > /dev/null 2>&1
done
ls $OUT | grep $TAG
