#!/bin/bash
# Round evidence under gpurun: GPU tests, bench lines for C5 (with e2e + CPU baseline) and C2..C4, the ncu launch
# list of the C5 bench command and one `ncu --set full` capture per hot kernel.  usage: bash scripts/round_profile.sh <tag>
TAG=${1:-r1}
OUT=gpurun_out; mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_$TAG.log 2>&1; tail -2 $OUT/pytest_gpu_$TAG.log
timeout 900 python bench.py --config c5 --steps 5 --warmup 3 > $OUT/bench_c5_$TAG.json 2> $OUT/bench_c5_$TAG.log
python scripts/bsum.py $OUT/bench_c5_$TAG.json
for C in c2 c3 c4; do
  timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu > $OUT/bench_${C}_$TAG.json 2> $OUT/bench_${C}_$TAG.log
  python scripts/bsum.py $OUT/bench_${C}_$TAG.json
done
BENCH="python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $OUT/launches_c5_$TAG.csv $BENCH > /dev/null 2>&1
python scripts/launch_summary.py $OUT/launches_c5_$TAG.csv > $OUT/launches_c5_$TAG.txt 2>&1; head -20 $OUT/launches_c5_$TAG.txt
for K in onesweep2 fused_extract extents2 compact_seg; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 0 -c 1 -o $OUT/prof_c5_${TAG}_$K $BENCH > /dev/null 2>&1
done
python scripts/ncu_summary.py $OUT/prof_c5_${TAG}_*.ncu-rep > $OUT/ncu_summaries_$TAG.txt 2>&1
ls $OUT | grep $TAG
