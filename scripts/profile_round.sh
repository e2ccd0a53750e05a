# round-end evidence: ncu launch lists (C5, C4) and --set full captures of the hot kernels; bash scripts/profile_round.sh <tag>
TAG=${1:-r2}; OUT=gpurun_out; mkdir -p $OUT
B="python bench.py --steps 2 --warmup 3 --no-e2e --no-cpu"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $OUT/launches_c5_$TAG.csv $B > /dev/null 2>&1
python scripts/launch_summary.py $OUT/launches_c5_$TAG.csv > $OUT/launches_c5_$TAG.txt 2>&1; head -16 $OUT/launches_c5_$TAG.txt
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $OUT/launches_c4_$TAG.csv $B --config c4 > /dev/null 2>&1
python scripts/launch_summary.py $OUT/launches_c4_$TAG.csv > $OUT/launches_c4_$TAG.txt 2>&1; head -16 $OUT/launches_c4_$TAG.txt
for K in extents_part onesweep2 bucket_local; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 0 -c 1 -o $OUT/prof_c5_${TAG}_$K $B > /dev/null 2>&1
done
for K in compact_seg_w conflict_kernel; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 0 -c 1 -o $OUT/prof_c4_${TAG}_$K $B --config c4 > /dev/null 2>&1
done
python scripts/ncu_summary.py $OUT/prof_c5_${TAG}_*.ncu-rep $OUT/prof_c4_${TAG}_*.ncu-rep > $OUT/ncu_summaries_$TAG.txt 2>&1
grep -E "==|duration|dram__bytes|gpu__time" $OUT/ncu_summaries_$TAG.txt | head -40
