OUT=gpurun_out; mkdir -p $OUT
for C in c2 c3 c4 c5; do timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu > $OUT/bench_${C}_r2s.json 2> $OUT/bench_${C}_r2s.log; python scripts/bsum.py $OUT/bench_${C}_r2s.json; done
bash scripts/profile_r2s.sh r2s
