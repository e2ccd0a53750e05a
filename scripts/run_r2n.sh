OUT=gpurun_out; mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_r2n.log 2>&1; tail -3 $OUT/pytest_gpu_r2n.log
timeout 600 python bench.py > $OUT/bench_c5_r2n.json 2> $OUT/bench_c5_r2n.log; python scripts/bsum.py $OUT/bench_c5_r2n.json
for C in c3 c4 c2; do timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu > $OUT/bench_${C}_r2n.json 2> $OUT/bench_${C}_r2n.log; python scripts/bsum.py $OUT/bench_${C}_r2n.json; done
