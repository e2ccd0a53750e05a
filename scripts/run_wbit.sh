OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_wbit.py tests/test_gpu_parity.py -m gpu -q -x -k "wbit or write_bit or fused or long_write or random" > $OUT/pytest_wbit.log 2>&1; tail -3 $OUT/pytest_wbit.log
for C in c4 c3; do timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu > $OUT/bench_${C}_wb.json 2> $OUT/bench_${C}_wb.log; python scripts/bsum.py $OUT/bench_${C}_wb.json; done
timeout 1200 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_sweep.py -m gpu -q -x > $OUT/pytest_wbit_full.log 2>&1; tail -3 $OUT/pytest_wbit_full.log
