OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_wbit.py tests/test_gpu_parity.py -m gpu -q -x -k "wbit or write_bit or fused or long_write or random" > $OUT/pytest_wbit.log 2>&1; tail -3 $OUT/pytest_wbit.log
bash scripts/run_ab.sh "--config c4 --steps 5 --warmup 3 --no-e2e --no-cpu" cur nowb; mv gpurun_out/ab.json gpurun_out/ab_c4c.json
bash scripts/run_ab.sh "--config c3 --steps 5 --warmup 3 --no-e2e --no-cpu" cur nowb; mv gpurun_out/ab.json gpurun_out/ab_c3c.json
bash scripts/run_ab.sh "--config c2 --steps 5 --warmup 3 --no-e2e --no-cpu" cur nowb; mv gpurun_out/ab.json gpurun_out/ab_c2c.json
