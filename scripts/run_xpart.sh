OUT=gpurun_out; mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_xpart.py -m gpu -q -x > $OUT/pytest_xpart.log 2>&1; tail -15 $OUT/pytest_xpart.log
bash scripts/run_ab.sh "--steps 5 --warmup 3 --no-e2e --no-cpu" cur noxp; mv gpurun_out/ab.json gpurun_out/ab_c5x.json
