OUT=gpurun_out; mkdir -p $OUT
bash scripts/run_ab.sh "--steps 5 --warmup 3 --no-e2e --no-cpu" cur noxp; mv gpurun_out/ab.json gpurun_out/ab_c5x.json
timeout 600 ncu --set full --clock-control none --import-source on -k regex:extents_part -s 0 -c 1 -o $OUT/prof_xpart python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu > $OUT/ncu_xpart.log 2>&1
python scripts/ncu_summary.py $OUT/prof_xpart.ncu-rep 2>/dev/null | head -40
timeout 900 python -m pytest tests/test_gpu_xpart.py -m gpu -q -x > $OUT/pytest_xpart.log 2>&1; tail -3 $OUT/pytest_xpart.log
