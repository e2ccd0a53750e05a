# full GPU suite + the default bench line + C2-C4 lines: bash scripts/run_full.sh <tag>
TAG=${1:-r2q}; OUT=gpurun_out; mkdir -p $OUT
timeout 1800 python -m pytest tests -m gpu -q -x > $OUT/pytest_gpu_$TAG.log 2>&1; tail -3 $OUT/pytest_gpu_$TAG.log
timeout 600 python bench.py > $OUT/bench_c5_$TAG.json 2> $OUT/bench_c5_$TAG.log; python scripts/bsum.py $OUT/bench_c5_$TAG.json
for C in c4 c3 c2; do timeout 600 python bench.py --config $C --steps 5 --warmup 3 --no-e2e --no-cpu > $OUT/bench_${C}_$TAG.json 2> $OUT/bench_${C}_$TAG.log; python scripts/bsum.py $OUT/bench_${C}_$TAG.json; done
python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_$TAG.log 2>&1; tail -1 $OUT/smoke_$TAG.log
