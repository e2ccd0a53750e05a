# round-end evidence: full GPU suite, every bench line, smoke, the reference arm; bash scripts/run_final.sh <tag>
TAG=${1:-r2z}; OUT=gpurun_out; mkdir -p $OUT
bash scripts/run_full.sh $TAG
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > $OUT/bench_ref_$TAG.json 2> $OUT/bench_ref_$TAG.log; tail -c 600 $OUT/bench_ref_$TAG.json
