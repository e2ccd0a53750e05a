#!/bin/bash
# compute-sanitizer over the small-trace suite (SURVEY §4.2 kernel hygiene); run under gpurun.
# usage: bash scripts/sanitize.sh <tag>      -> gpurun_out/sanitize_<tool>_<tag>.log
TAG=${1:-r2}
OUT=gpurun_out; mkdir -p $OUT
CS=/usr/local/cuda/bin/compute-sanitizer
$CS --tool memcheck --leak-check full --error-exitcode 9 python scripts/sanitize_suite.py --big > $OUT/sanitize_memcheck_$TAG.log 2>&1; echo "memcheck rc=$?"
for T in racecheck synccheck initcheck; do
  timeout 1500 $CS --tool $T --error-exitcode 9 python scripts/sanitize_suite.py --big > $OUT/sanitize_${T}_$TAG.log 2>&1; echo "$T rc=$?"
done
for T in memcheck racecheck synccheck initcheck; do echo "== $T"; tail -4 $OUT/sanitize_${T}_$TAG.log; done
