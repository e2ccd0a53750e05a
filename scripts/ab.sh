#!/bin/bash
# A/B timing on one box: ab.sh "<bench args>" <variant dirs...> — each abvar/<v>/libsesa.so is copied into the
# package and bench.py is run twice per variant (interleaved), one JSON line each into gpurun_out/ab.json
args=$1; shift
cp paper_conf_sc_lilg14_b200/libsesa.so /tmp/libsesa.orig.so
for rep in 1 2; do
  for v in "$@"; do
    cp abvar/$v/libsesa.so paper_conf_sc_lilg14_b200/libsesa.so
    python bench.py $args 2>/dev/null | tail -1 | python -c "import json,sys; d=json.loads(sys.stdin.readline()); d['variant']='$v'; print(json.dumps(d))" >> gpurun_out/ab.json
  done
done
cp /tmp/libsesa.orig.so paper_conf_sc_lilg14_b200/libsesa.so
