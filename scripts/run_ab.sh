# usage: bash scripts/run_ab.sh "<bench args>" variants...  (abvar/<v>/libsesa.so) -> gpurun_out/ab.json
rm -f gpurun_out/ab.json; mkdir -p gpurun_out
args=$1; shift
timeout 1500 bash scripts/ab.sh "$args" "$@"
python scripts/ab_show.py gpurun_out/ab.json
