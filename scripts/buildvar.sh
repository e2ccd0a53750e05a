#!/bin/bash
# build a variant .so: buildvar.sh <name> <defines...>
name=$1; shift
out=/root/repo/build/var_$name; mkdir -p $out
cd /root/repo/paper_conf_sc_lilg14_b200/csrc
NCCL=$(python -c "import nvidia.nccl,os;print(os.path.dirname(nvidia.nccl.__file__) if hasattr(nvidia.nccl,'__file__') and nvidia.nccl.__file__ else list(nvidia.nccl.__path__)[0])")
for f in *.cu; do nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 --expt-relaxed-constexpr -Xcompiler -fPIC -I../../include -I. -I$NCCL/include "$@" -c $f -o $out/$f.o & done; wait
nvcc -gencode arch=compute_100a,code=sm_100a -shared -o $out/libsesa.so $out/*.o -lcudart -L$NCCL/lib -l:libnccl.so.2 -Xlinker -rpath=$NCCL/lib
ls -la $out/libsesa.so
