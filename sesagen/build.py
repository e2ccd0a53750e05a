"""Build the generator libraries: host (gcc) and device (nvcc, sm_100a).  Test/bench infrastructure only."""
from __future__ import annotations

import os
import subprocess

HERE = os.path.dirname(os.path.abspath(__file__))
CSRC = os.path.join(HERE, "csrc")
HOST_SO = os.path.join(HERE, "_build", "libsesagen_host.so")
DEV_SO = os.path.join(HERE, "_build", "libsesagen.so")
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def _stale(out, srcs):
    return not os.path.exists(out) or os.path.getmtime(out) < max(os.path.getmtime(s) for s in srcs)


def build(force: bool = False):
    os.makedirs(os.path.dirname(HOST_SO), exist_ok=True)
    hdr = os.path.join(CSRC, "gen_common.h")
    hsrc = os.path.join(CSRC, "gen_host.c")
    dsrc = os.path.join(CSRC, "gen_dev.cu")
    if force or _stale(HOST_SO, [hdr, hsrc]):
        tmp = HOST_SO + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-fPIC", "-shared", "-Wall", "-o", tmp, hsrc])
        os.replace(tmp, HOST_SO)
    if force or _stale(DEV_SO, [hdr, dsrc]):
        tmp = DEV_SO + f".tmp{os.getpid()}"
        subprocess.check_call([NVCC, "-gencode", "arch=compute_100a,code=sm_100a", "-O3", "-lineinfo",
                               "-Xcompiler", "-fPIC", "-shared", "-o", tmp, dsrc])
        os.replace(tmp, DEV_SO)
    return HOST_SO, DEV_SO


if __name__ == "__main__":
    print(build())
