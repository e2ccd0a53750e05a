"""Small-trace suite for compute-sanitizer ("our own race checker gets race-checked").

    compute-sanitizer --tool {memcheck,racecheck,synccheck,initcheck} python scripts/sanitize_suite.py [--big]

Runs every kernel family of libsesa.so on small traces (fixtures, random traces through the fused, plain and
multi-granule paths, hot locations crossing conflict tiles, benign reporting, OOB, launches, the precise warp model,
expansion, loopback with 3 virtual ranks) and checks each result against the oracle; --big adds the bucket path
(2^24 + records).  Exit code 0 = all results equal.
"""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import sesagen as G  # noqa: E402
from oracle import oracle as O  # noqa: E402
from paper_conf_sc_lilg14_b200 import sesa as S  # noqa: E402


def same(got, exp, what):
    if got.tobytes() != exp.tobytes():
        print(f"MISMATCH {what}: {len(got)} vs {len(exp)}")
        sys.exit(1)
    print(f"ok {what}: {len(got)} races")


def main():
    big = "--big" in sys.argv
    S.load()
    for r, ls in ((G.f1_race(), 0), (G.f4_histo_prescan(), 0), (G.f5_binning(), 1), (G.c1(), 0)):
        t = S.Trace(32, ls, 4)
        t.check(S.to_device(r), len(r))
        same(t.races(), O.check(r, lockstep=ls), f"fixture n={len(r)}")
        t.close()
    for seed, (n, words, sort) in enumerate(((3000, 40, True), (40000, 33000, True), (20000, 3, False),
                                             (50000, 700, True))):
        r = G.random_trace(n, 77 + seed, threads=300, blocks=6, words=words, sort=sort)
        for benign in (False, True):
            t = S.Trace(32, seed % 2, 4, benign=benign)
            t.check(S.to_device(r), n)
            same(t.races(), O.check(r, lockstep=seed % 2, benign=benign), f"random {seed} benign={benign}")
            t.close()
    # many blocks, medium locations (C4-like): groups of ~100-1000 entries inside and across tile windows with
    # short sub-runs (mode 1 per-group path, thread and warp groups; mode 2 pieces with edge sub-runs)
    for ls, words in ((0, 2000), (1, 300)):
        r = G.random_trace(200000, 21 + ls, threads=32, blocks=2000, words=words, sort=True)
        t = S.Trace(32, ls, 4)
        t.check(S.to_device(r), len(r))
        same(t.races(), O.check(r, lockstep=ls), f"medium groups ls={ls} words={words}")
        t.close()
    r = G.random_trace(5000, 5, threads=64, words=300, sizes=(1, 6, 16))
    t = S.Trace(32, 0, 1)
    t.check(S.to_device(r), len(r))
    same(t.races(), O.check(r, granularity=1), "multi-granule G=1")
    t.close()
    # launches, precise warps, expansion, loopback
    r = G.random_trace(8000, 9, threads=128, words=200)
    t = S.Trace(32, 1, 4)
    offs = [0, 3000, 3000, 8000]
    t.check_launches(S.to_device(r), len(r), offs)
    same(t.races(), O.check(r, lockstep=1, launches=offs), "launches")
    e = G.random_ext(len(r), 3)
    t.check_warp(S.to_device(r), torch.from_numpy(e.view(np.uint8)).cuda(), len(r))
    same(t.races(), O.check_warp(r, e), "precise warps")
    t.close()
    fl = G.c2_flows(gx=2, gy=2)
    t = S.Trace()
    d_fl = torch.from_numpy(np.ascontiguousarray(fl).view(np.uint8).reshape(-1)).cuda()
    n = t.expand(d_fl, len(fl))
    out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
    t.expand(d_fl, len(fl), out, n)
    assert out.cpu().numpy().tobytes() == O.expand(fl).tobytes()
    print(f"ok expand: {n} records")
    t.close()
    r = G.random_trace(9000, 11, threads=100, words=500)
    same(S.check_loopback(S.to_device(r), [0, 2000, 6000, 9000]), O.check(r), "loopback x3")
    if big:
        from sesagen import configs as C
        n = (1 << 24) + 777
        dev = C.c5_device(n)
        t = S.Trace(32, 0, 4)
        t.check(dev, n)
        assert t.info()["bucket_path"] == 1
        same(t.races(), C.c5_truth(n), "bucket path (C5 recipe, 2^24 + 777)")
        t.close()
    del out, d_fl
    if big:
        del dev
    import gc
    gc.collect()
    torch.cuda.synchronize()
    torch.cuda.empty_cache()  # return torch's cached blocks, so that memcheck's leak report shows only ours
    print("SANITIZE SUITE OK")


if __name__ == "__main__":
    main()
