"""The seeded generators: host (C, feeds the oracle) and device (CUDA, feeds the bench) produce identical bytes,
and the configs have the documented shapes.  C5's injected races are the ground truth of the 1e9 trace."""
import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O
from sesagen import configs as C


def test_c5_shape_and_truth_small():
    n = 200000
    r = C.c5_host(n)
    assert len(r) == n
    assert np.array_equal(r["block"], np.arange(n) // 2048)
    assert np.array_equal(r["interval"], (np.arange(n) // 512) % 4)
    assert np.array_equal(r["thread"], np.arange(n) % 512)
    # unique words except the injected pairs
    _, counts = np.unique(r["addr"], return_counts=True)
    assert counts.max() == 2 and (counts == 2).sum() == n // 10000
    frac = np.bincount(r["rw"], minlength=3) / n
    assert abs(frac[0] - 0.70) < 0.01 and abs(frac[1] - 0.25) < 0.01 and abs(frac[2] - 0.05) < 0.01
    assert O.check(r).tobytes() == C.c5_truth(n).tobytes()


def test_c5_range_generation_consistent():
    n = 50000
    full = C.c5_host(n)
    part = C.c5_host(n, 12345, 23456)
    assert part.tobytes() == full[12345:23456].tobytes()


def test_c3_small_shape():
    s = C.C3(blocks=8, threads=64, ppt=12, nbins=64)
    r = s.host()
    T = 8 * 64
    assert (r["rw"] == 2).sum() == T * 12 and (r["rw"] == 0).sum() >= T * 12
    bins = r["addr"][r["rw"] == 2]
    counts = np.bincount(((bins - bins.min()) // 4).astype(np.int64))
    assert counts[0] == counts.max()  # Zipf: bin 0 is the hottest
    races = O.check(r)
    assert set(races["kind"].tolist()) <= {1}  # atomics exempt from each other: RW only (guard reads)


def test_c4_small_shape():
    s = C.C4(log2n=12)
    r = s.host()
    assert set(np.unique(r["rw"]).tolist()) <= {0, 1}
    races = O.check(r, lockstep=1)
    assert len(races) > 0 and set(races["kind"].tolist()) == {1}  # writes are benign (same level value)
    assert keyset_subset(O.check(r, lockstep=1), O.check(r, lockstep=0))


def keyset_subset(a, b):
    ka = {(int(x["addr"]), int(x["kind"])) for x in a}
    kb = {(int(x["addr"]), int(x["kind"])) for x in b}
    return ka <= kb


@pytest.mark.gpu
def test_device_generators_match_host():
    import torch
    n = 300000
    d = C.c5_device(n)
    assert d.cpu().numpy().view(G.REC_DTYPE).tobytes() == C.c5_host(n).tobytes()
    for s in (C.C3(blocks=16, threads=128, ppt=24, nbins=512), C.C4(log2n=14)):
        dev, n2 = s.device()
        torch.cuda.synchronize()
        assert dev.cpu().numpy().view(G.REC_DTYPE).tobytes() == s.host().tobytes()
