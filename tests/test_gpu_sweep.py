"""GPU parity sweep: 1,000 seeded random traces with n log-uniform in [1, 10^6] (10^3 seeds, n up
to 10^6), each compared byte for byte with the oracle (T-thread partitioned checker).  Per trace the structure
(blocks, threads, intervals, words, spaces, sizes, access kinds, values, record order) and the config (warp size,
lockstep, granularity, benign reporting) are drawn from the seed, so traces span one tile up to hundreds of
conflict tiles, with hot locations crossing tile boundaries, mixed-size multi-granule records and unsorted input.
"""
import math

import numpy as np
import pytest

from oracle import oracle as O
from sesagen import configs as C

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
torch = pytest.importorskip("torch")

CFGS = [(32, 0, 4), (32, 1, 4), (4, 1, 1), (1, 1, 2), (2, 0, 8), (8, 1, 16), (32, 1, 64), (3, 1, 4)]
SIZES = [(4,), (1, 2, 4, 8), (1, 1, 2, 2), (4, 8, 16, 3), (8, 8, 1, 4)]


def trace_params(seed: int):
    rng = np.random.default_rng(0xACE0 + seed)
    n = int(math.exp(rng.uniform(0, math.log(1e6))))
    words = int(math.exp(rng.uniform(0, math.log(max(2, n * 2)))))
    kw = dict(blocks=int(rng.integers(1, 65)), threads=int(rng.integers(1, 1025)), intervals=int(rng.integers(1, 9)),
              words=max(1, words), shared_frac=float(rng.choice([0.0, 0.5, 1.0])),
              sizes=SIZES[int(rng.integers(0, len(SIZES)))], atomic_frac=float(rng.choice([0.0, 0.05, 0.3])),
              write_frac=float(rng.choice([0.1, 0.35, 0.6])), values=int(rng.integers(1, 5)),
              sort=bool(rng.random() < 0.7), unaligned=bool(rng.random() < 0.5))
    return n, kw, CFGS[seed % len(CFGS)], bool(rng.random() < 0.25)


@pytest.fixture(scope="module")
def S():
    from paper_conf_sc_lilg14_b200 import sesa
    sesa.load()
    return sesa


@pytest.mark.parametrize("chunk", range(10))
def test_random_sweep(S, chunk):
    racy = 0
    for seed in range(chunk * 100, (chunk + 1) * 100):
        n, kw, (ws, ls, g), benign = trace_params(seed)
        r = C.rnd_host(n, seed, **kw)
        t = S.Trace(ws, ls, g, benign=benign)
        t.check(S.to_device(r), n)
        got = t.races()
        t.close()
        exp = O.check(r, warp_size=ws, lockstep=ls, granularity=g, benign=benign, method="partitioned")
        assert got.tobytes() == exp.tobytes(), (seed, n, kw, ws, ls, g, benign, len(got), len(exp))
        racy += len(exp) > 0
    assert racy > 0
