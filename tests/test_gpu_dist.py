"""Distributed check: sharding by location owner + exchanges must give exactly the
single-GPU race list (sharding invariance) and the oracle's.  Virtual ranks on one GPU (loopback exchange) run
the same kernels and data flow as the NCCL path; a real NCCL communicator is exercised with world size 1."""
import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O

pytestmark = pytest.mark.gpu
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def S():
    from paper_conf_sc_lilg14_b200 import sesa
    sesa.load()
    return sesa


def shards(n, W, rng=None):
    if rng is None:
        return [n * r // W for r in range(W + 1)]
    cuts = sorted(rng.integers(0, n + 1, W - 1).tolist())
    return [0] + cuts + [n]


@pytest.mark.parametrize("W", [1, 2, 3, 4, 8])
def test_loopback_equals_single_gpu_random(S, W):
    rng = np.random.default_rng(W)
    for seed in range(6):
        r = G.random_trace(3000 + 977 * seed, seed, blocks=9, threads=200, words=40 + 300 * seed, values=3,
                           sort=True)
        d = S.to_device(r)
        exp = O.check(r)
        for offs in (shards(len(r), W), shards(len(r), W, rng)):
            got = S.check_loopback(d, offs)
            assert got.tobytes() == exp.tobytes(), (W, seed, offs, len(got), len(exp))


@pytest.mark.parametrize("W", [2, 5])
def test_loopback_configs_and_index_base(S, W):
    for (ws, ls, gran) in [(32, 1, 4), (4, 1, 1), (1, 0, 8)]:
        r = G.random_trace(4000, 77, threads=64, words=200)
        d = S.to_device(r)
        got = S.check_loopback(d, shards(len(r), W), warp_size=ws, lockstep=ls, granularity=gran, index_base=123)
        assert got.tobytes() == O.check(r, index_base=123, warp_size=ws, lockstep=ls, granularity=gran).tobytes()


@pytest.mark.parametrize("W", [2, 4])
def test_loopback_fixtures(S, W):
    for r, ls in ((G.f1_race(), 0), (G.f4_histo_prescan(), 0), (G.f5_binning(), 1), (G.c1(), 0)):
        got = S.check_loopback(S.to_device(r), shards(len(r), W), lockstep=ls)
        assert got.tobytes() == O.check(r, lockstep=ls).tobytes()


def test_loopback_c5_truth(S):
    from sesagen import configs as C
    n = 2_000_000
    d = C.c5_device(n)
    for W in (2, 8):
        got = S.check_loopback(d, shards(n, W))
        assert got.tobytes() == C.c5_truth(n).tobytes()


def test_loopback_hot_crossing(S):
    r = G.random_trace(80000, 5, blocks=6, threads=300, words=3, values=3)
    got = S.check_loopback(S.to_device(r), shards(len(r), 4))
    assert got.tobytes() == O.check(r).tobytes()


def test_loopback_unsorted_input(S):
    r = G.random_trace(5000, 9, words=100, sort=False)
    got = S.check_loopback(S.to_device(r), shards(len(r), 3))
    assert got.tobytes() == O.check(r).tobytes()


def test_loopback_invalid_record(S):
    r = G.f1_race()
    r[70]["rw"] = 7
    with pytest.raises(S.SesaError) as e:
        S.check_loopback(S.to_device(r), shards(len(r), 3))
    assert e.value.status == S.SESA_EINVAL


def test_nccl_world_one(S):
    """A real NCCL communicator through sesa_trace_create_dist at world 1 (one rank owns every location, so the
    check runs the single-GPU pipeline; the exchange data flow is covered by the loopback tests)."""
    uid = S.nccl_unique_id()
    t = S.Trace(32, 0, 4, dist=(0, 1, uid))
    r = G.random_trace(20000, 3, words=500)
    t.check(S.to_device(r), len(r))
    assert t.races().tobytes() == O.check(r).tobytes()
    t.close()


@pytest.mark.slow
@pytest.mark.parametrize("W", [1, 2])
def test_loopback_bucket_path_c5(S, W):
    """Every virtual rank receives >= 2^24 keys spread evenly: the received keys go through the bucket path
    (unstable partition passes + chunk bitmaps); the merged list equals the C5 construction truth."""
    from sesagen import configs as C
    n = 40_000_000
    d = C.c5_device(n)
    got = S.check_loopback(d, shards(n, W))
    assert got.tobytes() == C.c5_truth(n).tobytes()
