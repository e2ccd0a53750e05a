"""GPU parity: the sm_100a pipeline (libsesa.so through the C ABI) against the CPU oracle, byte for byte.

The output is integer-only (record indices, addresses, kinds), so the bar is bit-exact equality of the sorted
race arrays.  Inputs come from sesagen (seeded); expected values only from oracle/.
"""
import ctypes

import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def sesa():
    from paper_conf_sc_lilg14_b200 import sesa as S
    S.load()
    return S


_traces = {}


def trace(S, ws=32, ls=0, G_=4):
    key = (ws, ls, G_)
    if key not in _traces or not _traces[key].h:  # (a test may have closed the shared handle)
        _traces[key] = S.Trace(ws, ls, G_)
    return _traces[key]


def gpu_check(S, recs, ws=32, ls=0, G_=4, base=0):
    t = trace(S, ws, ls, G_)
    d = S.to_device(recs)
    t.check(d, len(recs), index_base=base)
    torch.cuda.synchronize()
    return t.races()


def assert_same(S, recs, ws=32, ls=0, G_=4, base=0, method="grouped"):
    exp = O.check(recs, index_base=base, warp_size=ws, lockstep=ls, granularity=G_, method=method)
    got = gpu_check(S, recs, ws, ls, G_, base)
    if got.tobytes() != exp.tobytes():
        e, g = set(O.race_tuples(exp)), set(O.race_tuples(got))
        raise AssertionError(f"{len(exp)} expected, {len(got)} got; missing {sorted(e - g)[:5]} extra {sorted(g - e)[:5]}")
    return got


# ------------------------------------------------------------------------------------------------ paper fixtures
@pytest.mark.parametrize("ls", [0, 1])
@pytest.mark.parametrize("distinct", [True, False])
def test_f1_race(sesa, ls, distinct):
    assert_same(sesa, G.f1_race(distinct=distinct), ls=ls, method="brute")


def test_f1_paper_witness_on_gpu(sesa):
    got = O.race_tuples(gpu_check(sesa, G.f1_race()))
    assert (0, 0, 0, 0, 1, 1, 126) in got  # t0 writes v[0], t63 reads it (interval 0)


def test_f2_reduction(sesa):
    for ls in (0, 1):
        assert len(assert_same(sesa, G.f2_reduction(), ls=ls)) == 0


@pytest.mark.parametrize("B", [16, 32, 64, 128, 256])
def test_f3_bitonic(sesa, B):
    assert len(assert_same(sesa, G.f3_bitonic(B))) == 0


@pytest.mark.parametrize("ls,ws", [(0, 32), (1, 32), (1, 1)])
def test_f4_histo_prescan(sesa, ls, ws):
    assert_same(sesa, G.f4_histo_prescan(), ws=ws, ls=ls)


@pytest.mark.parametrize("ls", [0, 1])
def test_f5_binning(sesa, ls):
    assert len(assert_same(sesa, G.f5_binning(), ls=ls)) == 1


def test_c1(sesa):
    got = assert_same(sesa, G.c1(), method="brute")
    assert O.race_tuples(got) == [(0, 0, 5, 4, 2, 833, 836)]


# ------------------------------------------------------------------------------------------------ random traces
CONFIGS = [(32, 0, 4), (32, 1, 4), (4, 1, 1), (1, 1, 2), (2, 0, 8), (8, 1, 16)]


@pytest.mark.parametrize("cfg", CONFIGS)
def test_random_small(sesa, cfg):
    ws, ls, G_ = cfg
    for seed in range(40):
        n = 1 + (seed * 37) % 400
        r = G.random_trace(n, seed, threads=12 + seed % 60, sort=seed % 4 != 0, words=8 + seed % 40)
        assert_same(sesa, r, ws, ls, G_, base=seed * 1000)


@pytest.mark.parametrize("seed", range(6))
def test_random_medium_spans_tiles(sesa, seed):
    # 20k-150k entries: many 2048-entry conflict tiles, 4096-key sort tiles and a ragged tail
    n = [20000, 33333, 65537, 100000, 150001, 4097][seed]
    r = G.random_trace(n, seed, blocks=40, threads=256, intervals=4, words=5000 + 3000 * seed, values=5,
                       sort=seed != 3)
    assert_same(sesa, r, 32, seed % 2, 4)


@pytest.mark.parametrize("G_", [1, 64, 4096])
def test_wide_accesses_extreme_granularity(sesa, G_):
    # accesses of up to 300 bytes at G = 1 span up to 300 granules each (multi-granule extraction, entries >>
    # records, runs crossing conflict tiles); at G = 4096 the whole shared window is one granule per block
    for seed in range(3):
        r = G.random_trace(3000 + 4111 * seed, 500 + seed, blocks=5, threads=200, intervals=3, words=900,
                           sizes=(1, 3, 8, 64, 300), values=4, sort=seed != 1)
        for ws, ls in ((32, 0), (32, 1), (4, 1)):
            assert_same(sesa, r, ws, ls, G_, base=7 * seed)


def test_large_index_base(sesa):
    # witnesses are u64 record indices offset by index_base (include/sesa.h): a base past 2^32 and 2^40
    r = G.random_trace(5000, 77, blocks=4, threads=128, intervals=2, words=300)
    for base in ((1 << 32) - 17, (1 << 40) + 3):
        assert_same(sesa, r, 32, 0, 4, base=base)


@pytest.mark.parametrize("words", [1, 3, 40, 700])
def test_hot_locations_cross_tiles(sesa, words):
    # few words -> location runs of thousands of entries: runs and sub-runs cross conflict-tile boundaries
    r = G.random_trace(60000, 99 + words, blocks=6, threads=300, intervals=3, words=words, values=3)
    for ls in (0, 1):
        assert_same(sesa, r, 32, ls, 4)


def test_hot_benign_and_atomics(sesa):
    # a C4-like `changed` run: 50k same-valued writes from many blocks plus a few reads -> RW only, no WW
    n = 50000
    r = np.zeros(n, G.REC_DTYPE)
    r["block"] = np.arange(n) // 512
    r["thread"] = np.arange(n) % 512
    r["space"] = 1
    r["size"] = 4
    r["addr"] = 0x5000
    r["rw"] = 1
    r["value_hash"] = 77
    r["rw"][::9973] = 0
    got = assert_same(sesa, r, 32, 1, 4)
    assert set(got["kind"]) <= {1}


# ------------------------------------------------------------------------------------------------ expansion
@pytest.mark.parametrize("name", ["f1", "f2", "f5", "c1", "c2s", "c2m"])
def test_expand_parity(sesa, name):
    fl = {"f1": G.f1_flows(), "f2": G.f2_flows(), "f5": G.f5_flows(), "c1": G.c1_flows(),
          "c2s": G.c2_flows(gx=2, gy=3, K=80), "c2m": G.c2_mutant_flows(drop_barrier=3, gx=2, gy=2, K=64)}[name]
    exp = O.expand(fl)
    t = trace(sesa)
    d_fl = torch.from_numpy(np.ascontiguousarray(fl).view(np.uint8).reshape(-1)).cuda()
    n = t.expand(d_fl, len(fl))
    assert n == len(exp)
    out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
    assert t.expand(d_fl, len(fl), out, n) == n
    got = out.cpu().numpy().view(G.REC_DTYPE)
    assert got.tobytes() == exp.tobytes()
    if name.startswith("c2"):
        assert_same(sesa, exp)


def test_c2_full_expand_and_race_free(sesa):
    fl = G.c2_flows()
    t = trace(sesa)
    d_fl = torch.from_numpy(np.ascontiguousarray(fl).view(np.uint8).reshape(-1)).cuda()
    n = t.expand(d_fl, len(fl))
    assert n == 18300928
    out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
    t.expand(d_fl, len(fl), out, n)
    # the whole expansion at full size, byte for byte (the oracle expands the same descriptors)
    exp = O.expand(fl)
    assert out.cpu().numpy().tobytes() == exp.tobytes()
    assert t.check(out, n) == 0  # race-free by construction (double buffering, one barrier per k-tile)


# ------------------------------------------------------------------------------------------------ API behaviour
def test_empty_and_single(sesa):
    t = trace(sesa)
    assert t.check(0, 0) == 0
    assert len(t.races()) == 0
    assert_same(sesa, G.f1_race()[:1])


def test_invalid_record_lowest_index(sesa):
    r = G.f1_race()
    r[40]["rw"] = 3
    r[17]["size"] = 0
    t = trace(sesa)
    with pytest.raises(sesa.SesaError) as e:
        t.check(sesa.to_device(r), len(r))
    assert e.value.status == sesa.SESA_EINVAL and "record 17 " in str(e.value)
    n = ctypes.c_uint64()
    assert t.lib.sesa_races_get(t.h, None, 0, ctypes.byref(n)) == sesa.SESA_ESTATE  # all-or-nothing


def test_host_pointer_rejected(sesa):
    r = G.f1_race()
    t = trace(sesa)
    with pytest.raises(sesa.SesaError) as e:
        t.check(r.ctypes.data, len(r))
    assert e.value.status == sesa.SESA_EINVAL


def test_erange_wide_key(sesa):
    r = G.random_trace(1000, 5)
    r["addr"][::2] = np.uint64(1 << 63)  # 2^61-granule global span + shared + 10 position bits > 64
    t = trace(sesa)
    with pytest.raises(sesa.SesaError) as e:
        t.check(sesa.to_device(r), len(r))
    assert e.value.status == sesa.SESA_ERANGE


def test_races_get_truncation(sesa):
    r = G.f1_race()
    t = trace(sesa)
    d = sesa.to_device(r)
    assert t.check(d, len(r)) == 88
    out = np.zeros(10, sesa.RACE_DTYPE)
    n = ctypes.c_uint64()
    st = t.lib.sesa_races_get(t.h, ctypes.c_void_p(out.ctypes.data), 10, ctypes.byref(n))
    assert st == sesa.SESA_ETRUNC and n.value == 88
    assert out.tobytes() == O.check(r)[:10].tobytes()


def test_host_entry_point_matches(sesa):
    r = G.random_trace(5000, 11, words=300)
    t = trace(sesa)
    t.check_host(r, index_base=7)
    assert t.races().tobytes() == O.check(r, index_base=7).tobytes()


def test_profiling_stats(sesa):
    t = sesa.Trace()
    t.set_profiling(True)
    r = G.random_trace(30000, 3, words=2000)
    t.check(sesa.to_device(r), len(r))
    names = {s["name"] for s in t.kernel_stats()}
    assert {"extents", "extract_multi", "onesweep_pass", "conflict"} <= names  # sizes up to 8 B: multi-granule
    r1 = G.random_trace(30000, 4, words=2000, sizes=(4,), unaligned=False)
    t.check(sesa.to_device(r1), len(r1))
    assert "extract" in {s["name"] for s in t.kernel_stats()}
    info = t.info()
    assert info["n_records"] == 30000 and info["launches"] >= 4
    t.close()


@pytest.mark.parametrize("tail", ["none", "atomic", "other_value", "read"])
def test_long_write_run_skip(sesa, tail):
    # a C4-`changed`-like run of 60k same-valued writes crossing ~30 conflict tiles: its middle tiles skip the
    # crossing modes when the whole run cannot race; one atomic, other value or read at its end must still be found
    n = 60000
    r = np.zeros(n, G.REC_DTYPE)
    r["block"] = np.arange(n) // 256
    r["thread"] = np.arange(n) % 256
    r["space"] = 1
    r["size"] = 4
    r["addr"] = 0x9000
    r["rw"] = 1
    r["value_hash"] = 5
    if tail == "atomic":
        r["rw"][-1] = 2
    elif tail == "other_value":
        r["value_hash"][-1] = 6
    elif tail == "read":
        r["rw"][-1] = 0
    extra = G.random_trace(5000, 17, blocks=300, threads=256, intervals=1, words=50, shared_frac=0.0, sizes=(4,),
                           unaligned=False)
    extra["block"] = np.sort(extra["block"]) + 300
    recs = np.concatenate([r, extra])
    got = assert_same(sesa, recs, 32, 0, 4)
    assert (len([x for x in O.race_tuples(got) if x[3] == 0x9000]) == 0) == (tail == "none")


# ------------------------------------------------------------------------------------------------ fused first pass
@pytest.mark.parametrize("n,words,shift,fused", [(32768, 100, 77, 1), (40000, 30000, 1, 1), (65537, 3_000_000, 200, 1),
                                                 (200003, 50_000, 255, 1), (500000, 400_000_000, 13, 1),
                                                 (70000, 65_500, 255, 1), (70000, 65_000, 255, 1),
                                                 (40000, 2**34, 3, 0), (32767, 1000, 5, 0)])
def test_fused_first_pass_parity(sesa, n, words, shift, fused):
    # global-only, (block, interval)-ordered, one granule per record: the fused extract + first sort pass
    # (k_fused.cu) places tiles from the extents' raw-byte histograms rotated by gmin & 255 — shift moves gmin.
    # The later digits' histograms come from the extents' raw granule bytes once gmin is aligned down to
    # 2^(8 (npass - 1)) unless the aligned span needs an extra pass (65,500 words at gmin byte 255: fallback).
    r = G.random_trace(n, 7 + n % 97, blocks=64, threads=256, intervals=3, words=words, shared_frac=0.0,
                       sizes=(4,), unaligned=False, values=4)
    r["addr"] += np.uint64(4 * shift)
    assert_same(sesa, r, 32, 0, 4)
    assert trace(sesa).info()["fused_first_pass"] == fused  # > 32 sort bits or < 32768 records: separate extract


# ------------------------------------------------------------------------------------------------ benign W/W (NEXT-4)
_btraces = {}


def assert_same_benign(S, recs, ws=32, ls=0, G_=4, base=0, method="grouped"):
    key = (ws, ls, G_)
    if key not in _btraces:
        _btraces[key] = S.Trace(ws, ls, G_, benign=True)
    t = _btraces[key]
    t.check(S.to_device(recs), len(recs), index_base=base)
    torch.cuda.synchronize()
    got = t.races()
    exp = O.check(recs, index_base=base, warp_size=ws, lockstep=ls, granularity=G_, method=method, benign=True)
    if got.tobytes() != exp.tobytes():
        e, g = set(O.race_tuples(exp)), set(O.race_tuples(got))
        raise AssertionError(f"{len(exp)} expected, {len(got)} got; missing {sorted(e - g)[:5]} extra {sorted(g - e)[:5]}")
    return got


def test_benign_f1_equal_values(sesa):
    got = assert_same_benign(sesa, G.f1_race(distinct=False), method="brute")
    assert (got["kind"] == 3).sum() == 16


@pytest.mark.parametrize("cfg", CONFIGS)
def test_benign_random_small(sesa, cfg):
    ws, ls, G_ = cfg
    for seed in range(25):
        n = 2 + (seed * 41) % 500
        r = G.random_trace(n, 300 + seed, threads=8 + seed % 40, values=2, write_frac=0.6, atomic_frac=0.1,
                           sort=seed % 4 != 0, words=6 + seed % 30)
        assert_same_benign(sesa, r, ws, ls, G_, base=seed * 77)


@pytest.mark.parametrize("seed", range(4))
def test_benign_medium_and_hot(sesa, seed):
    # many tiles, hot locations crossing conflict tiles, few values: benign pairs everywhere
    n = [30000, 70001, 120000, 9000][seed]
    r = G.random_trace(n, 900 + seed, blocks=30, threads=256, intervals=3, words=[2000, 40, 7, 300][seed],
                       values=[3, 2, 4, 1][seed], write_frac=0.5, sort=seed != 2)
    assert_same_benign(sesa, r, 32, seed % 2, 4)


@pytest.mark.parametrize("sort", [True, False])
def test_benign_global_only(sesa, sort):
    # one space: with unordered input the global keys carry (block, interval) and runs are not position-ordered
    r = G.random_trace(40000, 77 + sort, blocks=50, threads=128, intervals=4, words=900, values=2, write_frac=0.5,
                       shared_frac=0.0, sort=sort)
    assert_same_benign(sesa, r, 32, 0, 4)


def test_benign_bfs_shape(sesa):
    # Table IV: the BFS kernel's W/W conflicts are benign — C4 recipe at 2^12 nodes, lockstep
    from sesagen import configs as GC
    r = GC.C4(log2n=12).host()
    got = assert_same_benign(sesa, r, 32, 1, 4)
    assert 2 not in set(got["kind"].tolist()) and 3 in set(got["kind"].tolist())


def test_benign_flag_on_distributed_handles(sesa):
    """Benign W/W reporting on the distributed path (records of multi-entry locations fetched from their owner
    ranks): loopback with 1-5 virtual ranks == the single-GPU list == the oracle's."""
    for W, seed in ((1, 0), (2, 1), (3, 2), (5, 3)):
        r = G.random_trace(6000, 600 + seed, threads=80, words=150, values=2, write_frac=0.6, atomic_frac=0.1,
                           sort=seed != 2)
        exp = O.check(r, benign=True, lockstep=seed % 2)
        assert (exp["kind"] == 3).any()
        offs = [len(r) * k // W for k in range(W + 1)]
        got = sesa.check_loopback(sesa.to_device(r), offs, lockstep=seed % 2, benign=True)
        assert got.tobytes() == exp.tobytes()


# ------------------------------------------------------------------------------------------------ OOB (NEXT-1)
def _oob_check(S, recs, regions, base=0):
    t = S.Trace(32, 0, 4)
    t.set_regions(regions)
    t.check(S.to_device(recs), len(recs), index_base=base)
    got = t.oob()
    t.close()
    cnt, first = O.oob(recs, regions, index_base=base)
    assert got["n_oob"] == cnt
    assert got["first_index"] == (first if first is not None else 2**64 - 1)
    if first is not None:
        assert got["first"].tobytes() == recs[first - base].tobytes()
    return got


def test_f6_histo_final_oob(sesa):
    got = _oob_check(sesa, G.f6_histo_final(), G.f6_regions())
    assert got["n_oob"] == 12288 and (int(got["first"]["block"]), int(got["first"]["thread"])) == (18, 0)


@pytest.mark.parametrize("seed", range(4))
def test_oob_random_regions(sesa, seed):
    rng = np.random.default_rng(seed)
    r = G.random_trace([5000, 70000, 200003, 33][seed], 40 + seed, words=3000, blocks=9, threads=200)
    # non-overlapping random regions over both spaces' word ranges (shared from 0, global from 2^40)
    regs = []
    for sp, base in ((0, 0), (1, 0x10000000000)):
        cuts = np.sort(rng.choice(np.arange(1, 12000), size=2 * (5 + seed), replace=False))
        for a, b in cuts.reshape(-1, 2):
            regs.append((base + int(a), int(b - a), sp))
    reg = np.zeros(len(regs), G.f6_regions().dtype)
    for i, (b, z, sp) in enumerate(regs):
        reg[i]["base"], reg[i]["size"], reg[i]["space"] = b, z, sp
    _oob_check(sesa, r, reg, base=seed * 7)
    _oob_check(sesa, r, reg[reg["space"] == 1])  # only global checked


def test_oob_region_validation(sesa):
    t = sesa.Trace(32, 0, 4)
    reg = np.zeros(2, sesa.REGION_DTYPE)
    reg["base"], reg["size"], reg["space"] = [0, 10], [16, 4], 1  # [0,16) and [10,14) overlap
    with pytest.raises(sesa.SesaError):
        t.set_regions(reg)
    reg["size"] = [10, 0]
    with pytest.raises(sesa.SesaError):
        t.set_regions(reg)
    reg["size"], reg["space"] = [10, 4], [1, 2]
    with pytest.raises(sesa.SesaError):
        t.set_regions(reg)
    reg["space"] = 1
    t.set_regions(reg)  # adjacent, fine
    t.set_regions(reg[:0])  # clears
    t.close()


# ------------------------------------------------------------------------------------------------ bucket path
# Large single-space traces with evenly spread granules take the bucket path (k_bucket.cu: two high-digit sort
# passes, per-chunk shared-memory bitmaps, survivors sorted per chunk); it must give the oracle's list exactly,
# through the bitonic (few survivors per chunk) and the overflow (> 4096 survivors per chunk) sorts.
@pytest.mark.slow
@pytest.mark.parametrize("words_log2,ls,benign", [(28, 0, False), (26, 1, False), (25, 0, True), (27, 1, True)])
def test_bucket_path_random(sesa, words_log2, ls, benign):
    from sesagen import configs as C
    n = 20_000_000
    r = C.rnd_host(n, 40 + words_log2, blocks=4096, threads=512, intervals=3, words=1 << words_log2,
                   shared_frac=0.0, sizes=(4,), unaligned=False, values=3, atomic_frac=0.05, write_frac=0.35)
    t = sesa.Trace(32, ls, 4, benign=benign)
    t.check(sesa.to_device(r), n)
    assert t.info()["bucket_path"] == 1
    got = t.races()
    t.close()
    exp = O.check(r, warp_size=32, lockstep=ls, benign=benign, method="partitioned")
    assert len(got) == len(exp) and got.tobytes() == exp.tobytes()


@pytest.mark.slow
def test_bucket_path_c5_reduced(sesa):
    """C5's recipe at 2^24 + 12345 records: the bucket path's race list equals the construction truth and the
    oracle's."""
    from sesagen import configs as C
    n = (1 << 24) + 12345
    dev = C.c5_device(n)
    t = sesa.Trace(32, 0, 4)
    t.check(dev, n)
    assert t.info()["bucket_path"] == 1
    got = t.races()
    t.close()
    assert got.tobytes() == C.c5_truth(n).tobytes()
    host = dev.cpu().numpy().view(G.REC_DTYPE)
    assert got.tobytes() == O.check(host, method="partitioned").tobytes()


@pytest.mark.slow
def test_hot_traces_keep_the_full_sort(sesa):
    """The sample test sends traces with a hot granule region to the full sort (C3-shaped: Zipf bins)."""
    from sesagen import configs as C
    cfg = C.C3(blocks=384)
    dev, n = cfg.device()
    assert n >= 1 << 24
    t = sesa.Trace(32, 0, 4)
    t.check(dev, n)
    assert t.info()["bucket_path"] == 0
    t.close()


# ------------------------------------------------------------------------------------------------ launches (NEXT-4)
@pytest.mark.parametrize("seed", range(8))
def test_launches_random(sesa, seed):
    """sesa_race_check_launches == the oracle's multi-launch check (launch = part of the location, R23): random
    traces cut into launches (empty ones included), benign reporting on some, one launch large enough to take the
    fused first pass."""
    rng = np.random.default_rng(500 + seed)
    n = [3000, 50000, 120000, 700][seed % 4]
    r = G.random_trace(n, 9000 + seed, threads=200, blocks=8, words=300 + 40 * seed, sort=seed % 3 != 0)
    k = int(rng.integers(1, 6))
    cuts = np.sort(rng.integers(0, n + 1, k - 1)) if k > 1 else np.array([], np.int64)
    offs = [0, *cuts.tolist(), n]
    if seed == 5:
        offs = [0, 0, n // 2, n // 2, n]  # empty launches
    ls, benign = seed % 2, seed % 3 == 1
    t = sesa.Trace(32, ls, 4, benign=benign)
    t.check_launches(sesa.to_device(r), n, offs, index_base=7 * seed)
    got = t.races()
    t.close()
    exp = O.check(r, launches=offs, lockstep=ls, benign=benign, index_base=7 * seed)
    assert got.tobytes() == exp.tobytes()


def test_launches_f1_twice_and_validation(sesa):
    f = G.f1_race()
    two = np.concatenate([f, f])
    t = sesa.Trace(32, 0, 4)
    t.check_launches(sesa.to_device(two), len(two), [0, len(f), len(two)])
    got = t.races()
    assert len(got) == 176 and (got["epoch"] == 0).sum() == 88
    assert got.tobytes() == O.check(two, launches=[0, len(f), len(two)]).tobytes()
    for bad in ([0, 10], [1, len(two)], [0, 500, 400, len(two)]):
        with pytest.raises(sesa.SesaError):
            t.check_launches(sesa.to_device(two), len(two), bad)
    t.close()


# ------------------------------------------------------------------------------------------------ precise warps (NEXT-3)
def _ext_dev(e):
    return torch.from_numpy(np.ascontiguousarray(e).view(np.uint8).reshape(-1)).cuda()


def test_precise_warp_f1_f4(sesa):
    for r, e, ws in ((G.f1_race(), G.f1_race_ext(), 32), (G.f4_histo_prescan(), G.f4_histo_prescan_ext(), 32),
                     (G.f4_histo_prescan(), G.f4_histo_prescan_ext(), 1)):
        t = sesa.Trace(ws, 1, 4)
        t.check_warp(sesa.to_device(r), _ext_dev(e), len(r))
        assert t.races().tobytes() == O.check_warp(r, e, warp_size=ws).tobytes()
        t.close()


@pytest.mark.parametrize("seed", range(10))
def test_precise_warp_random(sesa, seed):
    """Random traces with random {pc, div}: sizes from one tile to many (hot locations cross tiles), shared and
    global, warp sizes 32/4/3; equal to the oracle's precise-warp checker."""
    n = [500, 4000, 30000, 120000, 2000][seed % 5]
    ws = [32, 4, 3, 32, 8][seed % 5]
    r = G.random_trace(n, 8800 + seed, threads=[64, 256, 700][seed % 3], blocks=1 + seed % 4,
                       words=[5, 60, 2000][seed % 3], sort=seed % 4 != 3, values=3)
    e = G.random_ext(n, seed, npc=1 + seed % 5, ninst=1 + seed % 3, div_frac=[0.0, 0.5, 1.0][seed % 3])
    t = sesa.Trace(ws, 1, 4)
    t.check_warp(sesa.to_device(r), _ext_dev(e), n, index_base=seed)
    got = t.races()
    t.close()
    assert got.tobytes() == O.check_warp(r, e, warp_size=ws, index_base=seed).tobytes()


def test_precise_warp_lockstep_off_and_validation(sesa):
    r, e = G.f1_race(), G.f1_race_ext()
    t = sesa.Trace(32, 0, 4)
    t.check_warp(sesa.to_device(r), _ext_dev(e), len(r))
    assert t.races().tobytes() == O.check(r).tobytes()  # extension ignored without lockstep
    t.close()
    t = sesa.Trace(32, 1, 4, benign=True)
    with pytest.raises(sesa.SesaError):
        t.check_warp(sesa.to_device(r), _ext_dev(e), len(r))
    t.close()


@pytest.mark.slow
def test_precise_warp_large(sesa):
    """2 M records, ~100 entries per location (runs cross many conflict tiles), global + shared, the fused path
    not taken (mixed spaces): equal to the oracle."""
    from sesagen import configs as C
    n = 2_000_000
    r = C.rnd_host(n, 4242, blocks=64, threads=512, intervals=4, words=20000, shared_frac=0.3, sizes=(4, 8),
                   values=4, unaligned=False)
    e = G.random_ext(n, 99, npc=6, ninst=4, div_frac=0.6)
    t = sesa.Trace(32, 1, 4)
    t.check_warp(sesa.to_device(r), _ext_dev(e), n)
    got = t.races()
    t.close()
    exp = O.check_warp(r, e, warp_size=32)
    assert len(exp) > 1000 and got.tobytes() == exp.tobytes()


# ------------------------------------------------------------------------------------------------ descriptors (NEXT-2)
def _flows_dev(fl):
    return torch.from_numpy(np.ascontiguousarray(fl).view(np.uint8).reshape(-1)).cuda()


@pytest.mark.parametrize("name", ["f1", "f2", "f4", "f5", "c1", "c2", "c2m", "c2m7"])
def test_flow_check_equals_expand_then_check(sesa, name):
    """sesa_race_check_flows == expand-then-check (the oracle: oracle_expand + the checker) on the paper
    fixtures, C1, the full C2 and its mutants; race-free descriptor pairs are decided without instantiation."""
    fl = {"f1": G.f1_flows(), "f2": G.f2_flows(), "f4": G.f4_flows(), "f5": G.f5_flows(), "c1": G.c1_flows(),
          "c2": G.c2_flows(), "c2m": G.c2_mutant_flows(drop_barrier=3, gx=2, gy=2, K=64),
          "c2m7": G.c2_mutant_flows(drop_barrier=7)}[name]
    t = sesa.Trace(32, 0, 4)
    t.check_flows(_flows_dev(fl), len(fl))
    got = t.races()
    info = t.flow_info()
    t.close()
    exp = O.check(O.expand(fl), method="partitioned")
    assert got.tobytes() == exp.tobytes()
    assert info["n_records"] == len(O.expand(fl)) if name != "c2" else info["n_records"] == 18300928
    if name == "c2":  # race-free by construction: decided arithmetically, nothing instantiated
        assert info["n_records_checked"] == 0 and len(got) == 0
    if name == "c2m7":  # only the descriptors of the merged intervals are instantiated
        assert 0 < info["n_records_checked"] < info["n_records"] // 4


@pytest.mark.parametrize("seed", range(40))
def test_flow_check_random_descriptors(sesa, seed):
    fl = G.random_flows(seed, nd=4 + seed % 12)
    for ls, gran in ((0, 4), (1, 1), (1, 8)):
        t = sesa.Trace(4 if seed % 2 else 32, ls, gran)
        t.check_flows(_flows_dev(fl), len(fl))
        got = t.races()
        t.close()
        exp = O.check(O.expand(fl), warp_size=4 if seed % 2 else 32, lockstep=ls, granularity=gran)
        assert got.tobytes() == exp.tobytes(), (seed, ls, gran, len(got), len(exp))


def test_host_entry_pageable_chunks_and_pinned(sesa):
    """sesa_race_check_host: a pageable 96 MB array goes through the chunked pinned staging (two 64 MiB
    buffers), a page-locked one by one DMA; both give the oracle's list."""
    from sesagen import configs as C
    n = 3_000_000
    r = C.rnd_host(n, 31337, blocks=256, threads=512, intervals=2, words=1 << 22, shared_frac=0.0, sizes=(4,),
                   unaligned=False, values=3)
    exp = O.check(r, method="partitioned")
    t = trace(sesa)
    t.check_host(r)
    assert t.races().tobytes() == exp.tobytes()
    pinned = torch.from_numpy(r.view(np.uint8)).pin_memory()
    t.check_host_ptr(pinned.data_ptr(), n)
    assert t.races().tobytes() == exp.tobytes()
    t.close()


@pytest.mark.slow
def test_bucket_path_on_key_arrays(sesa):
    """The bucket path from a key array (no fused first pass): multi-granule records (8-byte accesses at G = 4)
    over an evenly spread region, 17 M records; equal to the oracle."""
    from sesagen import configs as C
    n = (1 << 24) + 4321
    r = C.rnd_host(n, 777, blocks=4096, threads=512, intervals=2, words=1 << 26, shared_frac=0.0, sizes=(4, 8),
                   unaligned=False, values=3)
    t = sesa.Trace(32, 0, 4)
    t.check(sesa.to_device(r), n)
    info = t.info()
    got = t.races()
    t.close()
    assert info["bucket_path"] == 1 and info["fused_first_pass"] == 0
    assert got.tobytes() == O.check(r, method="partitioned").tobytes()


# ------------------------------------------------------------------------------------- conflict fast paths (round 2)
# Mode 1 decides groups wholly inside a tile window group by group (one thread per group of <= 16 entries, one warp
# per longer group; partners in other blocks from the group summary, inside the (block, interval) sub-run pair by
# pair); a window with an inner sub-run > 64 entries keeps the segmented scans; mode 2 decides crossing pieces from
# carried summaries (edge sub-runs) or pair by pair.  These traces aim at each branch and at their boundaries.
@pytest.mark.parametrize("threads,words,sort", [(32, 4000, True), (32, 400, True), (2, 3000, True), (512, 60, True),
                                                (32, 4000, False), (512, 60, False)])
def test_conflict_group_paths(sesa, threads, words, sort):
    # many blocks x few threads: short sub-runs, groups of ~10-1000 entries inside and across windows;
    # 512 threads over 60 words: sub-runs longer than 64 (scan path); unsorted input: runs ordered by
    # (block, interval) first (lowG > 0: the x / y searches cannot stop early)
    r = G.random_trace(120000, 4242 + threads + words, blocks=3000 if threads < 512 else 4, threads=threads,
                       intervals=2, words=words, shared_frac=0.0, sort=sort, values=2)
    for ls in (0, 1):
        assert_same(sesa, r, 32, ls, 4)


@pytest.mark.parametrize("glen", [2, 15, 16, 17, 31, 32, 33, 64, 65, 1535, 1536, 1537, 4000])
def test_conflict_group_length_boundaries(sesa, glen):
    # one location per group of exactly glen entries (thread / warp group boundary at 16, warp chunks of 32,
    # tile window 1536): reads by many threads, one write in the middle by another block, another location after
    rng = np.random.default_rng(glen)
    n = glen * 7
    r = np.zeros(n, G.REC_DTYPE)
    r["space"] = G.GLOBAL
    r["size"] = 4
    r["block"] = np.arange(n) // 7
    r["thread"] = rng.integers(0, 64, n)
    r["interval"] = 0
    r["addr"] = 0x10000000000 + 4 * (np.arange(n) % 7)
    r["rw"] = np.where(rng.random(n) < 0.1, G.WRITE, G.READ)
    r["value_hash"] = rng.integers(0, 2, n)
    for ls in (0, 1):
        assert_same(sesa, r, 32, ls, 4)
