"""GPU parity of the bucket path with its first partition fused into the extents pass (k_extract.cu
"Extents fused with the bucket path's first partition", k_sort.cu UNST 3, sesa_api.cu try_extents_part).

The fused pass is speculative: a sample of 2^16 then 2^18 records predicts it, the pass's own summary decides it, and
anything the sample could not see — a shared record, a two-granule record, a (block, interval) inversion, an
invalid record between sampled positions, or a first digit so uneven that a region fills up — sends the check
back to the ordinary path.  Every case must give the oracle's race list byte for byte.
"""
import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
torch = pytest.importorskip("torch")

N = (1 << 24) + 4099  # >= BUCKET_MIN_N; the sample stride is 16, so odd indices are never sampled


@pytest.fixture(scope="module")
def S():
    from paper_conf_sc_lilg14_b200 import sesa
    sesa.load()
    return sesa


@pytest.fixture(scope="module")
def base_trace():
    from sesagen import configs as C
    return C.rnd_host(N, 77, blocks=4096, threads=512, intervals=3, words=1 << 27, shared_frac=0.0, sizes=(4,),
                      unaligned=False, values=3, atomic_frac=0.05, write_frac=0.35)


def run(S, a, ls=0, benign=False):
    t = S.Trace(32, ls, 4, benign=benign)
    t.set_profiling(True)
    t.check(S.to_device(a), len(a))
    got = t.races()
    info = t.info()
    names = {k["name"]: k["launches"] for k in t.kernel_stats()}
    t.close()
    exp = O.check(a, warp_size=32, lockstep=ls, benign=benign, method="partitioned")
    assert got.tobytes() == exp.tobytes(), (len(got), len(exp))
    return info, names


@pytest.mark.parametrize("ls,benign", [(0, False), (1, True)])
def test_fused_path_taken_and_exact(S, base_trace, ls, benign):
    info, names = run(S, base_trace, ls, benign)
    assert info["bucket_path"] == 1 and "presample" in names and "extract_pass0" not in names


def test_c5_recipe_through_the_fused_path(S):
    from sesagen import configs as C
    n = (1 << 24) + 12345
    dev = C.c5_device(n)
    t = S.Trace(32, 0, 4)
    t.set_profiling(True)
    t.check(dev, n)
    names = {k["name"] for k in t.kernel_stats()}
    got = t.races()
    t.close()
    assert "presample" in names and "extract_pass0" not in names
    assert got.tobytes() == C.c5_truth(n).tobytes()


@pytest.mark.parametrize("what", ["shared", "two_granules", "inversion", "far"])
def test_unsampled_exception_falls_back(S, base_trace, what):
    if what == "inversion":  # (an unsorted trace keys (block, interval) too: a span that fits 64 bits then)
        from sesagen import configs as C
        a = C.rnd_host(N, 78, blocks=4096, threads=512, intervals=3, words=1 << 24, shared_frac=0.0, sizes=(4,),
                       unaligned=False, values=3, atomic_frac=0.05, write_frac=0.35)
    else:
        a = base_trace.copy()
    i = 1_000_001  # odd: between sampled positions
    if what == "shared":
        a["space"][i] = G.SHARED
        a["addr"][i] = 64
    elif what == "two_granules":
        a["size"][i] = 8
    elif what == "far":  # a granule span beyond 2^30 that the sample did not see
        a["addr"][i] = a["addr"][i] + np.uint64(1 << 40)
    else:
        a["block"][i] = a["block"][i - 1] - 1 if a["block"][i - 1] > 0 else 0
        a["interval"][i] = 0
        a["block"][i - 1] = max(int(a["block"][i - 1]), 1)
    info, names = run(S, a)
    assert names["presample"] >= 1 and names["extents"] == 2  # the fused pass, then the ordinary path


def test_uneven_first_digit_overflows_and_falls_back(S, base_trace):
    # granule bit 14 always 0: chunks (2^15 granules) stay even, the first digit's odd regions stay empty and
    # the even ones overflow their capacity (1.125 x the mean) -> the ordinary path (granule-array bucket path)
    a = base_trace.copy()
    g = a["addr"] >> np.uint64(2)
    a["addr"] = (g & ~np.uint64(1 << 14)) << np.uint64(2)
    info, names = run(S, a)
    assert info["bucket_path"] == 1 and names["extents"] == 2 and "extract_pass0" in names


def test_invalid_record_between_samples(S, base_trace):
    a = base_trace.copy()
    a["rw"][3_000_003] = 7
    a["size"][5_000_001] = 0
    t = S.Trace(32, 0, 4)
    with pytest.raises(S.SesaError) as e:
        t.check(S.to_device(a), len(a))
    t.close()
    assert e.value.status == S.SESA_EINVAL and "record 3000003 " in str(e.value)  # the lowest bad index


def test_dense_chunks_overflow_sort(S):
    # 2^23 words for 2^24 records: almost every entry survives, every chunk has far more than 2,048 survivors,
    # so each is sorted by the global-memory (key_hi, position) radix sort — the fused pass writes its regions in
    # window order, so the survivors arrive in no particular position order
    from sesagen import configs as C
    a = C.rnd_host(N, 79, blocks=4096, threads=512, intervals=3, words=1 << 23, shared_frac=0.0, sizes=(4,),
                   unaligned=False, values=3, atomic_frac=0.05, write_frac=0.35)
    info, names = run(S, a, ls=1)
    assert info["bucket_path"] == 1 and names["extents"] == 1 and "presample" in names


def test_regions_registered_skip_the_fused_pass(S, base_trace):
    # the out-of-bound check (NEXT-1) runs in the ordinary extents pass: with regions the fused pass is not tried
    t = S.Trace(32, 0, 4)
    t.set_profiling(True)
    lo, hi = int(base_trace["addr"].min()), int(base_trace["addr"].max()) + 4
    reg = np.zeros(1, S.REGION_DTYPE)
    reg["base"], reg["size"], reg["space"] = lo, hi - lo, G.GLOBAL
    t.set_regions(reg)
    t.check(S.to_device(base_trace), len(base_trace))
    names = {k["name"]: k["launches"] for k in t.kernel_stats()}
    got = t.races()
    assert t.oob()["n_oob"] == 0
    t.close()
    assert "presample" not in names
    assert got.tobytes() == O.check(base_trace, method="partitioned").tobytes()


def test_precise_warp_through_the_fused_path(S, base_trace):
    # the precise warp model (NEXT-3) on a trace large enough for the fused path: random {pc, div} against the
    # oracle's precise-warp checker
    a = base_trace
    e = G.random_ext(len(a), 5, npc=3, ninst=2, div_frac=0.5)
    t = S.Trace(32, 1, 4)
    t.set_profiling(True)
    t.check_warp(S.to_device(a), torch.from_numpy(np.ascontiguousarray(e).view(np.uint8).reshape(-1)).cuda(), len(a))
    names = {k["name"] for k in t.kernel_stats()}
    got = t.races()
    t.close()
    assert "presample" in names
    assert got.tobytes() == O.check_warp(a, e, warp_size=32).tobytes()


def test_host_entry_through_the_fused_path(S, base_trace):
    # sesa_race_check_host (the e2e entry: pageable host records, chunked through pinned staging) takes the same
    # fused path and returns the oracle's list, index_base applied
    t = S.Trace(32, 0, 4)
    t.set_profiling(True)
    t.check_host(base_trace, index_base=123)
    names = {k["name"] for k in t.kernel_stats()}
    got = t.races()
    t.close()
    assert "presample" in names and "extract_pass0" not in names
    assert got.tobytes() == O.check(base_trace, index_base=123, method="partitioned").tobytes()
