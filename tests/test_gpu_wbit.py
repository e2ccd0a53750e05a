"""GPU parity of the write-bit compaction (KeyLayout::wbit, k_compact.cu compact_seg_w_kernel).

On the fused sort path the key carries one bit per entry — its record writes (WRITE or ATOMIC) — and compaction
drops location runs whose entries all read: P:43 needs a write for a race, so such a run can never report one.
Runs the compaction warp cannot see whole (crossing warp ranges or register batches) are kept.  These traces aim
at that logic: run lengths from 2 to 20,000 entries (spanning rows of 32, batches of 8 rows, warp ranges), the
only write of a run at its first / last / a middle entry, read-only and atomic-only runs, at sizes where warp
ranges hold several batches (m > 148 * 32 * 256).  The race list must equal the oracle's byte for byte; the
compacted count must lie between the exact count of entries at multi-entry locations with a write and the count
without the filter.
"""
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


def run_mix_trace(n_loc: int, seed: int, long_frac: float = 1e-4) -> np.ndarray:
    """Global-only, (block, interval)-ordered, one granule per record (the fused path).  Per location a run
    length (mostly 1-4, some up to 64, long_frac up to 20,000) and a write pattern: all reads, all atomics, one
    write at the first / last / a random entry, or a random mix."""
    rng = np.random.default_rng(0x3B17 + seed)
    u = rng.random(n_loc)
    lens = np.where(u < 0.5, 1, np.where(u < 0.8, rng.integers(2, 5, n_loc),
                    np.where(u < 1.0 - long_frac, rng.integers(5, 65, n_loc), rng.integers(65, 20001, n_loc))))
    n = int(lens.sum())
    loc = np.repeat(np.arange(n_loc), lens)
    idx_in = np.arange(n) - np.repeat(np.cumsum(lens) - lens, lens)
    pat = np.repeat(rng.integers(0, 6, n_loc), lens)
    L = np.repeat(lens, lens)
    rnd_pos = np.repeat((rng.random(n_loc) * lens).astype(np.int64), lens)
    rw = np.full(n, G.READ, np.uint8)
    rw[pat == 1] = G.ATOMIC
    rw[(pat == 2) & (idx_in == 0)] = G.WRITE
    rw[(pat == 3) & (idx_in == L - 1)] = G.WRITE
    rw[(pat == 4) & (idx_in == rnd_pos)] = G.WRITE
    mix = rng.random(n)
    rw[pat == 5] = np.where(mix[pat == 5] < 0.1, G.ATOMIC, np.where(mix[pat == 5] < 0.3, G.WRITE, G.READ))
    a = np.zeros(n, G.REC_DTYPE)
    # entries of a run land in random blocks; the trace is then ordered by (block, interval) (stable)
    a["block"] = rng.integers(0, 512, n)
    a["thread"] = rng.integers(0, 256, n)
    a["interval"] = 0
    a["space"] = G.GLOBAL
    a["size"] = 4
    perm = rng.permutation(n_loc).astype(np.uint64)  # location order unrelated to record order
    a["addr"] = np.uint64(0x10000000000) + np.uint64(4) * perm[loc]
    a["rw"] = rw
    a["value_hash"] = rng.integers(0, 3, n).astype(np.uint64)
    return a[np.argsort(a["block"], kind="stable")]


def exact_counts(a: np.ndarray):
    """(entries at locations touched >= 2 times, those of them at locations with a write) — plain numpy."""
    _, inv, cnt = np.unique(a["addr"], return_inverse=True, return_counts=True)
    wr = np.zeros(len(cnt), bool)
    np.logical_or.at(wr, inv, a["rw"] != G.READ)
    multi = cnt[inv] >= 2
    return int(multi.sum()), int((multi & wr[inv]).sum())


@pytest.mark.parametrize("n_loc,seed,ls", [(40_000, 0, 0), (300_000, 1, 0), (1_500_000, 2, 0), (1_500_000, 3, 1),
                                           (1_000_000, 4, 0)])
def test_write_bit_compaction(S, n_loc, seed, ls):
    a = run_mix_trace(n_loc, seed)
    t = S.Trace(32, ls, 4)
    t.check(S.to_device(a), len(a))
    got = t.races()
    info = t.info()
    t.close()
    exp = O.check(a, warp_size=32, lockstep=ls, granularity=4, method="partitioned")
    assert got.tobytes() == exp.tobytes(), (len(got), len(exp))
    assert info["fused_first_pass"] == 1 and info["wbit_filter"] == 1
    plain, exact = exact_counts(a)
    assert exact <= info["n_multi"] <= plain
    # read-only runs the warps see whole are dropped: most of them
    assert info["n_multi"] - exact <= 0.25 * (plain - exact) + 50_000, (info["n_multi"], exact, plain)


BASE = 0x10000000000 + 4 * 10_000_000  # above run_mix_trace's locations (a small span: the fused path)


def test_write_bit_single_write_positions(S):
    # one long run per pattern, each crossing many warp ranges and batches, plus 2-entry runs around them
    rows = []
    for k, where in enumerate(["none", "first", "last", "middle", "atomic_only", "atomic_plus_read"]):
        m = 30_000
        r = np.zeros(m, G.REC_DTYPE)
        r["block"] = np.arange(m) // 64
        r["thread"] = np.arange(m) % 64
        r["space"] = G.GLOBAL
        r["size"] = 4
        r["addr"] = BASE + 4 * k
        r["rw"] = G.READ
        if where == "first":
            r["rw"][0] = G.WRITE
        elif where == "last":
            r["rw"][-1] = G.WRITE
        elif where == "middle":
            r["rw"][m // 2 + 7] = G.WRITE
        elif where == "atomic_only":
            r["rw"][:] = G.ATOMIC
        elif where == "atomic_plus_read":
            r["rw"][:] = G.ATOMIC
            r["rw"][m - 40] = G.READ
        rows.append(r)
    small = run_mix_trace(200_000, 9, long_frac=0.0)
    a = np.concatenate(rows + [small])
    a = a[np.argsort(a["block"], kind="stable")]
    t = S.Trace(32, 0, 4)
    t.check(S.to_device(a), len(a))
    got = t.races()
    t.close()
    exp = O.check(a, warp_size=32, lockstep=0, granularity=4, method="partitioned")
    assert got.tobytes() == exp.tobytes()
    racy = {x[3] for x in O.race_tuples(got)}
    assert {BASE + 4, BASE + 8, BASE + 12, BASE + 20} <= racy and not {BASE, BASE + 16} & racy


def test_write_bit_kept_but_unused_on_atomic_runs(S):
    # C3-shaped: unique reads + atomics with a few guarded reads into hot bins — no read-only multi-entry
    # locations, so the sample keeps the plain compaction (which strips the bit); the result is unchanged
    rng = np.random.default_rng(5)
    n = 600_000
    a = np.zeros(n, G.REC_DTYPE)
    a["block"] = np.sort(rng.integers(0, 256, n))
    a["thread"] = rng.integers(0, 512, n)
    a["space"] = G.GLOBAL
    a["size"] = 4
    img = rng.random(n) < 0.5
    bins = np.minimum(rng.zipf(1.3, n), 4096).astype(np.uint64)
    a["addr"] = np.where(img, np.uint64(0x10000000000) + np.uint64(4) * np.arange(n, dtype=np.uint64),
                         np.uint64(0x10000000000 + 4 * n) + np.uint64(4) * bins)
    a["rw"] = np.where(img | (rng.random(n) < 1 / 64), G.READ, G.ATOMIC)
    t = S.Trace(32, 0, 4)
    t.check(S.to_device(a), n)
    got = t.races()
    info = t.info()
    t.close()
    exp = O.check(a, warp_size=32, lockstep=0, granularity=4, method="partitioned")
    assert got.tobytes() == exp.tobytes() and len(got) > 0
    assert info["fused_first_pass"] == 1 and info["wbit_filter"] == 0
