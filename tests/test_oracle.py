"""Pins for the CPU oracle (oracle/sesa_oracle.c) against what the paper and the mathematics fix.

Every expected value here is either printed in the paper (cited PAPER.md line), a closed form derived in the
test from the kernel's text, or brute force on tiny inputs; none comes from the CUDA path.
"""
import itertools

import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O

SH, GL = 0, 1
RW, WW = 1, 2
NOBI = 0xFFFFFFFF


def tuples(races):
    return O.race_tuples(races)


def keyset(races):
    """(λ, kind) projection: independent of record order / witnesses."""
    return {(int(r["space"]), int(r["block"]), int(r["interval"]), int(r["addr"]), int(r["kind"])) for r in races}


def idx_of(recs, **kw):
    m = np.ones(len(recs), bool)
    for k, v in kw.items():
        m &= recs[k] == v
    w = np.flatnonzero(m)
    assert len(w) == 1, (kw, w)
    return int(w[0])


# ------------------------------------------------------------------------------------------------ layouts
def test_layouts_agree():
    assert O.REC_DTYPE == G.REC_DTYPE and O.RACE_DTYPE == G.RACE_DTYPE and O.FLOW_DTYPE == G.FLOW_DTYPE
    O._load()  # asserts the C struct sizes


# ------------------------------------------------------------------------------------------------ F1 race()
def f1_closed_form(B=64, ls=False, distinct=True, ws=32):
    """Expected races of race() derived by hand from P:75 (see tests/golden/f1_race.txt)."""
    r = G.f1_race(B, distinct)
    out = set()
    # interval 0: v[k] written by thread k, read by thread k-1 (mod B): one RW per k (t1=k, t2=k-1).
    for k in range(B):
        w, rd = k, (k - 1) % B
        if ls and w // ws == rd // ws:
            continue
        i = idx_of(r, thread=w, interval=0, rw=1)
        j = idx_of(r, thread=rd, interval=0, rw=0)
        out.add((SH, 0, 0, 4 * k, RW, min(i, j), max(i, j)))
    # interval 1: odd t writes v[t>>2]; even t reads v[t].  v[j] (j < B/4) has writers 4j+1, 4j+3.
    for j in range(B // 4):
        writers = [t for t in (4 * j + 1, 4 * j + 3) if t < B]
        widx = sorted(idx_of(r, thread=t, interval=1, rw=1) for t in writers)
        if distinct and len(writers) == 2:  # WW, no warp exemption for write-write (reading R7)
            out.add((SH, 0, 1, 4 * j, WW, widx[0], widx[1]))
        if j % 2 == 0:  # reader thread j (even) reads v[j]
            ridx = idx_of(r, thread=j, interval=1, rw=0)
            racing = [idx_of(r, thread=t, interval=1, rw=1) for t in writers if not (ls and t // ws == j // ws)]
            if racing:
                cands = sorted((min(ridx, w), max(ridx, w)) for w in racing)
                out.add((SH, 0, 1, 4 * j, RW) + cands[0])
    return out


@pytest.mark.parametrize("method", ["brute", "grouped"])
def test_f1_paper_witnesses(method):
    r = G.f1_race()
    got = tuples(O.check(r, method=method))
    # first interval, WR race on v[0], witness t1.x = 0 (writes v[0]) and t2.x = bdim.x - 1 (reads it)
    i0 = idx_of(r, thread=0, interval=0, rw=1)
    i63 = idx_of(r, thread=63, interval=0, rw=0)
    assert (SH, 0, 0, 0, RW, i0, i63) in got
    # second interval, RW race, e.g. t1.x = 0 (then-part read of v[0]) and t2.x = 1 (else-part write
    # v[1 >> 2] = v[0]); it happens "no matter whether t1 and t2 are within a warp" -> lockstep off.
    a = idx_of(r, thread=0, interval=1, rw=0)
    b = idx_of(r, thread=1, interval=1, rw=1)
    assert (SH, 0, 1, 0, RW, a, b) in got


@pytest.mark.parametrize("method", ["brute", "grouped"])
@pytest.mark.parametrize("ls", [0, 1])
@pytest.mark.parametrize("distinct", [True, False])
def test_f1_closed_form(method, ls, distinct):
    got = set(tuples(O.check(G.f1_race(distinct=distinct), lockstep=ls, method=method)))
    assert got == f1_closed_form(ls=bool(ls), distinct=distinct)
    # counts quoted in DESIGN.md (88 / 22 / 72)
    if not ls:
        assert len(got) == (88 if distinct else 72)
    elif distinct:
        assert len(got) == 22


def test_f1_golden_file():
    """tests/golden/f1_race.txt was written by tests/golden/make_golden.py (oracle only) and is checked
    here against the closed form, so the stored file is pinned by the paper's kernel text."""
    rows = set()
    for line in open("tests/golden/f1_race.txt"):
        if line.startswith("#") or not line.strip():
            continue
        rows.add(tuple(int(x) for x in line.split()))
    assert rows == f1_closed_form()


# ------------------------------------------------------------------------------------------------ F2 / F3
@pytest.mark.parametrize("method", ["brute", "grouped"])
def test_f2_reduction_race_free(method):
    # the WW and RW queries of the reduction interval are unsat -> no race
    r = G.f2_reduction()
    assert len(r) == 189
    for ls in (0, 1):
        assert len(O.check(r, lockstep=ls, method=method)) == 0


@pytest.mark.parametrize("B", [16, 32, 64, 128, 256])
def test_f3_bitonic_race_free(B):
    # Table II: bitonic2.0 reports no races (RR column "-") at #T = 16 ... 256
    r = G.f3_bitonic(B)
    assert len(O.check(r)) == 0
    if B <= 64:
        assert len(O.check(r, method="brute")) == 0


def test_f3_bitonic_mutant_races():
    # deleting the barrier between two steps (merging intervals) must produce races: sanity of the fixture
    r = G.f3_bitonic(32)
    r2 = r.copy()
    r2["interval"] = np.where(r2["interval"] == 3, 2, r2["interval"])
    assert len(O.check(r2)) > 0


# ------------------------------------------------------------------------------------------------ F4 prescan
@pytest.mark.parametrize("method", ["grouped", "brute"])
def test_f4_histo_prescan(method):
    r = G.f4_histo_prescan()
    got = tuples(O.check(r, method=method))
    # closed form: SUM(32) writes Avg/StdDev[16..31] (threads 16..31), SUM(16) in the same interval reads
    # them (threads 0..15 read [t+16]): 16 + 16 RW races, nothing else (each [0..15] is touched by its own
    # thread only, [32..63] only read).
    assert len(got) == 32
    assert {(x[0], x[2], x[3], x[4]) for x in got} == {(SH, 4, base + 4 * k, RW)
                                                       for base in (0, G.F4_STD) for k in range(16, 32)}
    # the write in SUM(stride) by thread <17,0,0> races with the read in SUM(16) by thread <1,0,0>
    w17 = idx_of(r, thread=17, interval=4, rw=1, addr=4 * 17)
    r1 = np.flatnonzero((r["thread"] == 1) & (r["addr"] == 4 * 17) & (r["rw"] == 0))
    assert len(r1) == 1
    assert (SH, 0, 4, 4 * 17, RW, int(r1[0]), w17) in got
    # lockstep: all participants of the last interval are threads < 32 = warp 0 -> the warp-synchronous
    # idiom is exempt (refs [25], [26])
    assert len(O.check(r, lockstep=1, method=method)) == 0
    # but with warp size 1 the race is reported even in lockstep mode
    assert len(O.check(r, lockstep=1, warp_size=1, method=method)) == 32


# ------------------------------------------------------------------------------------------------ F5 binning
def test_f5_binning():
    r = G.f5_binning()
    assert len(r) == 3 * 16896  # Table IV: 16,896 threads
    got = tuples(O.check(r))
    i_r = idx_of(r, block=0, thread=0, rw=0, addr=G.F5_BINCOUNT)
    i_a = idx_of(r, block=0, thread=1, rw=2)
    # exactly one race: RW at binCount_g[0]; atomic-atomic pairs excluded; sample reads unique
    assert got == [(GL, NOBI, NOBI, G.F5_BINCOUNT, RW, i_r, i_a)]
    # the paper's witness (thread bid 32 tid 64 reads, bid 0 tid 0 atomicAdds) is a racing pair
    p = r[idx_of(r, block=32, thread=64, rw=0, addr=G.F5_BINCOUNT)]
    q = r[idx_of(r, block=0, thread=0, rw=2)]
    assert O.pair_kind(p, q) == RW
    got1 = tuples(O.check(r, lockstep=1))
    assert got1 == [(GL, NOBI, NOBI, G.F5_BINCOUNT, RW, i_r, idx_of(r, block=0, thread=32, rw=2))]


# ------------------------------------------------------------------------------------------------ C1
def test_c1_truth_by_construction():
    r = G.c1()
    assert len(r) == 959
    for method in ("brute", "grouped"):
        assert tuples(O.check(r, method=method)) == [(SH, 0, 5, 4, WW, 833, 836)]


# ------------------------------------------------------------------------------------------------ expansion
@pytest.mark.parametrize("name", ["f1", "f1c", "f2", "f5", "c1", "f4"])
def test_expand_matches_direct(name):
    direct, fl = {
        "f1": (G.f1_race(), G.f1_flows()),
        "f1c": (G.f1_race(distinct=False), G.f1_flows(distinct=False)),
        "f2": (G.f2_reduction(), G.f2_flows()),
        "f5": (G.f5_binning(), G.f5_flows()),
        "c1": (G.c1(), G.c1_flows()),
        "f4": (G.f4_histo_prescan(), G.f4_flows()),
    }[name]
    ex = O.expand(fl)
    assert len(ex) == len(direct)
    assert ex.tobytes() == direct.tobytes()


def test_expand_c2_counts_and_race_free():
    fl = G.c2_flows(gx=2, gy=2, K=64)
    ex = O.expand(fl)
    per_thread = 4 + 36 * (64 // 16 - 1) + 33
    assert len(ex) == 4 * 256 * per_thread
    assert len(O.check(ex)) == 0
    mut = O.expand(G.c2_mutant_flows(drop_barrier=2, gx=2, gy=2, K=64))
    assert len(O.check(mut)) > 0


def test_expand_full_c2_count():
    assert len(G.c2_flows()) == 628
    # 16,384 threads x 1,117 records: count without materialising through the C loop
    import ctypes
    lib = O._load()
    f = np.ascontiguousarray(G.c2_flows())
    n = lib.oracle_expand(f.ctypes.data, len(f), None, 0)
    assert n == 16384 * 1117 == 18300928


# ------------------------------------------------------------------------------------------------ brute == grouped
CONFIGS = [dict(ws=32, ls=0, G=4), dict(ws=32, ls=1, G=4), dict(ws=4, ls=1, G=1), dict(ws=1, ls=1, G=2),
           dict(ws=2, ls=0, G=8), dict(ws=8, ls=1, G=16)]


@pytest.mark.parametrize("cfg", CONFIGS)
def test_brute_equals_grouped_random(cfg):
    for seed in range(60):
        n = 1 + (seed * 7) % 90
        r = G.random_trace(n, seed, threads=12 + seed % 50, sort=seed % 3 != 0)
        a = O.check(r, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], method="brute")
        b = O.check(r, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], method="grouped")
        assert a.tobytes() == b.tobytes(), (cfg, seed)


def test_index_base_shifts_witnesses():
    r = G.f1_race()
    a = O.check(r)
    b = O.check(r, index_base=1000)
    assert np.array_equal(a["first"] + 1000, b["first"]) and np.array_equal(a["second"] + 1000, b["second"])


# ------------------------------------------------------------------------------------------------ invariants
def _rand(seed, n=70):
    return G.random_trace(n, seed, threads=40)


@pytest.mark.parametrize("seed", range(25))
def test_invariants(seed):
    r = _rand(seed)
    base = O.check(r)
    # witness validity: P(first, second) holds with the race's kind, both records cover the location
    for x in base:
        a, b = r[int(x["first"])], r[int(x["second"])]
        assert O.pair_kind(a, b) == x["kind"]
        for q in (a, b):
            assert q["space"] == x["space"]
            assert q["addr"] // 4 <= x["addr"] // 4 <= (int(q["addr"]) + int(q["size"]) - 1) // 4
            if x["space"] == SH:
                assert (q["block"], q["interval"]) == (x["block"], x["interval"])
    # lockstep only removes races
    assert keyset(O.check(r, lockstep=1)) <= keyset(base)
    # warp size 1 makes lockstep a no-op
    assert O.check(r, warp_size=1, lockstep=1).tobytes() == O.check(r, warp_size=1).tobytes()
    # permutation invariance of the (λ, kind) projection
    rng = np.random.default_rng(seed)
    assert keyset(O.check(r[rng.permutation(len(r))])) == keyset(base)
    # monotonicity: adding records never removes a (λ, kind)... except benign/ordering are pairwise, so it holds
    extra = _rand(seed + 1000, 20)
    assert keyset(base) <= keyset(O.check(np.concatenate([r, extra])))
    # the witness is the lexicographic minimum: no racing pair at (λ, K) is smaller (brute enumeration)
    for x in base:
        lam = (x["space"], x["block"], x["interval"], x["addr"] // 4)
        for i, j in itertools.combinations(range(int(x["second"]) + 1), 2):
            if (i, j) >= (int(x["first"]), int(x["second"])):
                continue
            a, b = r[i], r[j]
            cover = all(q["space"] == lam[0] and q["addr"] // 4 <= lam[3] <= (int(q["addr"]) + int(q["size"]) - 1) // 4
                        and (q["space"] == GL or (q["block"], q["interval"]) == (lam[1], lam[2])) for q in (a, b))
            assert not (cover and O.pair_kind(a, b) == x["kind"])


def test_all_writes_distinct_values_closed_form():
    """One block, one interval, every record a plain write by its own thread with a distinct value: every
    granule touched by >= 2 records is a WW race witnessed by its two lowest record indices."""
    rng = np.random.default_rng(7)
    n = 300
    r = np.zeros(n, G.REC_DTYPE)
    r["thread"] = np.arange(n)
    r["rw"] = 1
    r["space"] = SH
    r["size"] = 4
    r["addr"] = 4 * rng.integers(0, 90, n)
    r["value_hash"] = np.arange(n) + 1
    exp = []
    for w in sorted(set(r["addr"].tolist())):
        ids = np.flatnonzero(r["addr"] == w)
        if len(ids) >= 2:
            exp.append((SH, 0, 0, w, WW, int(ids[0]), int(ids[1])))
    assert tuples(O.check(r)) == exp
    # same values everywhere: all benign (Table IV "W/W (Benign)")
    r["value_hash"] = 5
    assert len(O.check(r)) == 0


def test_global_ordering_rule():
    """Same block, different intervals of global memory: ordered by __syncthreads (reading R2); different
    blocks: unordered."""
    rows = [(0x1000, 1, 0, 0, 0, 4, GL, 1),   # b0 t0 iv0 W
            (0x1000, 0, 0, 1, 1, 4, GL, 0),   # b0 t1 iv1 R   -> ordered after the barrier, no race
            (0x2000, 1, 0, 0, 0, 4, GL, 1),   # b0 t0 iv0 W
            (0x2000, 0, 1, 1, 1, 4, GL, 0),   # b1 t1 iv1 R   -> other block: race
            (0x3000, 0, 0, 0, 0, 4, GL, 1),   # b0 t0 iv0 W
            (0x3000, 0, 0, 0, 1, 4, GL, 0)]   # same thread, any interval: never a race
    got = tuples(O.check(G.recs(rows)))
    assert got == [(GL, NOBI, NOBI, 0x2000, RW, 2, 3)]


def test_atomics_and_benign_rules():
    rows = [(0x10, 0, 0, 0, 0, 4, GL, 2), (0x10, 0, 1, 0, 0, 4, GL, 2),      # A-A: never
            (0x20, 9, 0, 0, 0, 4, GL, 1), (0x20, 0, 1, 0, 0, 4, GL, 2),      # W-A: WW (A never benign)
            (0x30, 9, 0, 0, 0, 4, GL, 1), (0x30, 9, 1, 0, 0, 4, GL, 1),      # W-W same value: benign
            (0x40, 9, 0, 0, 0, 4, GL, 1), (0x40, 8, 1, 0, 0, 4, GL, 1),      # W-W different values: WW
            (0x50, 0, 0, 0, 0, 4, GL, 0), (0x50, 0, 1, 0, 0, 4, GL, 2)]      # R-A: RW
    got = tuples(O.check(G.recs(rows)))
    assert got == [(GL, NOBI, NOBI, 0x20, WW, 2, 3), (GL, NOBI, NOBI, 0x40, WW, 6, 7),
                   (GL, NOBI, NOBI, 0x50, RW, 8, 9)]


def test_granularity_byte_overlap():
    # G = 1: a 4-byte write at 0x100 and a 1-byte read at 0x103 overlap in byte 0x103 only
    rows = [(0x100, 1, 0, 0, 0, 4, GL, 1), (0x103, 0, 1, 0, 0, 1, GL, 0), (0x104, 0, 2, 0, 0, 1, GL, 0)]
    got = tuples(O.check(G.recs(rows), granularity=1))
    assert got == [(GL, NOBI, NOBI, 0x103, RW, 0, 1)]
    # G = 8: all three share granule 0x100/8 = 0x20
    got8 = tuples(O.check(G.recs(rows), granularity=8))
    assert got8 == [(GL, NOBI, NOBI, 0x100, RW, 0, 1)]


# ------------------------------------------------------------------------------------------------ validation
def test_validation_lowest_bad_index():
    r = G.f1_race()
    r[40]["rw"] = 3
    r[17]["size"] = 0
    assert O.validate(r) == 17
    with pytest.raises(O.OracleError) as e:
        O.check(r)
    assert e.value.code == 1 and e.value.detail == 17
    r2 = G.f1_race()
    r2[5]["addr"] = 2**64 - 2  # addr + size - 1 wraps
    assert O.validate(r2) == 5
    r3 = G.f1_race()
    r3[9]["space"] = 2
    assert O.validate(r3) == 9


def test_bad_config():
    r = G.f1_race()
    for kw in (dict(warp_size=0), dict(lockstep=2), dict(granularity=3), dict(granularity=8192)):
        with pytest.raises(O.OracleError):
            O.check(r, **kw)


def test_empty():
    assert len(O.check(np.zeros(0, G.REC_DTYPE))) == 0


# ------------------------------------------------------------------------------------------------ OOB (NEXT-1)
def _region(base, size, space=G.GLOBAL):
    r = np.zeros(1, G.f6_regions().dtype)
    r["base"], r["size"], r["space"] = base, size, space
    return r


def test_f6_histo_final_oob_closed_form():
    # Fig. 9 / P:569-571: iteration i = t_lin + 47 * 42 * 512 reads bytes [8i, 8i + 8) of an 8,159,232-byte region
    # -> out of bound iff 8 i + 8 > 8,159,232 <=> t_lin >= 9216 (only k = 47); 42 * 512 - 9216 = 12,288 records
    recs = G.f6_histo_final()
    assert len(recs) == 42 * 512 * 48
    count, first = O.oob(recs, G.f6_regions())
    assert count == 42 * 512 - 9216 == 12288
    # lowest index: block 18, thread 0, k = 47 (canonical order block, thread, k)
    assert first == 18 * 512 * 48 + 47
    r = recs[first]
    assert (int(r["block"]), int(r["thread"]), int(r["addr"]) - G.F6_HISTO) == (18, 0, 8 * (9216 + 47 * 21504))
    # the paper's witness bid = <24,0,0>, tid = <0,0,0> is an OOB access of iteration 47
    pw = 24 * 512 * 48 + 47
    addr = int(recs[pw]["addr"]) - G.F6_HISTO
    assert addr + 8 > G.F6_REGION and (int(recs[pw]["block"]), int(recs[pw]["thread"])) == (24, 0)
    # one iteration fewer: nothing is out of bound
    assert O.oob(G.f6_histo_final(iters=47), G.f6_regions()) == (0, None)


def test_oob_boundaries_and_scope():
    recs = np.zeros(5, O.REC_DTYPE)
    recs["space"] = [G.GLOBAL, G.GLOBAL, G.GLOBAL, G.SHARED, G.GLOBAL]
    recs["addr"] = [100, 196, 197, 0, 99]
    recs["size"] = [4, 4, 4, 8, 1]
    reg = _region(100, 100)  # bytes [100, 200)
    # [100,104) in, [196,200) in (last byte 199), [197,201) out, shared not checked (no shared regions), 99 out
    assert O.oob(recs, reg) == (2, 2)
    assert O.oob(recs, reg, index_base=1000) == (2, 1002)
    # a shared region makes the shared record checked: [0, 8) in [0, 8) -> in; [0, 7) -> out
    both = np.concatenate([reg, _region(0, 8, G.SHARED)])
    assert O.oob(recs, both) == (2, 2)
    assert O.oob(recs, np.concatenate([reg, _region(0, 7, G.SHARED)])) == (3, 2)
    # a record spanning two ADJACENT regions is not inside one allocation -> out of bound
    two = np.concatenate([_region(100, 98), _region(198, 2)])
    assert O.oob(recs[1:2], two) == (1, 0)
    assert O.oob(recs, np.zeros(0, reg.dtype)) == (0, None)


# ------------------------------------------------------------------------------------------------ benign W/W (NEXT-4)
WWB = 3


@pytest.mark.parametrize("method", ["brute", "grouped"])
def test_f1_equal_values_benign_closed_form(method):
    """race() of Fig. 2 with every thread writing the same value: the second interval's writes
    v[t >> 2] = ... by the odd threads t = 4k+1, 4k+3 (k = 0..15) are W/W pairs of one value — filtered from the
    race set (72 races, reading R18) and, with benign reporting on, reported as 16 kind-3 records, each witnessed
    by its two writers (record 128 + t: interval 0 holds 2 x 64 records, interval 1 one per thread)."""
    r = G.f1_race(distinct=False)
    plain = O.check(r, method=method)
    rep = O.check(r, method=method, benign=True)
    assert len(plain) == 72 and len(rep) == 88
    assert tuples(rep[rep["kind"] != WWB]) == tuples(plain)
    exp = [(SH, 0, 1, 4 * k, WWB, 128 + 4 * k + 1, 128 + 4 * k + 3) for k in range(16)]
    assert tuples(rep[rep["kind"] == WWB]) == exp
    # distinct values: every such pair is a real W/W race (kind 2), none is benign
    d = G.f1_race(distinct=True)
    assert O.check(d, method=method, benign=True).tobytes() == O.check(d, method=method).tobytes()


def test_benign_pair_rules():
    # rows: (addr, value_hash, block, thread, interval, size, space, rw)
    rows = [(0x30, 9, 0, 0, 0, 4, GL, 1), (0x30, 9, 1, 0, 0, 4, GL, 1),      # same value, other block: benign
            (0x40, 9, 0, 0, 0, 4, GL, 1), (0x40, 8, 1, 0, 0, 4, GL, 1),      # other value: a real WW
            (0x50, 9, 0, 0, 0, 4, GL, 1), (0x50, 9, 0, 0, 0, 4, GL, 1),      # same thread: never
            (0x60, 9, 0, 0, 0, 4, GL, 1), (0x60, 9, 0, 1, 1, 4, GL, 1),      # same block, other interval: ordered
            (0x70, 9, 0, 0, 0, 4, GL, 1), (0x70, 9, 1, 1, 1, 4, GL, 1),      # other block: unordered -> benign
            (0x80, 9, 0, 0, 0, 4, GL, 2), (0x80, 9, 1, 0, 0, 4, GL, 1),      # W-A: a real WW, never benign
            (0x90, 9, 0, 0, 0, 4, GL, 0), (0x90, 9, 1, 0, 0, 4, GL, 1)]      # R-W: RW
    rec = G.recs(rows)
    got = tuples(O.check(rec, benign=True))
    assert got == [(GL, NOBI, NOBI, 0x30, WWB, 0, 1), (GL, NOBI, NOBI, 0x40, WW, 2, 3),
                   (GL, NOBI, NOBI, 0x70, WWB, 8, 9), (GL, NOBI, NOBI, 0x80, WW, 10, 11),
                   (GL, NOBI, NOBI, 0x90, RW, 12, 13)]
    assert O.benign_pair(rec[0], rec[1]) == 1 and O.benign_pair(rec[10], rec[11]) == 0
    # lockstep exempts only pairs with a read: an intra-warp benign pair stays benign
    assert tuples(O.check(rec[:2], benign=True, lockstep=1)) == [(GL, NOBI, NOBI, 0x30, WWB, 0, 1)]


@pytest.mark.parametrize("cfg", CONFIGS)
def test_benign_brute_equals_grouped_random(cfg):
    for seed in range(40):
        n = 1 + (seed * 11) % 120
        r = G.random_trace(n, seed + 500, threads=6 + seed % 20, values=2, write_frac=0.6, atomic_frac=0.1,
                           sort=seed % 3 != 0)
        kw = dict(warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], benign=True)
        a = O.check(r, method="brute", **kw)
        b = O.check(r, method="grouped", **kw)
        assert a.tobytes() == b.tobytes(), (cfg, seed)
        # reporting adds kind-3 records and changes nothing else
        base = O.check(r, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"])
        assert a[a["kind"] != WWB].tobytes() == base.tobytes()
        for x in a[a["kind"] == WWB]:
            assert O.benign_pair(r[int(x["first"])], r[int(x["second"])]) == 1


def test_bfs_shape_is_benign_ww():
    """Table IV reports the Lonestar BFS kernel as "W/W (Benign)": every thread that relaxes a node
    writes the same level, so its write/write conflicts are all benign.  The C4 recipe at 2^10 nodes: with
    benign reporting the trace holds benign W/W records (at `changed` and at dist[] entries written by several
    frontier threads) and no real W/W race."""
    from sesagen import configs as GC
    c4 = GC.C4(log2n=10)
    r = c4.host()
    got = O.check(r, lockstep=1, benign=True)
    kinds = set(got["kind"].tolist())
    assert WW not in kinds and WWB in kinds
    changed = int(c4.cfg().changed_base)
    assert any(int(x["addr"]) == changed and int(x["kind"]) == WWB for x in got)


@pytest.mark.parametrize("G_", [1, 64, 4096])
def test_grouped_equals_brute_wide_accesses(G_):
    """Multi-granule accesses: the grouped oracle agrees with the O(n^2) pair definition (include/sesa.h rules)."""
    import sesagen as G
    for seed in range(4):
        r = G.random_trace(300, 900 + seed, blocks=3, threads=40, intervals=2, words=200,
                           sizes=(1, 3, 8, 64, 300), values=3, sort=seed % 2 == 0)
        for ws, ls in ((32, 0), (4, 1)):
            a = O.check(r, warp_size=ws, lockstep=ls, granularity=G_, method="grouped")
            b = O.check(r, warp_size=ws, lockstep=ls, granularity=G_, method="brute")
            assert a.tobytes() == b.tobytes()


# ------------------------------------------------------------------------------------------------ T-thread mode
@pytest.mark.parametrize("cfg", CONFIGS)
def test_partitioned_equals_grouped(cfg):
    """oracle_check_partitioned (SURVEY §8c.3 T-thread mode: locations split by hash) is byte-identical to the
    1-thread grouped checker, for any thread count."""
    for seed in range(12):
        n = 200 + seed * 900
        r = G.random_trace(n, 3000 + seed, threads=12 + 9 * seed, blocks=1 + seed % 5, words=8 + 40 * seed,
                           sort=seed % 3 != 0)
        a = O.check(r, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], method="grouped")
        b = O.check(r, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], method="partitioned",
                    threads=1 + seed % 6)
        assert a.tobytes() == b.tobytes(), (cfg, seed)


@pytest.mark.parametrize("benign", [False, True])
def test_partitioned_hot_location_parallel_path(benign):
    """A location with >= 2^20 entries takes the multi-threaded sort/count path of group_flags; same result."""
    from sesagen import configs as C
    r = C.rnd_host(1_200_000, 77, blocks=3, threads=256, intervals=2, words=3, shared_frac=0.0, sizes=(4,),
                   values=40, unaligned=False)
    a = O.check(r, warp_size=32, lockstep=1, benign=benign, method="grouped")
    b = O.check(r, warp_size=32, lockstep=1, benign=benign, method="partitioned", threads=4)
    assert len(a) > 0 and a.tobytes() == b.tobytes()


# ------------------------------------------------------------------------------------------------ launches (NEXT-4)
def test_launch_boundary_orders_accesses():
    """Reading R23: the launches of one trace run one after another on the stream, so a write in launch 0 and a
    read of the same word in launch 1 never race, while the same two records in ONE launch (same interval, other
    threads) do.  Closed form: launch 0 = v[k] written by thread k, launch 1 = v[k] read by thread k + 1."""
    B = 64
    r = np.zeros(2 * B, G.REC_DTYPE)
    r["size"] = 4
    r["space"] = 0
    r["addr"][:B] = 4 * np.arange(B)
    r["thread"][:B] = np.arange(B)
    r["rw"][:B] = 1
    r["value_hash"][:B] = np.arange(B) + 1
    r["addr"][B:] = 4 * np.arange(B)
    r["thread"][B:] = (np.arange(B) + 1) % B
    r["rw"][B:] = 0
    one = O.check(r)
    assert len(one) == B and set(one["kind"].tolist()) == {RW}
    for method in ("brute", "grouped", "partitioned"):
        assert len(O.check(r, launches=[0, B, 2 * B], method=method)) == 0
    # within each launch the slices are race-free on their own, too
    assert len(O.check(r[:B])) == 0 and len(O.check(r[B:])) == 0


@pytest.mark.parametrize("seed", range(6))
def test_launches_decompose_per_launch(seed):
    """A multi-launch check is the union of the per-launch checks, each with its records' global indices and its
    launch number in `epoch` (a consequence of λ including the launch; independent index arithmetic here)."""
    rng = np.random.default_rng(seed)
    n = 400 + 50 * seed
    r = G.random_trace(n, 7000 + seed, threads=30, words=20)
    cuts = np.sort(rng.integers(0, n, 3))
    offs = [0, *cuts.tolist(), n]
    got = O.check(r, launches=offs, warp_size=4, lockstep=seed % 2, benign=seed % 3 == 0)
    parts = []
    for e in range(len(offs) - 1):
        p = O.check(r[offs[e]:offs[e + 1]], index_base=offs[e], warp_size=4, lockstep=seed % 2, benign=seed % 3 == 0)
        p["epoch"] = e
        parts.append(p)
    exp = np.concatenate(parts)
    assert got.tobytes() == exp.tobytes()
    # and the F1 race() kernel launched twice: the same 88 races in each launch, indices shifted
    f = G.f1_race()
    two = O.check(np.concatenate([f, f]), launches=[0, len(f), 2 * len(f)])
    a, b = two[two["epoch"] == 0], two[two["epoch"] == 1]
    assert len(a) == len(b) == 88
    assert (b["first"] - a["first"] == len(f)).all() and (b["second"] - a["second"] == len(f)).all()


# ------------------------------------------------------------------------------------------------ precise warps (NEXT-3)
def test_f1_precise_warp_model():
    """race() under the precise warp model (reading R24: P:281 + P:87).  Interval 0 (`v[t] = v[(t+1)%B]`) is
    convergent: an intra-warp read (pc 0) precedes the other thread's write (pc 1) in lockstep, so only the two
    inter-warp pairs race (v[0]: reader 63 / writer 0; v[32]: reader 31 / writer 32).  Interval 1 diverges in
    every warp: the read side and the write side run in either order, so every RW pair races "no matter whether
    t1 and t2 are within a warp", and the two writers of v[j] write at the same instruction: all of
    interval 1 is as without lockstep.  26 races, from the hand-derived lockstep-0 set (f1_closed_form)."""
    r, e = G.f1_race(), G.f1_race_ext()
    full = f1_closed_form(ls=False)
    exp = {x for x in full if x[2] == 1} | {x for x in full if x[2] == 0 and x[3] in (0, 4 * 32)}
    assert len(exp) == 26
    for method in ("brute", "grouped"):
        got = set(tuples(O.check_warp(r, e, lockstep=1, method=method)))
        assert got == exp, method
    # lockstep off: the extension is ignored
    assert O.check_warp(r, e, lockstep=0).tobytes() == O.check(r, lockstep=0).tobytes()


def test_precise_warp_generic_example():
    """Fig. 1's Generic example shape and P:281: two threads of one warp writing one word."""
    def pair(div0, div1, pc0, pc1, v0=1, v1=2, t1=5, rw1=1):
        r = np.zeros(2, G.REC_DTYPE)
        r["size"], r["space"] = 4, 0
        r["thread"] = [3, t1]
        r["rw"] = [1, rw1]
        r["value_hash"] = [v0, v1]
        e = np.zeros(2, O.EXT_DTYPE)
        e["pc"], e["div"] = [pc0, pc1], [div0, div1]
        return [(int(x["kind"])) for x in O.check_warp(r, e, lockstep=1, method="brute")]
    I = 7 << 1
    assert pair(I | 0, I | 1, 10, 11) == [WW]        # the two sides of one branch: both orders occur
    assert pair(I | 0, I | 0, 10, 11) == []          # same side, two instructions: ordered by lockstep
    assert pair(I | 0, I | 0, 10, 10) == [WW]        # same instruction: a simultaneous write
    assert pair(0, 0, 10, 10, v0=4, v1=4) == []      # ... of one value: benign (rule 6)
    assert pair(I | 0, (I + 2) | 1, 10, 11) == []    # sides of two different branch instances: ordered
    assert pair(I | 0, I | 1, 10, 11, rw1=0) == [RW]  # a read on the other side
    assert pair(0, 0, 10, 10, rw1=0) == []           # convergent read/write: ordered by lockstep
    assert pair(0, 0, 10, 11, t1=40) == [WW]         # another warp: the plain rules


def test_precise_warp_reduces_to_coarse_and_f4():
    # one instruction and no divergence anywhere = rule (5) of the coarse model (intra-warp reads exempt,
    # intra-warp writes kept)
    for seed in range(20):
        r = G.random_trace(150, 4000 + seed, threads=64, words=12)
        z = np.zeros(len(r), O.EXT_DTYPE)
        for ws in (32, 4):
            assert O.check_warp(r, z, warp_size=ws).tobytes() == O.check(r, warp_size=ws, lockstep=1).tobytes()
    # histo_prescan (Fig. 8): SUM(32)'s write of Avg[17] happens before SUM(16)'s divergent read in lockstep
    f, fe = G.f4_histo_prescan(), G.f4_histo_prescan_ext()
    assert len(O.check_warp(f, fe)) == 0
    assert len(O.check_warp(f, fe, warp_size=1)) == 32  # warp size 1: the real RW race of P:567


@pytest.mark.parametrize("cfg", CONFIGS)
def test_precise_warp_brute_equals_grouped(cfg):
    for seed in range(40):
        n = 1 + (seed * 13) % 120
        r = G.random_trace(n, 5000 + seed, threads=8 + seed % 70, blocks=1 + seed % 3, words=6 + seed % 20,
                           sort=seed % 3 != 0)
        e = G.random_ext(n, seed, npc=1 + seed % 4, ninst=1 + seed % 3)
        a = O.check_warp(r, e, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], method="brute")
        b = O.check_warp(r, e, warp_size=cfg["ws"], lockstep=cfg["ls"], granularity=cfg["G"], method="grouped")
        assert a.tobytes() == b.tobytes(), (cfg, seed)
