"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

C5 (1e9 records) is compared in full with its construction truth; C2 (18.3 M) must be race-free; C3 (101.4 M) and
C4 (412 M) are checked on SAMPLED locations: the oracle gets every record touching a sampled location (taken from
the host generator, which produces the same bytes as the device generator — tests/test_generators.py), and the
GPU's races at those locations must equal the oracle's exactly (witnesses included).  Races are a property of one
location, so this is exact for the sample.  Plus whole-trace invariants.
"""
import numpy as np
import pytest

import sesagen as G
from oracle import oracle as O
from sesagen import configs as C

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
torch = pytest.importorskip("torch")


@pytest.fixture(scope="module")
def S():
    from paper_conf_sc_lilg14_b200 import sesa
    sesa.load()
    return sesa


def sampled_parity(S, dev_recs, n, host_recs, ws, ls, nsample=64, seed=0, benign=False):
    t = S.Trace(ws, ls, 4, benign=benign)
    t.check(dev_recs, n)
    got = t.races()
    t.close()
    assert len(host_recs) == n
    rng = np.random.default_rng(seed)
    gran = host_recs["addr"] // 4
    # sample: locations the GPU reported + random accessed locations (all global in C3/C4)
    pick = set((got["addr"][rng.choice(len(got), min(nsample, len(got)), replace=False)] // 4).tolist()) if len(got) else set()
    pick |= set(gran[rng.integers(0, n, nsample)].tolist())
    pick = np.array(sorted(pick), dtype=np.uint64)
    sel = np.flatnonzero(np.isin(gran, pick))
    exp = O.check(host_recs[sel], warp_size=ws, lockstep=ls, benign=benign)
    exp["first"] = sel[exp["first"].astype(np.int64)]
    exp["second"] = sel[exp["second"].astype(np.int64)]
    got_s = got[np.isin(got["addr"] // 4, pick)]
    assert got_s.tobytes() == exp.tobytes(), (len(got_s), len(exp))
    return got, len(pick), len(sel)


def test_c3_full_size_sampled(S):
    cfg = C.C3()
    dev, n = cfg.device()
    host = cfg.host()
    got, npick, nsel = sampled_parity(S, dev, n, host, 32, 0)
    assert n == 101447621
    # invariants: atomics never race with each other -> every race is RW at a bin (a guard read vs an atomic)
    assert set(got["kind"].tolist()) <= {1}
    bins_lo = cfg.cfg().bins_base
    assert (got["addr"] >= bins_lo).all()
    print(f"C3: {len(got)} races; {npick} sampled locations ({nsel} records) equal to the oracle")


def test_c4_full_size_sampled(S):
    cfg = C.C4()
    dev, n = cfg.device()
    host = cfg.host()
    got, npick, nsel = sampled_parity(S, dev, n, host, 32, 1)
    # invariants: all writes at one location carry the same value -> no WW; races only on dist[]
    assert set(got["kind"].tolist()) == {1}
    c = cfg.cfg()
    assert ((got["addr"] >= c.dist_base) & (got["addr"] < c.dist_base + 4 * (1 << cfg.log2n))).all()
    # lockstep only removes races
    t = S.Trace(32, 0, 4)
    t.check(dev, n)
    nols = t.races()
    t.close()
    key = lambda r: set(zip(r["addr"].tolist(), r["kind"].tolist()))  # noqa: E731
    assert key(got) <= key(nols)
    print(f"C4: {len(got)} races ({len(nols)} without lockstep); {npick} sampled locations ({nsel} records) ok")


def test_c4_full_size_benign(S):
    """Table IV reports the BFS kernel as "W/W (Benign)": with benign reporting the full-size C4 trace
    gets kind-3 records (at `changed` and at dist[] entries written by several frontier threads) and still no
    kind-2 race; sampled locations equal the oracle's, witnesses included."""
    cfg = C.C4()
    dev, n = cfg.device()
    host = cfg.host()
    got, npick, nsel = sampled_parity(S, dev, n, host, 32, 1, benign=True)
    kinds = set(got["kind"].tolist())
    assert kinds == {1, 3}
    assert int(cfg.cfg().changed_base) in set(got["addr"][got["kind"] == 3].tolist())
    print(f"C4 benign: {(got['kind'] == 3).sum()} benign locations; {npick} sampled ({nsel} records) ok")


def test_c5_full_size_truth(S):
    n = 10**9
    dev = C.c5_device(n)
    t = S.Trace(32, 0, 4)
    t.check(dev, n)
    assert t.races().tobytes() == C.c5_truth(n).tobytes()
    t.close()


def test_c2_full_size_race_free_and_mutant(S):
    t = S.Trace(32, 0, 4)
    for fl, expect_races in ((G.c2_flows(), False), (G.c2_mutant_flows(drop_barrier=7), True)):
        d_fl = torch.from_numpy(np.ascontiguousarray(fl).view(np.uint8).reshape(-1)).cuda()
        n = t.expand(d_fl, len(fl))
        out = torch.empty(n * 32, dtype=torch.uint8, device="cuda")
        t.expand(d_fl, len(fl), out, n)
        nr = t.check(out, n)
        assert (nr > 0) == expect_races
        if expect_races:  # parity for the mutant on the shared locations of two blocks (all their records)
            host = O.expand(fl)
            got = t.races()
            assert set(got["space"].tolist()) == {0}  # only the shared tiles lose their barrier
            blocks = (0, 63)
            sel = np.flatnonzero((host["space"] == 0) & np.isin(host["block"], blocks))
            exp = O.check(host[sel])
            exp["first"] = sel[exp["first"].astype(np.int64)]
            exp["second"] = sel[exp["second"].astype(np.int64)]
            assert got[np.isin(got["block"], blocks)].tobytes() == exp.tobytes()
    t.close()
