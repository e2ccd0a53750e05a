"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py times.

Every config is compared IN FULL: C5 (1e9 records) with its construction truth (itself pinned to the oracle at
reduced size, tests/test_oracle.py); C2 (18.3 M, and its one-barrier-removed mutant), C3 (101.4 M) and C4 (412 M,
with and without benign reporting) with the T-thread oracle (oracle_check_partitioned) run on the same bytes copied
back from the device — every race record, witnesses included (byte equality of the sorted race arrays).  Plus
whole-trace invariants.
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


def full_parity(S, dev_recs, n, ws, ls, benign=False, lockstep_subset=False):
    """The GPU race list of the whole trace against the T-thread oracle (oracle_check_partitioned, byte-identical
    to the 1-thread grouped checker) on the SAME bytes, copied back from the device: every race, every witness."""
    t = S.Trace(ws, ls, 4, benign=benign)
    t.check(dev_recs, n)
    got = t.races()
    t.close()
    host = dev_recs.cpu().numpy().view(G.REC_DTYPE)
    assert len(host) == n
    exp = O.check(host, warp_size=ws, lockstep=ls, benign=benign, method="partitioned")
    assert len(got) == len(exp), (len(got), len(exp))
    assert got.tobytes() == exp.tobytes()
    return got, host


def test_c3_full_size_parity(S):
    cfg = C.C3()
    dev, n = cfg.device()
    assert n == 101447621
    got, host = full_parity(S, dev, n, 32, 0)
    # invariants: atomics never race with each other -> every race is RW at a bin (a guard read vs an atomic)
    assert set(got["kind"].tolist()) <= {1}
    assert (got["addr"] >= cfg.cfg().bins_base).all()
    print(f"C3: {len(got)} races equal to the oracle's over all {n} records")


def test_c4_full_size_parity(S):
    """C4 (lockstep) in full, with and without benign reporting, against ONE oracle run with benign reporting (its
    kinds 1-2 are the plain list: rule (6) keeps benign pairs out of them either way).  Table IV reports the BFS
    kernel as "W/W (Benign)": kind-3 records appear (at `changed` and at dist[] entries written by several
    frontier threads) and still no kind-2 race."""
    cfg = C.C4()
    dev, n = cfg.device()
    host = dev.cpu().numpy().view(G.REC_DTYPE)
    exp = O.check(host, warp_size=32, lockstep=1, benign=True, method="partitioned")
    for benign in (False, True):
        t = S.Trace(32, 1, 4, benign=benign)
        t.check(dev, n)
        got = t.races()
        t.close()
        want = exp if benign else exp[exp["kind"] != 3]
        assert len(got) == len(want) and got.tobytes() == want.tobytes()
    assert set(exp["kind"].tolist()) == {1, 3}
    assert int(cfg.cfg().changed_base) in set(exp["addr"][exp["kind"] == 3].tolist())
    # invariants: all writes at one location carry the same value -> no WW; races only on dist[]
    rw = exp[exp["kind"] == 1]
    c = cfg.cfg()
    assert ((rw["addr"] >= c.dist_base) & (rw["addr"] < c.dist_base + 4 * (1 << cfg.log2n))).all()
    # lockstep only removes races
    t = S.Trace(32, 0, 4)
    t.check(dev, n)
    nols = t.races()
    t.close()
    key = lambda r: set(zip(r["addr"].tolist(), r["kind"].tolist()))  # noqa: E731
    assert key(rw) <= key(nols)
    print(f"C4: {len(rw)} races ({len(nols)} without lockstep), {(exp['kind'] == 3).sum()} benign locations: "
          f"equal to the oracle's over all {n} records")


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
        host = O.expand(fl)  # the oracle's own expansion of the same descriptors
        assert out.cpu().numpy().tobytes() == host.tobytes()  # the whole expansion, byte for byte
        got = t.races()
        exp = O.check(host, method="partitioned")  # the whole race list of the expanded trace
        assert got.tobytes() == exp.tobytes()
        if expect_races:
            assert set(got["space"].tolist()) == {0}  # only the shared tiles lose their barrier
    t.close()
