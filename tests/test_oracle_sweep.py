"""The oracle's checkers against each other on 1e5 random small traces (brute == count on >= 1e5).

``tests/native/oracle_sweep.c`` (a test harness, compiled here with gcc) runs oracle_check_brute (every pair: the
definition of c.1), oracle_check_grouped (inclusion-exclusion counting) and oracle_check_partitioned (the grouped
checker on T threads over a hash partition of the locations) on seeded counter-based traces (sesagen
gen_common.h) with per-trace structure and config drawn from the seed — warp sizes 1..32, lockstep on/off,
granularity 1..64, benign reporting on a third, mixed sizes and unaligned accesses — and requires byte-identical
race lists.  Brute force and counting share only the pair predicate, so a slip in either (a dropped term, a wrong
index, an off-by-one in a range) shows up as a disagreement.
"""
import os
import subprocess

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
EXE = os.path.join(ROOT, "build", "oracle_sweep")


@pytest.fixture(scope="module")
def sweep_exe():
    os.makedirs(os.path.dirname(EXE), exist_ok=True)
    srcs = [os.path.join(ROOT, "tests", "native", "oracle_sweep.c"), os.path.join(ROOT, "oracle", "sesa_oracle.c")]
    subprocess.check_call(["gcc", "-O2", "-std=gnu11", "-pthread", "-I", os.path.join(ROOT, "sesagen", "csrc")] +
                          srcs + ["-o", EXE])
    return EXE


def test_brute_grouped_partitioned_agree_on_1e5_traces(sweep_exe):
    shards, per = 4, 25000
    procs = [subprocess.Popen([sweep_exe, str(k * per), str(per)], stdout=subprocess.PIPE, text=True)
             for k in range(shards)]
    outs = [p.communicate()[0].strip() for p in procs]
    for p, o in zip(procs, outs):
        assert p.returncode == 0, o
    tot = {}
    for o in outs:
        for kv in o.split():
            k, v = kv.split("=")
            tot[k] = tot.get(k, 0) + int(v)
    assert tot["traces"] == shards * per
    # the sweep is not vacuous: race-free and racy traces, all three kinds
    assert 0 < tot["racy"] < tot["traces"]
    assert tot["rw"] > 0 and tot["ww"] > 0 and tot["benign"] > 0
    print(tot)
