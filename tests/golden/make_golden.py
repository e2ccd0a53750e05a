"""Writes the stored fixtures of tests/golden/ by calling ONLY oracle/ (never the CUDA path).

Each file's header cites the paper passage that pins it; tests/test_oracle.py checks every stored row set
against a closed form derived from the kernel's text, so the files are pinned by the paper, not by the oracle.
Run from the repo root:  python tests/golden/make_golden.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.dirname(os.path.abspath(__file__)))))
import sesagen as G  # noqa: E402
from oracle import oracle as O  # noqa: E402

HERE = os.path.dirname(os.path.abspath(__file__))
FIXTURES = {
    "f1_race.txt": (G.f1_race, dict(), "race() of P:75 (PAPER.md §II), B=64, distinct write values; "
                    "P:79-81 witness (t0 W, t63 R) on v[0] in interval 0; P:87 witness (t0 R, t1 W) in interval 1"),
    "f1_race_lockstep.txt": (G.f1_race, dict(lockstep=1), "race() with warp-lockstep (P:281, reading R6)"),
    "f4_histo_prescan.txt": (G.f4_histo_prescan, dict(), "Fig. 8 histo_prescan (P:587-601); P:567 witness "
                             "thread <17,0,0> W vs <1,0,0> R on Avg[17]"),
    "f5_binning.txt": (G.f5_binning, dict(), "Fig. 10 binning (P:617-629); P:573 inter-block R vs atomicAdd"),
    "c1_reduction.txt": (G.c1, dict(), "BASELINE config 1 (Fig. 1 Reduction P:111 + one injected WW)"),
}

for name, (gen, kw, cite) in FIXTURES.items():
    races = O.check(gen(), **kw)
    with open(os.path.join(HERE, name), "w") as f:
        f.write(f"# {cite}\n# written by tests/golden/make_golden.py (oracle only); config warp_size=32 "
                f"granularity=4 {kw}\n# space block interval addr kind first second\n")
        for t in O.race_tuples(races):
            f.write(" ".join(str(x) for x in t) + "\n")
    print(name, len(races))
