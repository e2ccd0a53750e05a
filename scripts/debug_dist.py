import sys
sys.path.insert(0, ".")
import numpy as np
import sesagen as G
from oracle import oracle as O
from paper_conf_sc_lilg14_b200 import sesa as S


def shards(n, W):
    return [n * r // W for r in range(W + 1)]


for n, words, W in ((5000, 100, 3), (400, 30, 2), (60, 10, 2), (2000, 100, 1)):
    r = G.random_trace(n, 9, words=words, sort=False)
    got = S.check_loopback(S.to_device(r), shards(len(r), W))
    exp = O.check(r)
    t = S.Trace()
    t.check(S.to_device(r), len(r))
    single = t.races()
    e, g = set(O.race_tuples(exp)), set(O.race_tuples(got))
    print(n, words, W, "single==oracle", single.tobytes() == exp.tobytes(), "loop==oracle", got.tobytes() == exp.tobytes(),
          len(exp), len(got), "missing", sorted(e - g)[:4], "extra", sorted(g - e)[:4])
