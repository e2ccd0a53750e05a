"""Per-rank kernel times of the distributed pipeline, measured with virtual ranks on one GPU (DESIGN.md §6 model).

    ncu --metrics gpu__time_duration.sum --csv --log-file OUT python scripts/loopback_profile.py [W] [n]

Runs sesa_race_check_loopback on the C5 recipe (n records, default 1e9) split into W shards (default 8); the
kernels of each virtual rank run one after another on this GPU, so an ncu launch list gives every rank's kernel
time per phase.  The exchanges are device-to-device copies here (NVLink in a real run: modelled in §6)."""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

from sesagen import configs as C  # noqa: E402
from paper_conf_sc_lilg14_b200 import sesa as S  # noqa: E402

W = int(sys.argv[1]) if len(sys.argv) > 1 else 8
n = int(float(sys.argv[2])) if len(sys.argv) > 2 else 10**9
S.load()
d = C.c5_device(n)
torch.cuda.synchronize()
offs = [r * n // W for r in range(W + 1)]
got = S.check_loopback(d, offs)
exp = C.c5_truth(n)
print(f"W={W} n={n}: {len(got)} races, identical to the construction truth: {got.tobytes() == exp.tobytes()}")
