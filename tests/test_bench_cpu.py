"""bench.py's reference arm (the oracle on host cores) keeps the JSON-line contract on CPU: one line on rank 0
with impl/cpu_baseline/e2e keys, nothing (and exit 0) on other ranks of a multi-rank launch."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(env_extra, *args):
    env = dict(os.environ, **env_extra)
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", *args],
                          capture_output=True, text=True, env=env, cwd=ROOT, timeout=300)


def test_reference_arm_line_rank0():
    r = _run({}, "--steps", "2", "--warmup", "1", "--ref-records", "100000")
    assert r.returncode == 0, r.stderr
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["unit"] == "Grec/s" and d["higher_is_better"] is True
    assert d["steps"] == 2 and d["warmup"] == 1 and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["cpu_baseline"]["value"] == d["value"]
    assert d["e2e"] == {"value": d["value"], "unit": "Grec/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}
    assert "C5" in d["config"]["workload"]


def test_reference_arm_silent_on_other_ranks():
    r = _run({"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"}, "--steps", "1", "--warmup", "1",
             "--ref-records", "100000")
    assert r.returncode == 0 and r.stdout.strip() == ""


def test_gpus_flag_self_launches_one_process_per_gpu():
    """`bench.py --gpus 2` outside torchrun starts torch.distributed.run with 2 ranks itself; rank 0 alone prints
    (shown here with the CPU reference arm, which needs no GPU)."""
    env = {k: v for k, v in os.environ.items() if k not in ("RANK", "WORLD_SIZE", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                        "--steps", "1", "--warmup", "1", "--ref-records", "100000"],
                       capture_output=True, text=True, env=env, cwd=ROOT, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.strip().startswith("{")]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["n_gpus"] == 2
