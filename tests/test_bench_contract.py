"""bench.py contract checks that run on CPU: the --impl reference arm (the
CPU oracle, BASELINE has no installable reference) prints one JSON line with
the contract keys; under a world size > 1 only rank 0 prints."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(args, env=None):
    e = dict(os.environ)
    e.update(env or {})
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True,
                       text=True, timeout=600, env=e, cwd=ROOT)
    assert r.returncode == 0, r.stderr
    return [l for l in r.stdout.splitlines() if l.startswith("{")]


def test_reference_arm_json_line():
    lines = run(["--impl", "reference", "--steps", "2", "--warmup", "1", "--batch", "600",
                 "--cpu-seconds", "0.5"])
    assert len(lines) == 1
    d = json.loads(lines[0])
    for k in ("metric", "value", "unit", "n_gpus", "steps", "warmup", "ms_per_step",
              "higher_is_better", "scaling", "vs_baseline", "dtype", "data", "config",
              "cpu_baseline", "e2e", "impl"):
        assert k in d, k
    assert d["impl"] == "reference" and d["value"] > 0 and d["dtype"] == "f64"
    assert d["e2e"]["h2d_bytes_per_step"] == 0 and d["cpu_baseline"]["kind"] == "oracle"
    assert d["config"]["workload"].startswith("xgc992")


def test_reference_arm_nonzero_rank_is_silent():
    lines = run(["--impl", "reference", "--steps", "1", "--warmup", "0", "--batch", "64"],
                env={"RANK": "1", "WORLD_SIZE": "2", "LOCAL_RANK": "1"})
    assert lines == []


def test_reference_arm_banded_solver():
    """--solver banded --impl reference times the oracle's banded LU (the
    dgbsv analogue's CPU reference) with the same contract keys."""
    lines = run(["--impl", "reference", "--solver", "banded", "--steps", "1", "--warmup", "1",
                 "--batch", "200", "--cpu-seconds", "0.3"])
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference" and d["value"] > 0
    assert d["config"]["solver"].startswith("banded") and "banded LU" in d["note"]
