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


def _standin(gpus, scaling, batch=16):
    lines = run(["--gpus", str(gpus), "--standin", "--backend", "gloo", "--batch", str(batch),
                 "--nx", "6", "--ny", "5", "--steps", "2", "--warmup", "1", "--scaling", scaling])
    assert len(lines) == 1, lines
    return json.loads(lines[-1])


def test_gpus2_spawns_two_ranks_and_gathers_like_one_process():
    """`bench.py --gpus 2` outside torchrun re-launches itself as 2 ranks
    (the driver's N-GPU entry point), here over gloo with
    the CPU stand-in solver: one JSON line, n_gpus = 2, the gathered
    per-system stats equal the single-process run's bit for bit, and rank 0's
    cross-P re-solve matches every rank."""
    one = _standin(1, "strong")
    two = _standin(2, "strong")
    assert one["n_gpus"] == 1 and two["n_gpus"] == 2
    assert two["gathered"] == one["gathered"]
    assert two["cross_p"]["bitwise_equal"] and two["cross_p"]["ranks"] == 2
    weak = _standin(2, "weak", batch=8)   # 2 x 8 systems = the strong run's 16
    assert weak["gathered"] == one["gathered"] and weak["config"]["global_batch"] == 16
