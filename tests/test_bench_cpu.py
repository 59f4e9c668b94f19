"""bench.py contract checks that run without a GPU: the reference arm of this tier (the CPU
oracle timed on the host cores) prints one JSON line with the base contract's keys, and
ranks other than 0 exit without work under torchrun."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None):
    e = dict(os.environ)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True,
                          text=True, timeout=600, env=e, cwd=ROOT)


def test_reference_arm_json_line():
    r = _run(["--impl", "reference", "--steps", "2", "--warmup", "3", "--config", "toy-a"])
    assert r.returncode == 0, r.stderr
    lines = [l for l in r.stdout.splitlines() if l.strip()]
    assert len(lines) == 1
    d = json.loads(lines[0])
    assert d["impl"] == "reference"
    assert d["metric"] == "candidate configs evaluated/sec" and d["unit"] == "configs/s"
    assert d["higher_is_better"] is True and d["value"] > 0
    assert d["steps"] == 2 and d["warmup"] == 3
    cb = d["cpu_baseline"]
    assert cb["kind"] == "oracle" and cb["cores"] >= 1 and cb["value"] == d["value"] and cb["sample"]
    assert d["e2e"] == {"value": d["value"], "unit": "configs/s", "h2d_bytes_per_step": 0,
                        "d2h_bytes_per_step": 0}
    assert d["config"]["workload"]


def test_reference_arm_other_ranks_exit_quietly():
    r = _run(["--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "3", "--config", "toy-a"],
             env={"RANK": "1", "WORLD_SIZE": "2"})
    assert r.returncode == 0, r.stderr
    assert r.stdout.strip() == ""


def test_gpus_mismatch_with_world_size_is_refused():
    r = _run(["--impl", "reference", "--gpus", "4", "--steps", "1", "--config", "toy-a"],
             env={"RANK": "0", "WORLD_SIZE": "2"})
    assert r.returncode == 2 and "WORLD_SIZE" in r.stderr


def test_gpus_n_self_launches_n_ranks():
    """--gpus 2 without torchrun relaunches under torch.distributed.run: two ranks, rank 0
    alone prints (the reference arm needs no GPU)."""
    r = _run(["--impl", "reference", "--gpus", "2", "--steps", "1", "--warmup", "1", "--config", "toy-a"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1 and json.loads(lines[0])["n_gpus"] == 2
