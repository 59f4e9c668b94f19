"""bench.py with two ranks (torchrun) on one GPU: the N > 1 host path — per-rank shards with
global offsets, per-step packed keys gathered into a vector and all-reduced (MIN), max-over-ranks
timing, rank-0 JSON line — checked against the oracle's selection over the union of the two
shards of the last timed step. NCCL refuses two ranks on one GPU, so the collective runs on the
test-only gloo backend (ACESO_BENCH_BACKEND=gloo; eager issue instead of a CUDA graph)."""
import json
import os
import socket
import subprocess
import sys

import numpy as np
import pytest

import aceso_inputs as ai
import oracle
from aceso_inputs import profiles as P

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.gpu
def test_bench_two_ranks_selects_the_global_oracle_optimum():
    steps, world = 12, 2
    env = dict(os.environ, ACESO_BENCH_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", "--master-port", str(_free_port()), "bench.py",
           "--gpus", str(world), "--steps", str(steps), "--warmup", "3", "--config", "gpt3-1.3b",
           "--no-cpu", "--no-e2e", "--no-dedup", "--no-dp", "--no-all", "--search-budget", "0"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.strip().splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == world and d["value"] > 0 and d["steps"] == steps
    n = d["config"]["batch_per_gpu"]
    nbuf = int(d["config"]["l2"].split()[0])
    b = (steps - 1) % nbuf  # the last timed step's batch buffer
    prof = P.WORKLOADS["gpt3-1.3b"]()
    parts = [ai.search_shaped(prof, 20240422, (b * world + rk) * n, n, group_size=1024) for rk in range(world)]
    codes = np.concatenate([c for c, _ in parts])
    hdr = np.concatenate([h for _, h in parts])
    o = oracle.evaluate(prof, codes, hdr, threads=16)
    assert (d["result"]["cls"], d["result"]["cost"], d["result"]["index"]) == oracle.select(o)


@pytest.mark.gpu
def test_bench_captured_nccl_key_vector_one_rank():
    """The graph-captured per-step key vector + NCCL all-reduce MIN path (the one a multi-GPU
    run times) on a one-rank NCCL group (ACESO_BENCH_FORCE_DIST=1): captured, and the global
    selection of the last step equals the oracle's."""
    steps = 40
    env = dict(os.environ, ACESO_BENCH_FORCE_DIST="1", WORLD_SIZE="1", RANK="0", LOCAL_RANK="0",
               MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port()))
    cmd = [sys.executable, "bench.py", "--gpus", "1", "--steps", str(steps), "--warmup", "3",
           "--config", "gpt3-1.3b", "--no-cpu", "--no-dedup", "--no-dp", "--no-all", "--search-budget", "0",
           "--keys-per-allreduce", "16"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.strip().splitlines() if l.startswith("{")][-1])
    assert d["timing"].startswith("K steps captured in one CUDA graph"), d["timing"]
    assert "NCCL" in d["config"]["parallelism"] and d["e2e"]["value"] > 0
    n = d["config"]["batch_per_gpu"]
    nbuf = int(d["config"]["l2"].split()[0])
    b = (steps - 1) % nbuf
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, hdr = ai.search_shaped(prof, 20240422, b * n, n, group_size=1024)
    o = oracle.evaluate(prof, codes, hdr, threads=16)
    assert (d["result"]["cls"], d["result"]["cost"], d["result"]["index"]) == oracle.select(o)


@pytest.mark.gpu
def test_bench_fused_global_key_symmetric_memory_one_rank():
    """--global-select symm: every timed launch joins rank 0's symmetric-memory key slot by an
    atomic MIN (aceso_eval_global through the peer mapping; here one rank maps its own buffer);
    no collective per step. The last step's global selection equals the oracle's."""
    steps = 24
    env = dict(os.environ, ACESO_BENCH_FORCE_DIST="1", WORLD_SIZE="1", RANK="0", LOCAL_RANK="0",
               MASTER_ADDR="127.0.0.1", MASTER_PORT=str(_free_port()))
    cmd = [sys.executable, "bench.py", "--gpus", "1", "--steps", str(steps), "--warmup", "3",
           "--config", "gpt3-1.3b", "--no-cpu", "--no-e2e", "--no-dedup", "--no-dp", "--no-all",
           "--search-budget", "0", "--global-select", "symm"]
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    d = json.loads([l for l in r.stdout.strip().splitlines() if l.startswith("{")][-1])
    assert d["timing"].startswith("K steps captured in one CUDA graph"), d["timing"]
    assert "symmetric" in d["config"]["parallelism"]
    n = d["config"]["batch_per_gpu"]
    nbuf = int(d["config"]["l2"].split()[0])
    b = (steps - 1) % nbuf
    prof = P.WORKLOADS["gpt3-1.3b"]()
    codes, hdr = ai.search_shaped(prof, 20240422, b * n, n, group_size=1024)
    o = oracle.evaluate(prof, codes, hdr, threads=16)
    assert (d["result"]["cls"], d["result"]["cost"], d["result"]["index"]) == oracle.select(o)
