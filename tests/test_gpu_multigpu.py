"""Multi-GPU parity (SURVEY 8(e), §4 'Multi-GPU parity'): the
partitioned evaluation with the halo sum equals the serial CPU oracle on every
rank's nodes (R and the halo-summed J.v output Y within 1e-12 of sum|contrib|),
and the valence probe is bit-exact through the halo, for both halo paths
(fused peer-memory atomics, and pack / NCCL send-recv / unpack-add).

Runs tests/_multirank.py under torch.distributed.run (one process per rank):
  >= 2 visible GPUs  world = 2, 4, 8 (capped at the GPU count), NCCL, one GPU per rank
                     (the data plane the N>1 bench uses: CUDA IPC peer pointers over NVLink)
  1 visible GPU      world = 2, 3 sharing GPU 0 over gloo (same kernels, same IPC mapping
                     between processes; the NCCL transport itself is not exercised)
Also checks that `bench.py --gpus N` starts its own ranks and reports n_gpus = N
with the halo check inside the line."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _gpus():
    import torch
    return torch.cuda.device_count() if torch.cuda.is_available() else 0


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worlds():
    n = _gpus()
    if n == 0:
        return []
    if n == 1:
        return [2, 3]
    return [w for w in (2, 4, 8) if w <= n]


def _run_multirank(world, configs, timeout=900):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={world}",
           "--master-addr", "127.0.0.1", f"--master-port={_port()}", os.path.join(ROOT, "tests", "_multirank.py"),
           "--configs", configs]
    p = subprocess.run(cmd, capture_output=True, text=True, timeout=timeout, cwd=ROOT)
    assert p.returncode == 0, p.stdout[-3000:] + p.stderr[-3000:]
    lines = [ln for ln in p.stdout.splitlines() if ln.startswith("{")]
    assert lines, p.stdout[-2000:] + p.stderr[-2000:]
    return json.loads(lines[-1])


@pytest.mark.parametrize("world", [2, 3, 4, 8])
def test_partitioned_halo_sum_equals_oracle(world):
    if world not in _worlds():
        pytest.skip(f"world {world} not run with {_gpus()} visible GPU(s)")
    configs = "C1,C1w,C4p" if world <= 4 else "C1,C4p"
    out = _run_multirank(world, configs)
    assert out["world"] == world
    assert out["backend"] == ("nccl" if _gpus() >= world else "gloo")
    assert len(out["results"]) == 2 * len(configs.split(","))
    for r in out["results"]:
        bad = [x for x in r["ranks"] if not x["ok"]]
        assert r["ok"] and not bad, json.dumps(bad)[:2000]
        # every rank had at least one neighbour: the halo actually carried data
        assert all(x["neighbors"] for x in r["ranks"])


def test_bench_gpus_n_self_launch():
    """`python bench.py --gpus 2` (no torchrun environment) starts 2 ranks itself
    and rank 0 prints n_gpus = 2 with the halo check in the line."""
    n = _gpus()
    if n == 0:
        pytest.skip("no CUDA device")
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    if n < 2:
        env["STOKESFO_BENCH_BACKEND"] = "gloo"
    for halo in ("p2p", "nccl"):
        cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--config", "C4p", "--steps", "3",
               "--warmup", "3", "--check", "--halo", halo, "--no-e2e"]
        p = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
        assert p.returncode == 0, p.stdout[-3000:] + p.stderr[-3000:]
        line = json.loads([ln for ln in p.stdout.splitlines() if ln.startswith("{")][-1])
        assert line["n_gpus"] == 2
        assert len(line["per_rank"]) == 2
        assert line["halo"].startswith("fused" if halo == "p2p" else "nccl")
        assert line["halo_check_max_rel_err"] <= 1e-12
