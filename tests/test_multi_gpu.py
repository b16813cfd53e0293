"""Multi-process runs of the sharded path
through torchrun:
  * NCCL over NVLink, one rank per GPU -- skipped unless >= 2 GPUs are
    visible (the lease here has one);
  * every rank on GPU 0 over gloo: the same code path of tools/dist_check.py
    (bit-exact shards and reconstruction vs the oracle) and bench.py's
    sharded RTM mode (both all-gathers inside the timed region).
"""
from __future__ import annotations

import json
import os
import socket
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port() -> int:
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _torchrun(n: int, args: list[str], share: bool, timeout=1200):
    env = dict(os.environ, OMP_NUM_THREADS="1")
    if share:
        env["CUSZP_BENCH_SHARE_GPU"] = "1"
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={n}",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), *args]
    return subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=timeout)


@pytest.mark.skipif(torch.cuda.device_count() < 2, reason="needs >= 2 GPUs for NCCL ranks")
@pytest.mark.parametrize("n", [2, 4, 8])
def test_nccl_ranks_bit_exact(n):
    if torch.cuda.device_count() < n:
        pytest.skip(f"needs {n} GPUs")
    r = _torchrun(n, [os.path.join("tools", "dist_check.py")], share=False)
    assert r.returncode == 0 and f"world={n}" in r.stdout and "ok=True" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]


def test_two_ranks_one_gpu_gloo_bit_exact():
    r = _torchrun(2, [os.path.join("tools", "dist_check.py")], share=True)
    assert r.returncode == 0 and "ok=True" in r.stdout, r.stdout[-2000:] + r.stderr[-4000:]


@pytest.mark.slow
def test_bench_sharded_rtm_two_ranks_one_gpu():
    r = _torchrun(2, ["bench.py", "--gpus", "2", "--steps", "2", "--warmup", "3", "--no-e2e"], share=True)
    assert r.returncode == 0, r.stderr[-4000:]
    line = json.loads(r.stdout.strip().splitlines()[-1])
    assert line["n_gpus"] == 2 and line["config"]["workload"] == "c5_rtm"
    assert sum(line["config"]["n_per_rank"]) == line["config"]["n_elements"] and len(line["config"]["n_per_rank"]) == 2
    assert line["value"] > 0 and line["scaling"] == "strong"
