"""bench.py under torchrun with 2 ranks (the driver's N > 1 launch), on the
gloo wire so both ranks can share one GPU: the JSON line, the fixed-config
strong-scaling block (configs[4] shape, shrunk) and the separately reported
broadcast / placement / all-gather times."""
from __future__ import annotations

import json
import os
import signal
import socket
import subprocess
import sys

import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _torchrun(extra, env_extra=None, timeout=300):
    # gloo over the loopback interface (the box's hostname may not resolve)
    env = dict(os.environ, TT_DIST_BACKEND="gloo", GLOO_SOCKET_IFNAME="lo", TT_BENCH_TRACE="1", **(env_extra or {}))
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
           "--master-addr=127.0.0.1", f"--master-port={_free_port()}", os.path.join(ROOT, "bench.py"),
           "--gpus", "2"] + extra
    # own process group, so that a hang kills torchrun and both ranks
    p = subprocess.Popen(cmd, cwd=ROOT, env=env, stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True,
                         start_new_session=True)
    try:
        out, err = p.communicate(timeout=timeout)
    except subprocess.TimeoutExpired:
        os.killpg(p.pid, signal.SIGKILL)
        out, err = p.communicate()
        raise AssertionError(f"torchrun timed out after {timeout} s; trace:\n{err[-4000:]}")
    return subprocess.CompletedProcess(cmd, p.returncode, out, err)


@pytest.mark.gpu
def test_bench_two_ranks_line():
    r = _torchrun(["--steps", "2", "--warmup", "3", "--points-per-rank", "64000", "--strong-points", "256000",
                   "--no-cpu-baseline", "--no-e2e", "--no-chase"])
    assert r.returncode == 0, r.stderr[-3000:]  # (phase trace of both ranks in stderr)
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout  # rank 0 alone prints
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["scaling"] == "weak"
    assert d["config"]["global_points"] == 128000
    assert d["bcast_ms"] is not None and d["placement_ms"] is not None and d["allgather_ms"] is not None
    s = d["strong_16m"]
    # cost-balanced shards: rank 0's is warp-aligned and near half
    assert s["scaling"] == "strong" and s["points"] == 256000
    assert s["points_per_rank"] % 64 == 0 and abs(s["points_per_rank"] - 128000) < 12800
    assert s["value"] > 0 and s["bcast_ms"] is not None and s["allgather_ms"] is not None
    assert s["shards"].startswith("cost-balanced")
    # balanced within a warp of points of the ideal (the rounding can leave
    # it a hair above an already even equal-count split)
    assert s["shard_cost_max_over_mean"]["balanced"] <= max(s["shard_cost_max_over_mean"]["equal_count"], 1.01)
    sk = d["strong_16m_knn"]
    assert sk["workload"] == "knn_16m_7d" and sk["points"] == 256000
    assert sk["points_per_rank"] % 64 == 0 and abs(sk["points_per_rank"] - 128000) < 38400
    assert sk["value"] > 0 and sk["bcast_ms"] is not None and sk["allgather_ms"] is not None
    assert sk["shard_cost_max_over_mean"]["balanced"] <= max(sk["shard_cost_max_over_mean"]["equal_count"], 1.01)


@pytest.mark.gpu
def test_bench_uneven_shards_fail_loudly():
    r = _torchrun(["--steps", "1", "--warmup", "3", "--points-per-rank", "64000", "--strong-points", "100001",
                   "--no-cpu-baseline", "--no-e2e", "--no-chase"])
    assert r.returncode != 0
    assert "equal warp-aligned shards" in (r.stdout + r.stderr)
