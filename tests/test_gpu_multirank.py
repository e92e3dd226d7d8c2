"""The multi-rank bench path (shard, evaluate, all-gather of decisions, max-over-
ranks timing) with 2 ranks sharing the box's GPU over host-staged gloo
collectives (SEL_DIST_BACKEND=gloo).  NCCL itself needs one GPU per rank and
is exercised by the driver's 2/4/8-GPU runs."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_bench_two_ranks_one_gpu():
    import __graft_entry__
    __graft_entry__.build()
    env = dict(os.environ, SEL_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--steps", "2", "--warmup", "3", "--candidates", "3000000", "--no-e2e",
           "--no-cpu-baseline", "--no-next"]
    p = subprocess.run(cmd, capture_output=True, text=True, timeout=900, cwd=ROOT, env=env)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [l for l in p.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, p.stdout[-2000:]
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["value"] > 0 and d["invalid"] == 0
    assert d["wa_covered_per_step"] > 0 and d["config"]["candidates"] == 3000000
