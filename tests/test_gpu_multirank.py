"""The bench's multi-rank path end to end on one GPU: two torchrun ranks share the
device over a gloo process group (NCCL refuses two ranks on one GPU), strong and
weak batch sharding, max-over-ranks timing and the C1 verification gather with the
oracle check on rank 0.  (A functional test: two ranks on one GPU are not a scaling
measurement.)"""
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


@pytest.mark.parametrize("mode", ["strong", "weak"])
def test_bench_two_ranks_gloo(mode):
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"),
           "--gpus", "2", "--config", "c1", "--backend", "gloo", "--scaling", mode, "--steps", "4",
           "--warmup", "3", "--no-stream", "--no-offload", "--no-e2e"]
    res = subprocess.run(cmd, capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert res.returncode == 0, res.stderr[-3000:]
    lines = [ln for ln in res.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, res.stdout[-2000:]                   # one JSON line, from rank 0
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == mode
    assert d["config"]["global_batch"] == (4 if mode == "strong" else 8)
    assert d["config"]["batch_per_gpu"] == (2 if mode == "strong" else 4)
    v = d["verify"]
    assert v["pass"] and v["ranks"] == 2 and v["max_normwise_err"] <= 2e-3
    assert "gloo" in v["gather"]
