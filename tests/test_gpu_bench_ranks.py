"""bench.py's N > 1 path (independent replicas, no data-path
collective; the process group carries the start barrier and the
max-over-ranks / summed reductions) run as two ranks sharing one GPU over
gloo, launched the way the driver launches it (torch.distributed.run)."""
from __future__ import annotations

import json
import os
import socket
import subprocess
import sys

import pytest
import torch

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a GPU", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_two_ranks_on_one_gpu_gloo():
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2",
           "--workload", "B", "--steps", "3", "--warmup", "3", "--dist-backend", "gloo", "--no-cpu-baseline",
           "--mig-blocks", "64"]
    r = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]  # rank 0 alone prints the line
    d = json.loads(lines[0])
    assert d["n_gpus"] == 2 and d["scaling"] == "weak" and d["value"] > 0
    assert d["config"]["dist_backend"] == "gloo"
    assert d["e2e"]["value"] > 0 and d["migration"]["aggregate_h2d_gbs"] > 0
    # summed work of two replicas (seeds 2 and 1002) over the max time
    assert abs(d["value"] * d["ms_per_step"] / 1000.0 - 2 * d["config"]["records_per_step"]) \
        < 0.05 * d["value"] * d["ms_per_step"] / 1000.0
