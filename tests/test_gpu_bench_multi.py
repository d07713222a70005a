"""bench.py at N = 2 (one process per GPU under torch.distributed.run, the driver's launch line),
with both stage hand-offs.  Skips when fewer than 2 GPUs are visible (the gpurun boxes of this
build have one).  Checks the JSON contract: n_gpus, one bubble fraction per stage measured from
CUDA events in the real pipeline, the hand-off used."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


@pytest.mark.timeout(1200)
@pytest.mark.parametrize("handoff", ["peer", "nccl"])
def test_bench_two_gpus(handoff):
    import torch
    if torch.cuda.device_count() < 2:
        pytest.skip("needs 2 GPUs")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2",
           "--master-addr", "127.0.0.1", "--master-port", str(_port()), "bench.py", "--gpus", "2",
           "--steps", "4", "--warmup", "3", "--preroll", "60", "--handoff", handoff, "--no-cpu-baseline"]
    p = subprocess.run(cmd, cwd=ROOT, capture_output=True, text=True, timeout=1100)
    assert p.returncode == 0, p.stderr[-3000:]
    line = [l for l in p.stdout.splitlines() if l.startswith("{")][-1]
    out = json.loads(line)
    assert out["n_gpus"] == 2 and out["config"]["handoff"] == handoff
    assert len(out["bubble_fraction"]["per_stage"]) == 2
    assert out["value"] > 0 and out["e2e"]["value"] > 0
    if handoff == "nccl":
        assert "NCCL communicator nranks=2" in p.stderr
