"""Programmatic dependent launch (csrc/launch.cuh): the stage path must agree with the oracle with
PDL on and off.  PDL is on by default, so the rest of the -m gpu suite covers it; GLLM_PDL is read
once per process, so the PDL-off mode runs parity cases spanning the GEMM schedules (stream-K,
whole tiles), both attention kernels and chunked prefill in a child pytest process."""
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

CASES = "c0_mixed_batch or c0b_chunked or gqa_bias or c1_stream_long_chunk"


@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["0"])
def test_stage_parity_without_pdl(mode):
    env = dict(os.environ, GLLM_PDL=mode)
    r = subprocess.run(
        [sys.executable, "-m", "pytest", "-q", "-x", "-m", "gpu", "-p", "no:cacheprovider",
         os.path.join(ROOT, "tests", "test_gpu_parity.py"), "-k", CASES],
        cwd=ROOT, env=env, capture_output=True, text=True, timeout=900)
    tail = (r.stdout + r.stderr)[-3000:]
    assert r.returncode == 0, f"GLLM_PDL={mode}:\n{tail}"
    assert " passed" in r.stdout and "deselected" in r.stdout, tail
