"""The C-ABI library loads and exports every symbol include/*.h declares (CPU, no compute calls)."""
import ctypes
import glob
import os
import re

from paper_conf_sc_00090d00l25_b200 import gllm

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    names = set()
    for h in glob.glob(os.path.join(ROOT, "include", "*.h")):
        src = open(h).read()
        names |= set(re.findall(r"GLLM_API\s+[\w\s\*]+?\b(gllm_\w+)\s*\(", src))
    return sorted(names)


def test_every_declared_symbol_is_exported():
    names = declared_symbols()
    assert len(names) >= 25, names
    L = ctypes.CDLL(gllm.LIB_PATH)
    missing = [n for n in names if not hasattr(L, n)]
    assert not missing, missing


def test_version_and_error_string():
    assert "sm_100a" in gllm.version()
    try:
        gllm.Sched(gllm.SchedCfg(0, 0, 0, 0, 0, 0, 0, 0, 0, 0, 0))
    except gllm.GllmError as e:
        assert e.code == -1 and "cfg" in str(e)
    else:
        raise AssertionError("expected EINVAL")


def test_stage_init_without_gpu_fails_loudly():
    import torch
    if torch.cuda.is_available():
        return
    from workloads.configs import MODELS
    try:
        gllm.Stage(MODELS["C0"], 0, 2, 64, 128, 16)
    except gllm.GllmError as e:
        assert e.code == -3          # ECUDA: no device -> no silent fallback
    else:
        raise AssertionError("stage init must fail without a GPU")
