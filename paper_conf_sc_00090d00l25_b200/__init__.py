"""B200-native per-stage mixed-batch forward of gLLM (SC'25): Token-Throttling scheduler,
paged-KV block manager and the tcgen05 stage forward, behind the C ABI in include/gllm.h.

`gllm` is the ctypes binding (marshalling only); `runtime` drives stages as a pipeline.
"""
from . import gllm  # noqa: F401

__all__ = ["gllm"]
