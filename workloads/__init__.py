"""Seeded synthetic workloads shared by the oracle and the product path.

This package holds ONLY input generation and configuration data: model shapes,
scheduler hyper-parameters and request streams.  It contains none of the
method's arithmetic (no throttling, no block management, no forward math), so
that `oracle/` and `paper_conf_sc_00090d00l25_b200/` can both import it while
sharing no code with each other.
"""
from .configs import MODELS, SCHED, STREAMS, ModelShape, SchedParams, config
from .streams import Request, Stream, make_stream

__all__ = ["MODELS", "SCHED", "STREAMS", "ModelShape", "SchedParams", "config",
           "Request", "Stream", "make_stream"]
