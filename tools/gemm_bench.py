"""Micro-benchmark of the stage GEMM through gllm_op_gemm (CUDA events, L2-flushed between reps).

    python tools/gemm_bench.py [--shapes C1]      # prints one line per (M, N, K, epi)
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_00090d00l25_b200 import gllm  # noqa: E402

SHAPES = {
    # (M, N, K, epi): C1 projections at the PP=1 window mean T ~ 2094, and C4's small-T stage
    "C1": [(2094, 6144, 4096, 0), (2094, 4096, 4096, 1), (2094, 28672, 4096, 2), (2094, 4096, 14336, 1)],
    "C4": [(128, 10240, 8192, 0), (128, 8192, 8192, 1), (128, 57344, 8192, 2), (128, 8192, 28672, 1)],
    "sq": [(8192, 8192, 8192, 0)],
    # emulated PP stages at their window-mean T: C2 (PP=4, T ~ 625) and C3 (PP=8, T ~ 900)
    "C2": [(625, 7168, 5120, 0), (625, 5120, 5120, 1), (625, 27648, 5120, 2), (625, 5120, 13824, 1)],
    "C3": [(900, 7168, 5120, 0), (900, 5120, 5120, 1), (900, 55296, 5120, 2), (900, 5120, 27648, 1)],
    # C3's O shape with the plain store epilogue, and with K cut to 512 / 1024 (prologue + epilogue
    # dominated): separates the residual epilogue's cost from the mainloop's
    "C3s": [(900, 5120, 5120, 0), (900, 5120, 512, 1), (900, 5120, 512, 0), (900, 5120, 1024, 1), (900, 5120, 1024, 0)],
    # small-T fixed vs per-k-block cost: C4's O shape with K from 1k to 16k (store / residual epilogues)
    "C4k": [(128, 8192, k, e) for e in (0, 1) for k in (1024, 2048, 4096, 8192, 16384)],
    # the C1 O / down shapes with the plain bf16-store epilogue (isolates the residual epilogue)
    "C1s": [(2094, 4096, 4096, 0), (2094, 4096, 14336, 0)],
    # LM head + greedy argmax (epi 3) at the sampled-row counts of C1 (~800), C2 (~250), C3 (~15), C4 (128)
    "lm": [(800, 128256, 4096, 3), (250, 152064, 5120, 3), (300, 152064, 5120, 3), (16, 152064, 5120, 3),
           (128, 128256, 8192, 3)],
}


_FLUSH = None


def flush_read():
    """Evict L2 by READING a 256 MB buffer (clean lines: a write-flush would leave ~126 MB of dirty
    lines whose write-back the timed kernel then pays for)."""
    global _FLUSH
    if _FLUSH is None:
        _FLUSH = torch.ones(64 << 20, dtype=torch.float32, device="cuda")
    _FLUSH.sum()


def bench_cublas(M, N, K, reps=20):
    """cuBLAS (torch.mm, bf16 out) on the same shape: the library reference for the plain GEMM."""
    A = torch.randn((M, K), device="cuda").to(torch.bfloat16)
    W = (torch.randn((N, K), device="cuda") * K ** -0.5).to(torch.bfloat16)
    for _ in range(3):
        torch.mm(A, W.t())
    ts = []
    for _ in range(reps):
        flush_read()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        torch.mm(A, W.t())
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    ms = ts[len(ts) // 2]
    return dict(M=M, N=N, K=K, epi="cublas", us=round(ms * 1e3, 1), tflops=round(2.0 * M * N * K / (ms * 1e-3) / 1e12, 1))


def bench(M, N, K, epi, reps=20):
    A = torch.randn((M, K), device="cuda").to(torch.bfloat16)
    W = (torch.randn((N, K), device="cuda") * K ** -0.5).to(torch.bfloat16)
    if epi == 3:
        out = torch.empty((M,), dtype=torch.int32, device="cuda")
    elif epi == 1:
        out = torch.zeros((M, N), device="cuda")
    elif epi == 2:
        out = torch.empty((M, N // 2), dtype=torch.bfloat16, device="cuda")
    else:
        out = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):
        gllm.op_gemm(A.data_ptr(), W.data_ptr(), M, N, K, epi, out.data_ptr(), 0, s)
    ts = []
    for _ in range(reps):
        flush_read()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        gllm.op_gemm(A.data_ptr(), W.data_ptr(), M, N, K, epi, out.data_ptr(), 0, s)
        e1.record()
        torch.cuda.synchronize()
        ts.append(e0.elapsed_time(e1))
    ts.sort()
    ms = ts[len(ts) // 2]
    tf = 2.0 * M * N * K / (ms * 1e-3) / 1e12
    gbs = (N * K * 2 + M * K * 2) / (ms * 1e-3) / 1e9
    return dict(M=M, N=N, K=K, epi=epi, us=round(ms * 1e3, 1), tflops=round(tf, 1), weight_gbs=round(gbs, 1))


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--shapes", default="C1,C4,sq")
    ap.add_argument("--variants", default="0", help="comma list: 0 auto, 1 one-CTA, 2 CTA pair")
    ap.add_argument("--cublas", action="store_true", help="also time torch.mm (cuBLAS) per shape")
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--det", action="store_true", help="gllm_op_set_deterministic: whole tiles / cluster split-K only")
    a = ap.parse_args()
    gllm.op_set_deterministic(a.det)
    if a.cublas:
        for key in a.shapes.split(","):
            for shp in SHAPES[key]:
                print(json.dumps({"variant": "cublas", "set": key, **bench_cublas(*shp[:3])}), flush=True)
    for v in [int(x) for x in a.variants.split(",")]:
        gllm.op_set_gemm_variant(v)
        for key in a.shapes.split(","):
            for shp in SHAPES[key]:
                print(json.dumps({"variant": v, "det": a.det, "set": key, **bench(*shp, reps=a.reps)}), flush=True)
    gllm.op_set_gemm_variant(0)
