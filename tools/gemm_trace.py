"""Per-CTA phase timeline of one stage GEMM (measurement build, build.py --variant=trace).

    python -m paper_conf_sc_00090d00l25_b200.build --variant=trace
    GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so python tools/gemm_trace.py 128 8192 1024 0

Prints, over the CTAs, the mean / max time (us, from the first CTA's entry) of each stamp:
entry, setup done, last MMA issued, accumulator ready, partial tile stored / first tile drained,
cluster sync, reduce + epilogue done, exit.
"""
import ctypes as C
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_00090d00l25_b200 import gllm  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from gemm_bench import flush_read  # noqa: E402

GM_TR = 48
NAMES = ["entry", "setup", "mma_issued", "acc_ready", "drained", "cl_sync", "reduced", "exit", None, "first_stage"]


def main():
    M, N, K, epi = (int(x) for x in sys.argv[1:5])
    A = torch.randn((M, K), device="cuda").to(torch.bfloat16)
    W = (torch.randn((N, K), device="cuda") * K ** -0.5).to(torch.bfloat16)
    out = (torch.zeros((M, N), device="cuda") if epi == 1 else
           torch.empty((M, N // 2 if epi == 2 else N), dtype=torch.bfloat16, device="cuda"))
    s = torch.cuda.current_stream().cuda_stream
    for _ in range(3):
        gllm.op_gemm(A.data_ptr(), W.data_ptr(), M, N, K, epi, out.data_ptr(), 0, s)
    buf = torch.zeros(GM_TR * 4096, dtype=torch.int64, device="cuda")
    L = gllm.lib()
    L.gllm_gemm_trace_arm.argtypes = [C.c_void_p]
    res = []
    for rep in range(5):
        buf.zero_()
        flush_read()
        L.gllm_gemm_trace_arm(buf.data_ptr())
        gllm.op_gemm(A.data_ptr(), W.data_ptr(), M, N, K, epi, out.data_ptr(), 0, s)
        torch.cuda.synchronize()
        L.gllm_gemm_trace_arm(None)
        r = buf.cpu().numpy().reshape(-1, GM_TR)
        r = r[r[:, 7] > 0]
        t0 = r[:, 0].min()
        row = {"rep": rep, "ctas": len(r), "span_us": round((r[:, 7].max() - t0) / 1e3, 2)}
        for i, nm in enumerate(NAMES):
            if nm is None:
                continue
            v = r[:, i]
            v = v[v > 0]
            if len(v):
                row[nm] = [round((v.mean() - t0) / 1e3, 2), round((v.max() - t0) / 1e3, 2)]
        # per tile j of a CTA: accumulator ready / drained (mean, max over CTAs that ran tile j)
        tiles = []
        for j in range(16):
            a, d = r[:, 10 + 2 * j], r[:, 11 + 2 * j]
            if (a > 0).sum() == 0:
                break
            tiles.append([int((a > 0).sum()), round((a[a > 0].mean() - t0) / 1e3, 2), round((d[d > 0].mean() - t0) / 1e3, 2),
                          round((d[d > 0].max() - t0) / 1e3, 2)])
        row["tiles"] = tiles
        res.append(row)
        print(json.dumps(row), flush=True)


if __name__ == "__main__":
    main()
