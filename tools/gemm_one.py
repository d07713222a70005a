"""One stage GEMM through gllm_op_gemm (for ncu captures):  python tools/gemm_one.py M N K epi [reps]"""
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_00090d00l25_b200 import gllm  # noqa: E402

M, N, K, epi = (int(x) for x in sys.argv[1:5])
reps = int(sys.argv[5]) if len(sys.argv) > 5 else 3
A = torch.randn((M, K), device="cuda").to(torch.bfloat16)
W = (torch.randn((N, K), device="cuda") * K ** -0.5).to(torch.bfloat16)
out = (torch.zeros((M, N), device="cuda") if epi == 1 else
       torch.empty((M, N // 2 if epi == 2 else N), dtype=torch.bfloat16, device="cuda"))
for _ in range(reps):
    gllm.op_gemm(A.data_ptr(), W.data_ptr(), M, N, K, epi, out.data_ptr(), 0, torch.cuda.current_stream().cuda_stream)
torch.cuda.synchronize()
print("ok", M, N, K, epi)
