O=gpurun_out/t29; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
