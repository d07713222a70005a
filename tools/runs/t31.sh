O=gpurun_out/t31; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > $O/pytest_parity.log 2>&1; tail -2 $O/pytest_parity.log
