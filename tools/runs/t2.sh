O=gpurun_out/t2; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -3 $O/pytest_gemm.log
timeout 300 python tools/gemm_bench.py --shapes C1,C2,C3 > $O/gemm_bench.jsonl 2>&1
GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 120 python tools/gemm_trace.py 2094 4096 4096 1 > $O/trace_o.jsonl 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > $O/pytest_parity.log 2>&1; tail -3 $O/pytest_parity.log
timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > $O/bench_C1.json 2> $O/bench_C1.err
