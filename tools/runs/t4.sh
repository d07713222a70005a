O=gpurun_out/t4; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -3 $O/pytest_gemm.log
timeout 300 python tools/gemm_bench.py --shapes C4 > $O/gemm_bench.jsonl 2>&1; cat $O/gemm_bench.jsonl
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_determinism.py -x -q > $O/pytest_parity.log 2>&1; tail -3 $O/pytest_parity.log
timeout 600 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $O/bench_C4.json 2> $O/bench_C4.err
