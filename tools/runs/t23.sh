O=gpurun_out/t23; mkdir -p $O
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
timeout 300 python tools/gemm_bench.py --shapes C1,C4,C2,C3 > $O/gb.jsonl 2>&1; cat $O/gb.jsonl
for s in "2094 4096 4096 1" "2094 6144 4096 0"; do GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 120 python tools/gemm_trace.py $s 2>&1 | tail -1 >> $O/trace.jsonl; done
cut -c1-500 $O/trace.jsonl
