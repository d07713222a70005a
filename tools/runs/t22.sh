O=gpurun_out/t22; mkdir -p $O
timeout 300 python tools/gemm_bench.py --shapes C1,C4,C2,C3 > $O/gb.jsonl 2>&1; grep '"epi": 2' $O/gb.jsonl
for s in "128 57344 8192 2" "2094 28672 4096 2"; do GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 120 python tools/gemm_trace.py $s 2>&1 | tail -1 >> $O/trace.jsonl; done
cut -c1-400 $O/trace.jsonl
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
