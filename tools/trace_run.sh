#!/bin/bash
# GEMM phase traces + isolated GEMM timings (+ cuBLAS) + prefill trace (measurement build).
O=${OUT:-gpurun_out/t1}; mkdir -p $O
export GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so
for s in "128 10240 8192 0" "128 8192 8192 1" "128 8192 28672 1" "128 57344 8192 2" "2094 4096 4096 1" "2094 6144 4096 0" "2094 28672 4096 2" "625 7168 5120 0" "625 5120 5120 1" "900 5120 5120 1"; do
  echo "# $s" >> $O/gemm_trace.jsonl
  timeout 120 python tools/gemm_trace.py $s 2>&1 | tail -2 >> $O/gemm_trace.jsonl
done
timeout 300 python tools/prefill_trace.py --config C3 --tick 500 > $O/prefill_trace.txt 2>&1
timeout 300 python tools/prefill_trace.py --config C1 --tick 403 >> $O/prefill_trace.txt 2>&1
unset GLLM_LIB
timeout 600 python tools/gemm_bench.py --shapes C4,C1,C2,C3 --cublas > $O/gemm_bench.jsonl 2>&1
