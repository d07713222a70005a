O=gpurun_out/t11; mkdir -p $O
GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 300 python tools/prefill_trace.py --config C3 --tick 500 > $O/prefill_trace.txt 2>&1
GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 300 python tools/prefill_trace.py --config C1 --tick 412 >> $O/prefill_trace.txt 2>&1
cat $O/prefill_trace.txt
