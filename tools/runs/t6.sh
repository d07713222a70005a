O=gpurun_out/t6; mkdir -p $O
for t in 403 412; do timeout 300 python tools/attn_bench.py --tick $t >> $O/attn_bench.jsonl 2>&1; done
timeout 300 python tools/attn_bench.py --config C3 --tick 500 >> $O/attn_bench.jsonl 2>&1
cat $O/attn_bench.jsonl
GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 300 python tools/prefill_trace.py --config C3 --tick 500 > $O/prefill_trace.txt 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q > $O/pytest_parity.log 2>&1; tail -3 $O/pytest_parity.log
