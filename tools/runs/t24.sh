O=gpurun_out/t24; mkdir -p $O
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
for lib in head new; do
  if [ $lib = head ]; then export GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_head.so; else unset GLLM_LIB; fi
  echo "lib=$lib" >> $O/attn_ab.jsonl
  timeout 90 python tools/attn_bench.py --config C3 --tick 500 >> $O/attn_ab.jsonl 2>&1
  timeout 90 python tools/attn_bench.py --tick 412 >> $O/attn_ab.jsonl 2>&1
  timeout 90 python tools/attn_bench.py --tick 403 >> $O/attn_ab.jsonl 2>&1
  timeout 90 python tools/attn_bench.py --config C3 --pp 8 --tick 410 >> $O/attn_ab.jsonl 2>&1
done
cat $O/attn_ab.jsonl
GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so timeout 90 python tools/prefill_trace.py --config C3 --tick 500 > $O/prefill_trace.txt 2>&1
cat $O/prefill_trace.txt
