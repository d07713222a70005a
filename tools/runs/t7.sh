O=gpurun_out/t8; mkdir -p $O
for rep in 1 2; do
for lib in head new; do
  if [ $lib = head ]; then export GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_head.so; else unset GLLM_LIB; fi
  echo "lib=$lib" >> $O/attn_ab.jsonl
  timeout 300 python tools/attn_bench.py --config C3 --tick 500 >> $O/attn_ab.jsonl 2>&1
  timeout 300 python tools/attn_bench.py --tick 412 >> $O/attn_ab.jsonl 2>&1
done; done
cat $O/attn_ab.jsonl
