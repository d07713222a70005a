O=gpurun_out/t13; mkdir -p $O
for rep in 1 2; do
for lib in head new emu1 emu2 emu4; do
  case $lib in head) export GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_head.so;; new) unset GLLM_LIB;; *) export GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_$lib.so;; esac
  echo "lib=$lib $(timeout 300 python tools/attn_bench.py --config C3 --tick 500 2>&1 | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["prefill"]["us"])') $(timeout 300 python tools/attn_bench.py --tick 412 2>&1 | python -c 'import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print(d["prefill"]["us"])')" >> $O/ab.txt
done; done
cat $O/ab.txt
