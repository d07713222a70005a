O=gpurun_out/t19; mkdir -p $O
for cfg in "C2 --pp 4 --tick 410" "C3 --pp 8 --tick 410" "C4 --pp 8 --tick 410" "C1 --tick 403" "C1 --tick 412"; do
for dv in 1 2 4; do for mp in 4 8 16; do
  echo "$cfg div=$dv minp=$mp $(GLLM_DEC_DIV=$dv GLLM_DEC_MINPAGES=$mp timeout 300 python tools/attn_bench.py --config $cfg 2>&1 | tail -1 | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"])')" >> $O/dec_ab.txt
done; done; done
cat $O/dec_ab.txt
