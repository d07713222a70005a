O=gpurun_out/t15; mkdir -p $O
for cfg in "C3 --pp 8 --tick 410" "C2 --pp 4 --tick 410" "C4 --pp 8 --tick 410"; do
for ms in 32 16 8 4; do for mp in 16 32; do
  echo "$cfg cap=$ms minp=$mp $(GLLM_DEC_MAXSPLIT=$ms GLLM_DEC_MINPAGES=$mp timeout 300 python tools/attn_bench.py --config $cfg 2>&1 | tail -1)" >> $O/dec_ab.txt
done; done; done
cat $O/dec_ab.txt
