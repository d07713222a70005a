#!/bin/bash
# r2 A/B of the decode kernel's ring depth / warps (GLLM_DECODE_CFG) and split policy (GLLM_DECODE_SPLIT)
OUT=${OUT:-gpurun_out/r2f}; mkdir -p $OUT
for cfg in 0 1 2; do for sp in 0 1; do
  export GLLM_DECODE_CFG=$cfg GLLM_DECODE_SPLIT=$sp
  echo "cfg=$cfg split=$sp C1 $(timeout 300 python tools/attn_bench.py --tick 403)" >> $OUT/attn.txt
  echo "cfg=$cfg split=$sp C3 $(timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
  for c in C3 C4; do
    timeout 600 python bench.py --config $c --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_${c}_$cfg$sp.json 2>&1
    python -c "import json,sys;d=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]);k=d['kernels']['decode_attn'];print(sys.argv[1],d['value'],k['frac'],k['ms'])" $OUT/bench_${c}_$cfg$sp.json >> $OUT/bench.txt
  done
done; done
cat $OUT/attn.txt $OUT/bench.txt
for cfg in 1 2; do GLLM_DECODE_CFG=$cfg timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k "long_context or warm or c1_stream or c0" 2>&1 | tail -2; done
