#!/bin/bash
# persistent warp-specialised prefill (under gpurun)
OUT=${OUT:-gpurun_out/s3k}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c0 or gqa or long or c3 or other_shapes" > $OUT/pytest_parity.log 2>&1; tail -2 $OUT/pytest_parity.log
for pr in 0 3; do
  echo "PROBE=$pr C3 $(GLLM_PREFILL_PROBE=$pr timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
  echo "PROBE=$pr C1 412 $(GLLM_PREFILL_PROBE=$pr timeout 300 python tools/attn_bench.py --tick 412)" >> $OUT/attn.txt
done
echo "C1 403 $(timeout 300 python tools/attn_bench.py --tick 403)" >> $OUT/attn.txt
cat $OUT/attn.txt
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C1.json 2> $OUT/bench_C1.err
