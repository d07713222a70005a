#!/bin/bash
# ws2 prefill (two S buffers per Q tile, 64-key tiles) behind GLLM_PREFILL_WS2=1 (under gpurun)
OUT=${OUT:-gpurun_out/s3m}
mkdir -p $OUT
GLLM_PREFILL_WS2=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c0 or gqa or long or c3 or other_shapes" > $OUT/pytest_parity.log 2>&1; tail -4 $OUT/pytest_parity.log
for v in 1 0; do
  echo "WS2=$v C3 $(GLLM_PREFILL_WS2=$v timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
  echo "WS2=$v C1 412 $(GLLM_PREFILL_WS2=$v timeout 300 python tools/attn_bench.py --tick 412)" >> $OUT/attn.txt
  echo "WS2=$v C1 403 $(GLLM_PREFILL_WS2=$v timeout 300 python tools/attn_bench.py --tick 403)" >> $OUT/attn.txt
done
cat $OUT/attn.txt
