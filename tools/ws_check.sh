#!/bin/bash
# warp-specialised prefill: parity, isolated A/B vs v1, C1 bench A/B; C4 stage launch list (under gpurun)
OUT=${OUT:-gpurun_out/ws}
mkdir -p $OUT
GLLM_PREFILL_WS=1 timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c0 or gqa or long or other_shapes" > $OUT/pytest_ws.log 2>&1; tail -3 $OUT/pytest_ws.log
for v in 1 0; do
  for t in 403 412; do echo "WS=$v C1 tick $t $(GLLM_PREFILL_WS=$v timeout 300 python tools/attn_bench.py --tick $t)" >> $OUT/attn.txt; done
  echo "WS=$v C3 tick 500 $(GLLM_PREFILL_WS=$v timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
done
cat $OUT/attn.txt
OUT=$OUT/ab AB="base GLLM_PREFILL_WS=1" bash tools/ab_bench.sh
OUT=$OUT/ab3 CONFIG=C3 EXTRA="--pp 8 --stage 7" AB="base GLLM_PREFILL_WS=1" bash tools/ab_bench.sh
timeout 600 python tools/gemm_bench.py --shapes C4 > $OUT/gemm_c4.txt 2>&1; cat $OUT/gemm_c4.txt
timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file $OUT/launches_c4.csv python bench.py --config C4 --pp 8 --stage 7 --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_c4.json 2>&1
