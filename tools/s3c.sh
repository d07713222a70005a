#!/bin/bash
# hybrid CTA-pair stream-K tail + ws prefill default + EMU A/B (under gpurun)
OUT=${OUT:-gpurun_out/s3c}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_gemm.py -x -q -k "residual" > $OUT/pytest_gemm.log 2>&1; tail -3 $OUT/pytest_gemm.log
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c3 or c1_stream_long or other_shapes or c0" > $OUT/pytest_parity.log 2>&1; tail -3 $OUT/pytest_parity.log
for v in 0 1; do
  for t in 403 412; do echo "EMU=$v C1 tick $t $(GLLM_PREFILL_EMU=$v timeout 300 python tools/attn_bench.py --tick $t)" >> $OUT/attn.txt; done
  echo "EMU=$v C3 tick 500 $(GLLM_PREFILL_EMU=$v timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
done
cat $OUT/attn.txt
OUT=$OUT/ab3 CONFIG=C3 EXTRA="--pp 8 --stage 7" AB="base GLLM_GEMM_NO_HYBRID=1 GLLM_PREFILL_EMU=1" bash tools/ab_bench.sh
OUT=$OUT/ab1 CONFIG=C1 AB="base GLLM_PREFILL_EMU=1" bash tools/ab_bench.sh
OUT=$OUT/ab2 CONFIG=C2 EXTRA="--pp 4 --stage 3" AB="base" bash tools/ab_bench.sh
OUT=$OUT/ab4 CONFIG=C4 EXTRA="--pp 8 --stage 7" AB="base" bash tools/ab_bench.sh
