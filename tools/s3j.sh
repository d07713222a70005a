#!/bin/bash
# prefill timing probes; pipelined residual epilogue (under gpurun)
OUT=${OUT:-gpurun_out/s3j}
mkdir -p $OUT
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q -k "residual" > $OUT/pytest_gemm.log 2>&1; tail -2 $OUT/pytest_gemm.log
for pr in 0 2 3; do
  echo "PROBE=$pr C3 $(GLLM_PREFILL_PROBE=$pr timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
  echo "PROBE=$pr C1 $(GLLM_PREFILL_PROBE=$pr timeout 300 python tools/attn_bench.py --tick 412)" >> $OUT/attn.txt
done
cat $OUT/attn.txt
timeout 600 python tools/gemm_bench.py --shapes C1,C2,C3,C3s --variants 0 > $OUT/gemm.txt 2>&1; cat $OUT/gemm.txt
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C1.json 2> $OUT/bench_C1.err
timeout 900 python tools/pipeline_model.py --config C4 --pp 8 --stage 7 --ticks 160 --policies 0,1 > $OUT/pm_C4.txt 2>&1; tail -1 $OUT/pm_C4.txt
