#!/bin/bash
# prefill softmax with pipelined TMEM loads + vectorised stream-K finish pass (under gpurun)
OUT=${OUT:-gpurun_out/s3f}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c0 or gqa or long or c3 or other_shapes" > $OUT/pytest_parity.log 2>&1; tail -2 $OUT/pytest_parity.log
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q -k "store or silu" > $OUT/pytest_gemm.log 2>&1; tail -2 $OUT/pytest_gemm.log
for t in 403 412; do echo "C1 tick $t $(timeout 300 python tools/attn_bench.py --tick $t)" >> $OUT/attn.txt; done
echo "C3 tick 500 $(timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
cat $OUT/attn.txt
timeout 900 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C4.json 2> $OUT/bench_C4.err
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 1200 ncu --nvtx --nvtx-include "timed/" --set full --clock-control none --import-source on \
  -k regex:prefill_attn_ws -c 4 -o $OUT/prof_prefill_C3 -f python bench.py --config C3 --pp 8 --stage 7 --steps 1 --warmup 3 --no-cpu-baseline > $OUT/ncu_prefill_C3.log 2>&1
timeout 1200 ncu --nvtx --nvtx-include "timed/" --set full --clock-control none --import-source on \
  -k regex:gemm_tc -c 8 -o $OUT/prof_gemm_C3 -f python bench.py --config C3 --pp 8 --stage 7 --steps 1 --warmup 3 --no-cpu-baseline > $OUT/ncu_gemm_C3.log 2>&1
ls $OUT
