#!/bin/bash
# prefill softmax: warp-uniform masking + FFMA2/FADD2; GEMM epilogue L2 prefetch (under gpurun)
OUT=${OUT:-gpurun_out/s3g}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c0 or gqa or long or c3 or other_shapes" > $OUT/pytest_parity.log 2>&1; tail -2 $OUT/pytest_parity.log
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q -k "residual or rope or store" > $OUT/pytest_gemm.log 2>&1; tail -2 $OUT/pytest_gemm.log
for t in 403 412; do echo "C1 tick $t $(timeout 300 python tools/attn_bench.py --tick $t)" >> $OUT/attn.txt; done
echo "C3 tick 500 $(timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
cat $OUT/attn.txt
timeout 600 python tools/gemm_bench.py --shapes C1,C2,C3 --variants 0 > $OUT/gemm.txt 2>&1; cat $OUT/gemm.txt
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C2.json 2> $OUT/bench_C2.err
timeout 900 python bench.py --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C1.json 2> $OUT/bench_C1.err
