#!/bin/bash
# measurement pass: GEMM tests, C1-C4 bench lines, pipeline model (policies 0/1/4), ncu evidence (under gpurun)
OUT=${OUT:-gpurun_out/s3e}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_gemm.py -x -q > $OUT/pytest_gemm.log 2>&1; tail -2 $OUT/pytest_gemm.log
timeout 600 python tools/gemm_bench.py --shapes C2,C3,C4 --variants 0 > $OUT/gemm.txt 2>&1
timeout 900 python bench.py --steps 10 --warmup 5 > $OUT/bench_C1.json 2> $OUT/bench_C1.err
timeout 900 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C2.json 2> $OUT/bench_C2.err
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C4.json 2> $OUT/bench_C4.err
timeout 900 python tools/pipeline_model.py --config C3 --pp 8 --stage 7 --ticks 160 --policies 0,4,1 > $OUT/pm_C3.txt 2>&1
timeout 900 python tools/pipeline_model.py --config C2 --pp 4 --stage 3 --ticks 160 --policies 0,4,1 > $OUT/pm_C2.txt 2>&1
tail -n 4 $OUT/pm_C3.txt $OUT/pm_C2.txt
OUT=$OUT/prof STEPS=10 bash profiles/profile.sh > $OUT/profile.log 2>&1
ls $OUT/prof
