#!/bin/bash
# stream-K fixup (no memset / finish pass) + GEMM schedule data for the C2/C3/C4 stage shapes (under gpurun)
OUT=${OUT:-gpurun_out/s3d}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_gemm.py -x -q > $OUT/pytest_gemm.log 2>&1; tail -3 $OUT/pytest_gemm.log
timeout 1200 python -m pytest tests/test_gpu_parity.py -x -q > $OUT/pytest_parity.log 2>&1; tail -3 $OUT/pytest_parity.log
timeout 600 python tools/gemm_bench.py --shapes C2,C3,C4 --variants 0,1,2 > $OUT/gemm.txt 2>&1
GLLM_GEMM_NO_SK=1 timeout 600 python tools/gemm_bench.py --shapes C2,C3,C4 --variants 0,1 | sed 's/"variant"/"nosk": 1, "variant"/' >> $OUT/gemm.txt 2>&1
cat $OUT/gemm.txt
OUT=$OUT/ab4 CONFIG=C4 EXTRA="--pp 8 --stage 7" AB="base" bash tools/ab_bench.sh
OUT=$OUT/ab2 CONFIG=C2 EXTRA="--pp 4 --stage 3" AB="base GLLM_GEMM_NO_SK=1" bash tools/ab_bench.sh
