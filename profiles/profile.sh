#!/bin/bash
# Reproduces the profiles/ evidence on a B200 (run under gpurun from the repo root):
#   1. bench line (clocks sampled in the run)          -> gpurun_out/bench.json
#   2. launch list of the timed region (cold, serial)  -> gpurun_out/launches.csv
#   3. one `ncu --set full` capture of the top kernels  -> gpurun_out/prof_<name>.ncu-rep
set -x
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
STEPS=${STEPS:-20}
timeout 900 python bench.py --steps $STEPS --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
tail -c 3000 $OUT/bench.err
timeout 900 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_bench.json 2>&1
for K in ${KERNELS:-gemm_tc_kernel decode_attn_kernel prefill_attn_kernel}; do
  timeout 900 ncu --nvtx --nvtx-include "timed/" --set full --clock-control none --import-source on \
    -k regex:$K -c ${NCU_COUNT:-4} -o $OUT/prof_$K -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline \
    > $OUT/ncu_$K.log 2>&1
done
ls -la $OUT
