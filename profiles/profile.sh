#!/bin/bash
# Reproduces the profiles/ evidence on a B200 (run under gpurun from the repo root):
#   1. bench line (clocks sampled in the run)                 -> $OUT/bench.json
#   2. launch list of the timed region (cold, serialised)     -> $OUT/launches.csv
#   3. one `ncu --set full` capture per hot kernel family     -> $OUT/prof_<name>.ncu-rep
#   4. isolated attention numbers (tools/attn_bench.py)       -> $OUT/attn_bench.jsonl
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
STEPS=${STEPS:-20}
timeout 900 python bench.py --steps $STEPS --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
tail -c 2000 $OUT/bench.err
for t in 403 412; do timeout 300 python tools/attn_bench.py --tick $t >> $OUT/attn_bench.jsonl; done
timeout 300 python tools/attn_bench.py --config C3 --tick 500 >> $OUT/attn_bench.jsonl
timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_bench.json 2>&1
for K in ${KERNELS:-gemm_tc_kernel decode_attn_tma_kernel prefill_attn_ws_kernel}; do
  timeout 1200 ncu --nvtx --nvtx-include "timed/" --set full --clock-control none --import-source on \
    -k regex:$K -c ${NCU_COUNT:-5} -o $OUT/prof_$K -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline \
    > $OUT/ncu_$K.log 2>&1
done
ls -la $OUT
