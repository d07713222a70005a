#!/bin/bash
# Reproduces the profiles/ evidence on a B200 (run under gpurun from the repo root):
#   1. bench line of the headline (C1, PP=1) and the emulated C2 / C3 / C4 stages
#   2. launch list of the C1 timed region (ncu, cold and serialised; NVTX range "timed")
#   3. one `ncu --set full` capture of the dominant kernel and of the attention kernels
#   4. isolated attention numbers (tools/attn_bench.py) and small-T GEMMs (tools/gemm_bench.py)
OUT=${OUT:-gpurun_out/profile}
mkdir -p $OUT
STEPS=${STEPS:-20}
timeout 900 python bench.py --steps $STEPS --warmup 5 > $OUT/bench_C1.json 2> $OUT/bench_C1.err
tail -c 1500 $OUT/bench_C1.json
for c in "C2 --pp 4 --stage 3" "C3 --pp 8 --stage 7" "C4 --pp 8 --stage 7"; do
  n=${c%% *}
  timeout 900 python bench.py --config $c --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_$n.json 2> $OUT/bench_$n.err
done
for t in 403 412; do timeout 300 python tools/attn_bench.py --tick $t >> $OUT/attn_bench.jsonl; done
timeout 300 python tools/attn_bench.py --config C3 --tick 500 >> $OUT/attn_bench.jsonl
timeout 300 python tools/gemm_bench.py --shapes C1,C4 > $OUT/gemm_bench.jsonl 2>&1
timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 --preroll 400 --no-cpu-baseline > $OUT/ncu_bench.json 2>&1
for K in ${KERNELS:-gemm_tc_kernel decode_attn_tma_kernel prefill_attn_ws_kernel}; do
  timeout 1200 ncu --nvtx --nvtx-include "timed/" --set full --clock-control none --import-source on \
    -k regex:$K -c ${NCU_COUNT:-4} -o $OUT/prof_$K -f python bench.py --steps 1 --warmup 3 --no-cpu-baseline \
    > $OUT/ncu_$K.log 2>&1
done
ls -la $OUT
