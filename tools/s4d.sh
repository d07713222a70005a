#!/bin/bash
# ncu evidence at the PDL build (under gpurun): C1 launch list of the timed region + --set full
# captures of the GEMMs and decode attention, C4 stage launch list
OUT=${OUT:-gpurun_out/s4d}
mkdir -p $OUT
OUT=$OUT STEPS=10 KERNELS="gemm_tc_kernel decode_attn_tma_kernel" NCU_COUNT=5 bash profiles/profile.sh > $OUT/profile.log 2>&1
timeout 900 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file $OUT/launches_C4.csv python bench.py --config C4 --pp 8 --stage 7 --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_c4.json 2>&1
ls -la $OUT
