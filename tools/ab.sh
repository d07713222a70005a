#!/bin/bash
# A/B of environment switches on the C1 bench and the isolated attention bench (run under gpurun).
#   AB="base GLLM_PREFILL_V1=1 GLLM_ATTN_SERIAL=1" bash tools/ab.sh
OUT=${OUT:-gpurun_out}
mkdir -p $OUT
CONFIG=${CONFIG:-C1}
STEPS=${STEPS:-20}
for v in ${AB:-base}; do
  envs=""
  [ "$v" != "base" ] && envs="$v"
  for t in ${TICKS:-403 405 412}; do
    echo "$v tick $t $(env $envs timeout 300 python tools/attn_bench.py --config $CONFIG --tick $t)" >> $OUT/ab_attn.txt
  done
  env $envs timeout 900 python bench.py --config $CONFIG --steps $STEPS --warmup 5 --no-cpu-baseline > $OUT/ab_$v.json 2> $OUT/ab_$v.err
  python - "$v" "$OUT/ab_$v.json" >> $OUT/ab_summary.txt <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1])
    k = d["kernels"]
    print(sys.argv[1], d["value"], d["ms_per_step"], d["e2e"]["value"], d["clocks"]["sm_mhz"],
          {n: (v["frac"], v["ms"]) for n, v in k.items()})
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
cat $OUT/ab_summary.txt $OUT/ab_attn.txt
