#!/bin/bash
# A/B of environment switches on the C1 bench line (run under gpurun):
#   AB="base GLLM_GEMM_CG2=1" bash tools/ab_bench.sh
OUT=${OUT:-gpurun_out/ab_bench}
mkdir -p $OUT
for rep in ${REPS:-1}; do
for v in ${AB:-base}; do
  envs=""; [ "$v" != "base" ] && envs="${v//,/ }"
  env $envs timeout 900 python bench.py --config ${CONFIG:-C1} ${EXTRA} --steps ${STEPS:-10} --warmup 5 --no-cpu-baseline > $OUT/$v.json 2> $OUT/$v.err
  python - "$v" "$OUT/$v.json" <<'PY'
import json, sys
try:
    d = json.loads(open(sys.argv[2]).read().strip().splitlines()[-1])
    print(sys.argv[1], d["value"], d["ms_per_step"], d["clocks"]["sm_mhz"],
          {n: (v["frac"], v["ms"]) for n, v in d["kernels"].items()})
except Exception as e:
    print(sys.argv[1], "FAILED", e)
PY
done
done
