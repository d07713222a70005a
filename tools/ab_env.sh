#!/bin/bash
# A/B of environment switches on the isolated attention bench (run under gpurun):
#   AB="base GLLM_PREFILL_W4=1" CASES="C1:403 C3:500" bash tools/ab_env.sh
for v in ${AB:-base}; do
  envs=""; [ "$v" != "base" ] && envs="${v//,/ }"
  for c in ${CASES:-C1:403 C1:412 C3:500 C4:500}; do
    echo "$v $c $(env $envs timeout 300 python tools/attn_bench.py --config ${c%%:*} --tick ${c##*:} | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us"], d["prefill"]["us"], d["prefill"]["TFLOPs"], d["mixed"]["us"])')"
  done
done
