for v in "base" "GLLM_SIDE_PRIO=1" "GLLM_SIDE_PRIO=1 GLLM_PREFILL_PAD_KB=114" "GLLM_PREFILL_PAD_KB=114"; do
  envs=""; [ "$v" != "base" ] && envs="$v"
  for c in C1:403 C1:412 C3:500 C4:500; do
    echo "$v $c $(env $envs timeout 300 python tools/attn_bench.py --config ${c%%:*} --tick ${c##*:} | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us"], d["prefill"]["us"], d["mixed"]["us"])')"
  done
done
