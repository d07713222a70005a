O=gpurun_out/t30; mkdir -p $O
for v in 0 1 0 1; do
  if [ $v = 1 ]; then export GLLM_LM_CG2=1; else unset GLLM_LM_CG2; fi
  timeout 600 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $O/b$v.json 2>/dev/null
  python -c "import json; d=json.loads(open('$O/b$v.json').read().strip().splitlines()[-1]); print('$v', d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['kernels']['lm_head'])" >> $O/res.txt
done
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/c1_0.json 2>/dev/null; GLLM_LM_CG2=1 timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/c1_1.json 2>/dev/null
for v in 0 1; do python -c "import json; d=json.loads(open('$O/c1_$v.json').read().strip().splitlines()[-1]); print('C1 $v', d['value'], d['ms_per_step'], d['kernels']['lm_head'])" >> $O/res.txt; done
cat $O/res.txt
