O=gpurun_out/t18; mkdir -p $O
timeout 300 python tools/gemm_bench.py --shapes C4 > $O/gb.jsonl 2>&1
echo "skc_add" >> $O/gb.jsonl; GLLM_SKC_ADD=1 timeout 300 python tools/gemm_bench.py --shapes C4 >> $O/gb.jsonl 2>&1
cat $O/gb.jsonl
GLLM_SKC_ADD=1 timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q -k "small_t or add or resid" > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
for v in 0 1; do
if [ $v = 1 ]; then export GLLM_SKC_ADD=1; fi
timeout 600 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $O/bench_C4_$v.json 2> $O/bench_C4_$v.err
python -c "import json; d=json.loads(open('$O/bench_C4_$v.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], {k:(v['frac'],round(v['ms'],2)) for k,v in d['kernels'].items()})"
done
