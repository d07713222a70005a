O=gpurun_out/t17; mkdir -p $O
timeout 300 python tools/gemm_bench.py --shapes C2 > $O/gb.jsonl 2>&1
for S in 2 3 4; do echo "S=$S" >> $O/gb.jsonl; GLLM_SKC_S=$S timeout 300 python tools/gemm_bench.py --shapes C4 >> $O/gb.jsonl 2>&1; done
cat $O/gb.jsonl
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
timeout 600 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $O/bench_C2.json 2> $O/bench_C2.err
python -c "import json; d=json.loads(open('$O/bench_C2.json').read().strip().splitlines()[-1]); print(d['value'], d['ms_per_step'], {k:(v['frac'],round(v['ms'],2)) for k,v in d['kernels'].items()})"
