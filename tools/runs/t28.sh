O=gpurun_out/t28; mkdir -p $O
timeout 120 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 600 python -m pytest tests/test_gpu_gemm.py -x -q > $O/pytest_gemm.log 2>&1; tail -2 $O/pytest_gemm.log
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_determinism.py -x -q > $O/pytest_parity.log 2>&1; tail -2 $O/pytest_parity.log
for c in "C3 --pp 8 --stage 7" "C4 --pp 8 --stage 7" "C2 --pp 4 --stage 3"; do
  n=${c%% *}
  timeout 600 python bench.py --config $c --steps 10 --warmup 5 --no-cpu-baseline > $O/bench_$n.json 2> $O/bench_$n.err
  python -c "import json; d=json.loads(open('$O/bench_$n.json').read().strip().splitlines()[-1]); print('$n', d['value'], d['ms_per_step'], d['clocks']['sm_mhz'], {k:(v['frac'],round(v['ms'],2)) for k,v in d['kernels'].items()})"
done
