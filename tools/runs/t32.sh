O=gpurun_out/t32; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1; tail -2 $O/pytest.log
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_C1.json 2> $O/bench_C1.err
for c in "C2 --pp 4 --stage 3" "C3 --pp 8 --stage 7" "C4 --pp 8 --stage 7"; do
  n=${c%% *}
  timeout 900 python bench.py --config $c --steps 10 --warmup 5 --no-cpu-baseline > $O/bench_$n.json 2> $O/bench_$n.err
done
for n in C1 C2 C3 C4; do python -c "import json; d=json.loads(open('$O/bench_$n.json').read().strip().splitlines()[-1]); print('$n', d['value'], d['e2e']['value'], d['ms_per_step'], d['clocks']['sm_mhz'], d['roofline']['kernel'], d['roofline']['frac'])"; done
