O=gpurun_out/v1; mkdir -p $O
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv > $O/gpu.txt 2>&1
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1
timeout 900 python bench.py --steps 20 --warmup 5 > $O/bench_C1.json 2> $O/bench_C1.err
for c in "C2 --pp 4 --stage 3" "C3 --pp 8 --stage 7" "C4 --pp 8 --stage 7"; do
  n=${c%% *}
  timeout 900 python bench.py --config $c --steps 10 --warmup 5 --no-cpu-baseline > $O/bench_$n.json 2> $O/bench_$n.err
done
tail -3 $O/pytest.log
