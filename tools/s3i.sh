#!/bin/bash
# round-end evidence: full GPU suite, smoke, C1 bench line (+cpu baseline), C2-C4 stage lines, ncu (under gpurun)
OUT=${OUT:-gpurun_out/s3i}
mkdir -p $OUT
timeout 1500 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C1.json 2> $OUT/bench_C1.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $OUT/bench_ref.json 2> $OUT/bench_ref.err
timeout 900 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C2.json 2> $OUT/bench_C2.err
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C4.json 2> $OUT/bench_C4.err
for t in 403 412; do timeout 300 python tools/attn_bench.py --tick $t >> $OUT/prof_attn_bench.jsonl; done
timeout 300 python tools/attn_bench.py --config C3 --tick 500 >> $OUT/prof_attn_bench.jsonl
OUT=$OUT/prof STEPS=10 bash profiles/profile.sh > $OUT/profile.log 2>&1
timeout 1200 ncu --nvtx --nvtx-include "timed/" --set full --clock-control none --import-source on \
  -k regex:prefill_attn_ws -c 4 -o $OUT/prof/prof_prefill_C3 -f python bench.py --config C3 --pp 8 --stage 7 --steps 1 --warmup 3 --no-cpu-baseline > $OUT/ncu_prefill_C3.log 2>&1
timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum --clock-control none \
  --csv --log-file $OUT/launches_C4.csv python bench.py --config C4 --pp 8 --stage 7 --steps 2 --warmup 3 --no-cpu-baseline > $OUT/ncu_c4.json 2>&1
ls $OUT $OUT/prof
