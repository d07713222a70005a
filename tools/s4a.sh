#!/bin/bash
# re-entry validation pass at HEAD (under gpurun): -m gpu suite, smoke, C1 bench line
OUT=${OUT:-gpurun_out/s4a}
mkdir -p $OUT
timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; tail -3 $OUT/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.log 2>&1; tail -2 $OUT/smoke.log
timeout 900 python bench.py > $OUT/bench_C1.json 2> $OUT/bench_C1.err
tail -c 400 $OUT/bench_C1.json
