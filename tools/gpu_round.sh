#!/bin/bash
# One measurement pass under gpurun: GPU parity tests, isolated attention bench, C1 bench line.
#   OUT=gpurun_out/rX bash tools/gpu_round.sh
OUT=${OUT:-gpurun_out/round}
mkdir -p $OUT
if [ -z "$SKIP_TESTS" ]; then
  timeout 900 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu.log 2>&1; tail -3 $OUT/pytest_gpu.log
fi
for t in ${TICKS:-403 412}; do echo "tick $t $(timeout 300 python tools/attn_bench.py --tick $t)" >> $OUT/attn.txt; done
echo "C3 tick 500 $(timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
timeout 600 python bench.py --steps ${STEPS:-10} --warmup 5 > $OUT/bench.json 2> $OUT/bench.err
cat $OUT/attn.txt; cat $OUT/bench.json
