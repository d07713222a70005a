#!/bin/bash
# prefill: separate K / V slot release; fused peer hand-off (2 processes on one GPU) (under gpurun)
OUT=${OUT:-gpurun_out/s3h}
mkdir -p $OUT
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "c0 or gqa or long or c3 or other_shapes" > $OUT/pytest_parity.log 2>&1; tail -2 $OUT/pytest_parity.log
timeout 900 python -m pytest tests/test_gpu_peer.py -x -q > $OUT/pytest_peer.log 2>&1; tail -15 $OUT/pytest_peer.log
for t in 403 412; do echo "C1 tick $t $(timeout 300 python tools/attn_bench.py --tick $t)" >> $OUT/attn.txt; done
echo "C3 tick 500 $(timeout 300 python tools/attn_bench.py --config C3 --tick 500)" >> $OUT/attn.txt
cat $OUT/attn.txt
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
