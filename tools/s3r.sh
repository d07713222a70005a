#!/bin/bash
# final bench lines with the event-free timed pass (under gpurun)
OUT=${OUT:-gpurun_out/s3r}
mkdir -p $OUT
timeout 900 python bench.py > $OUT/bench_C1.json 2> $OUT/bench_C1.err
timeout 900 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C2.json 2> $OUT/bench_C2.err
timeout 900 python bench.py --config C3 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C3.json 2> $OUT/bench_C3.err
timeout 900 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/bench_C4.json 2> $OUT/bench_C4.err
timeout 900 python bench.py --impl reference --steps 2 --warmup 3 > $OUT/bench_ref.json 2> $OUT/bench_ref.err
tail -c 600 $OUT/bench_C1.json
