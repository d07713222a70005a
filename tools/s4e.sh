#!/bin/bash
# pipeline model at the PDL build (under gpurun): Token Throttling vs Sarathi-Serve on measured stage times
OUT=${OUT:-gpurun_out/s4e}
mkdir -p $OUT
timeout 400 python tools/pipeline_model.py --config C4 --pp 8 --stage 7 --ticks 160 >> $OUT/pipeline_model.jsonl 2> $OUT/c4.err
timeout 400 python tools/pipeline_model.py --config C2 --pp 4 --stage 3 --ticks 160 --preroll 800 >> $OUT/pipeline_model.jsonl 2> $OUT/c2.err
timeout 400 python tools/pipeline_model.py --config C3 --pp 8 --stage 7 --ticks 160 >> $OUT/pipeline_model.jsonl 2> $OUT/c3.err
cat $OUT/pipeline_model.jsonl | cut -c 1-400
