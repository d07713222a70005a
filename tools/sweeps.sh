#!/bin/bash
# SURVEY §8(f) items 1 and 3 on measured B200 stage times (tools/pipeline_model.py):
#   f1: Token Throttling vs Sarathi-Serve and the §4.5 ablations (w/o WT, w/o UT) on C2 / C3 / C4
#   f3: hyperparameter sensitivity (§4.6, Fig. 16): #T, #MaxP, #MinP, KV_thresh on C2; KV_thresh on C4
OUT=${OUT:-gpurun_out/sweeps}; mkdir -p $OUT
T=${TICKS:-160}
run() { timeout 900 python tools/pipeline_model.py "$@" --ticks $T 2>&1 | tail -1 >> $OUT/pipeline_model.jsonl; }
run --config C2 --pp 4 --stage 3 --policies 0,1,2,3
run --config C3 --pp 8 --stage 7 --policies 0,1,2,3
run --config C4 --pp 8 --stage 7 --policies 0,1,2,3
run --config C2 --pp 4 --stage 3 --sweep iterp=1,2,4,8,16
run --config C2 --pp 4 --stage 3 --sweep maxp=512,1024,2048
run --config C2 --pp 4 --stage 3 --sweep minp=16,32,64
run --config C2 --pp 4 --stage 3 --sweep kvthresh_num=0,1,2
run --config C4 --pp 8 --stage 7 --sweep kvthresh_num=0,1,2
wc -l $OUT/pipeline_model.jsonl
