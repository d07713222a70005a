O=gpurun_out/t9; mkdir -p $O
timeout 600 ncu --set full --import-source on --clock-control none -k regex:prefill_attn_ws -s 3 -c 1 -o $O/pf_c3 -f python tools/attn_bench.py --config C3 --tick 500 --reps 3 > $O/ncu_pf.log 2>&1
tail -3 $O/ncu_pf.log
