O=gpurun_out/t16; mkdir -p $O
timeout 300 python tools/gemm_bench.py --shapes C2,C3,C1 > $O/gb.jsonl 2>&1
timeout 300 python tools/gemm_bench.py --shapes C2,C3,C1 --det >> $O/gb.jsonl 2>&1
timeout 300 python tools/gemm_bench.py --shapes C2,C3 --variants 1 >> $O/gb.jsonl 2>&1
cat $O/gb.jsonl
