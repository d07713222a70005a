O=gpurun_out/t5; mkdir -p $O
for cl in 1 2 4; do echo "cl=$cl" >> $O/gemm_bench.jsonl; GLLM_SMALLT_CL=$cl timeout 300 python tools/gemm_bench.py --shapes C4 >> $O/gemm_bench.jsonl 2>&1; done
cat $O/gemm_bench.jsonl
