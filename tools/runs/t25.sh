O=gpurun_out/t25; mkdir -p $O
timeout 300 python tools/gemm_bench.py --shapes lm > $O/gb.jsonl 2>&1
echo lm_cg2 >> $O/gb.jsonl; GLLM_LM_CG2=1 timeout 300 python tools/gemm_bench.py --shapes lm >> $O/gb.jsonl 2>&1
cat $O/gb.jsonl
GLLM_LM_CG2=1 timeout 300 python -m pytest tests/test_gpu_gemm.py -x -q -k argmax > $O/pytest.log 2>&1; tail -2 $O/pytest.log
