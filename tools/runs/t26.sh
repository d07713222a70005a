O=gpurun_out/t26; mkdir -p $O
for lib in base nostore base nostore; do
  if [ $lib = base ]; then unset GLLM_LIB; else export GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_nostore.so; fi
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $O/b_$lib.json 2> $O/b_$lib.err
  python -c "import json; d=json.loads(open('$O/b_$lib.json').read().strip().splitlines()[-1]); print('$lib', d['ms_per_step'], d['kernels']['qkv_gemm'])" >> $O/res.txt
done
cat $O/res.txt
