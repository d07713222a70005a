O=gpurun_out/t3; mkdir -p $O
for s in "128 57344 8192 2" "128 10240 8192 0" "2094 28672 4096 2"; do
  n=$(echo $s | tr ' ' '_')
  timeout 300 ncu --set full --import-source on --clock-control none -k regex:gemm_tc_kernel -s 2 -c 1 -o $O/g_$n -f python tools/gemm_one.py $s > $O/ncu_$n.log 2>&1
done
ls -la $O
