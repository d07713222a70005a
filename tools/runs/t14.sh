O=gpurun_out/t14; mkdir -p $O
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,sm__cycles_active.avg --clock-control none --csv --log-file $O/c3_launches.csv python bench.py --config C3 --pp 8 --stage 7 --steps 2 --warmup 3 --no-cpu-baseline > $O/c3.log 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum --clock-control none --csv --log-file $O/c4_launches.csv python bench.py --config C4 --pp 8 --stage 7 --steps 2 --warmup 3 --no-cpu-baseline > $O/c4.log 2>&1
ls -la $O
