O=gpurun_out/t27; mkdir -p $O
for r in 1 2 3; do timeout 600 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > $O/c1_rep$r.json 2> $O/c1_rep$r.err; done
for r in 1 2; do timeout 600 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $O/c4_rep$r.json 2>/dev/null; done
timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/c4_launches.csv python bench.py --config C4 --pp 8 --stage 7 --steps 1 --warmup 3 --no-cpu-baseline > $O/c4_ncu.log 2>&1
timeout 1200 ncu --nvtx --nvtx-include "timed/" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file $O/c3_launches.csv python bench.py --config C3 --pp 8 --stage 7 --steps 1 --warmup 3 --no-cpu-baseline > $O/c3_ncu.log 2>&1
ls -la $O
