#!/bin/bash
# PDL A/B (under gpurun): -m gpu suite with GLLM_PDL=1, then interleaved bench lines PDL off/on
OUT=${OUT:-gpurun_out/s4b}
mkdir -p $OUT
GLLM_PDL=1 timeout 1200 python -m pytest tests -m gpu -x -q > $OUT/pytest_gpu_pdl.log 2>&1; tail -3 $OUT/pytest_gpu_pdl.log
GLLM_PDL=1 timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke_pdl.log 2>&1; tail -1 $OUT/smoke_pdl.log
for rep in 1 2; do
  for p in 0 1; do
    GLLM_PDL=$p timeout 600 python bench.py --steps 10 --warmup 5 --no-cpu-baseline > $OUT/C1_pdl${p}_$rep.json 2> $OUT/C1_pdl${p}_$rep.err
    GLLM_PDL=$p timeout 600 python bench.py --config C4 --pp 8 --stage 7 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/C4_pdl${p}_$rep.json 2> $OUT/C4_pdl${p}_$rep.err
    GLLM_PDL=$p timeout 600 python bench.py --config C2 --pp 4 --stage 3 --steps 10 --warmup 5 --no-cpu-baseline > $OUT/C2_pdl${p}_$rep.json 2> $OUT/C2_pdl${p}_$rep.err
  done
done
for f in $OUT/C*_pdl*.json; do echo "$f $(python -c "import json,sys; d=json.loads(open('$f').read().strip().splitlines()[-1]); print(d['value'], d['e2e']['value'], d['clocks']['sm_mhz'])" 2>&1 | tail -1)"; done
