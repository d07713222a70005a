#!/bin/bash
# Round-end evidence at HEAD (run under gpurun from the repo root): smoke, the full -m gpu suite,
# profiles/profile.sh (bench lines C1-C4, isolated attention / GEMMs, ncu launch list + --set full
# captures), and the reference arm (the oracle on the host cores).
O=${OUT:-gpurun_out/final}; mkdir -p $O
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > $O/smoke.log 2>&1; tail -1 $O/smoke.log
timeout 1500 python -m pytest tests -m gpu -x -q > $O/pytest.log 2>&1; tail -2 $O/pytest.log
OUT=$O timeout 2400 bash profiles/profile.sh > $O/profile.log 2>&1
timeout 900 python bench.py --impl reference --steps 3 --warmup 1 > $O/bench_reference.json 2> $O/bench_reference.err
tail -c 600 $O/bench_reference.json
ls $O
