#!/bin/bash
# A/B of measurement builds (libgllm_<variant>.so, built with build(variant=...)) on the isolated
# attention bench:  LIBS="default simpleissue" CASES="C1:403 C3:500" bash tools/ab_lib.sh
for rep in 1 2; do
for lib in ${LIBS:-default}; do
  L=""; [ "$lib" != "default" ] && L="$PWD/paper_conf_sc_00090d00l25_b200/libgllm_$lib.so"
  for c in ${CASES:-C1:403 C1:412 C3:500 C4:500}; do
    echo "$lib ${c} $(GLLM_LIB=$L timeout 300 python tools/attn_bench.py --config ${c%%:*} --tick ${c##*:} | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["decode"]["us"], d["decode"]["GBs"], d["mixed"]["us"])')"
  done
done
done
