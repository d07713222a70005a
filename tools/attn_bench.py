"""Isolated attention micro-benchmark through the C ABI: the C1 stream is fast-forwarded on the
host to tick `--tick` (PP=1), and that tick's batch is split into its decode rows and its
prefill chunks; each part runs through a one-layer stage (KV pages hold O4 values) with the
stage's per-category CUDA-event timing.  Prints achieved HBM GB/s (decode) and TFLOP/s (prefill).

    python tools/attn_bench.py --tick 403 --reps 20
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_00090d00l25_b200 import gllm  # noqa: E402
from workloads.configs import MODELS, SCHED  # noqa: E402
from workloads.streams import make_stream  # noqa: E402


def subset(a, seqs):
    """desc dict restricted to sequences `seqs` (prefill chunks first, as in the ABI layout)."""
    cu, kv, bt = a["cu_q"], a["kv_len"], a["block_table"]
    NP = a["num_prefill_seqs"]
    ids, pos, ncu, nkv, rows, samp = [], [], [0], [], [], []
    for i in seqs:
        t0, t1 = int(cu[i]), int(cu[i + 1])
        ids += list(a["token_ids"][t0:t1])
        pos += list(a["positions"][t0:t1])
        ncu.append(ncu[-1] + t1 - t0)
        nkv.append(int(kv[i]))
        rows.append(bt[i])
    T = ncu[-1]
    return dict(tick=0, num_tokens=T, num_seqs=len(seqs), num_prefill_seqs=sum(1 for i in seqs if i < NP),
                token_ids=np.array(ids, np.int32), positions=np.array(pos, np.int32),
                slot_mapping=np.zeros(T, np.int32), cu_q=np.array(ncu, np.int32), kv_len=np.array(nkv, np.int32),
                block_table=np.stack(rows).astype(np.int32), sample_idx=np.zeros(0, np.int32),
                seq_req_ids=np.zeros(len(seqs), np.int64))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C1")
    ap.add_argument("--tick", type=int, default=403)
    ap.add_argument("--reps", type=int, default=20)
    ap.add_argument("--pp", type=int, default=1, help="scheduler pipeline depth (the stage micro-batches of PP > 1)")
    a = ap.parse_args()
    m = MODELS[a.config].with_layers(2)
    sp = SCHED[a.config].with_(pp_depth=a.pp, num_blocks=60000 if a.config == "C1" else SCHED[a.config].num_blocks)
    s = gllm.Sched(sp)
    s.add_stream(make_stream(a.config, m.vocab))
    for _ in range(a.tick):
        s.build_batch()
    full = s.build_batch().to_numpy()
    NP, S = full["num_prefill_seqs"], full["num_seqs"]
    st = gllm.Stage(m, 1, 2, sp.num_blocks, sp.maxp + sp.max_seqs + 64, sp.max_seqs)
    # non-zero cache contents for the batch's pages (O4 warm-KV values; the timing does not depend on them)
    st.fill_warm_kv(np.arange(S), full["kv_len"], full["block_table"])
    x = torch.randn((sp.maxp + sp.max_seqs + 64, m.hidden), device="cuda")
    out = {}
    kvb = 2 * m.n_kv_heads * m.head_dim * 2
    for name, seqs in (("decode", list(range(NP, S))), ("prefill", list(range(NP))), ("mixed", list(range(S)))):
        if not seqs:
            continue
        d, keep = gllm.desc_from_arrays(subset(full, seqs))
        for _ in range(3):
            st.forward(d, x.data_ptr(), x.data_ptr(), 0, 0)
        st.sync()
        st.set_profiling(True)
        st.last_timing()
        for _ in range(a.reps):
            st.forward(d, x.data_ptr(), x.data_ptr(), 0, 0)
        tm = st.last_timing()
        st.set_profiling(False)
        if name == "mixed":
            # the whole batch's attention phase (prefill || decode), timed on the main stream
            span = tm["attention_span"]
            out[name] = {"us": round(span / a.reps * 1e3, 1),
                         "serial_us": round((out.get("decode", {}).get("us", 0) + out.get("prefill", {}).get("us", 0)), 1)}
            continue
        ms = tm[name + "_attn"] / a.reps
        kvl, cu = keep["kv_len"], keep["cu_q"]
        if name == "decode":
            nbytes = float(kvl.sum()) * kvb + len(seqs) * m.q_dim * 4
            out[name] = {"rows": len(seqs), "mean_ctx": round(float(kvl.mean()), 1), "us": round(ms * 1e3, 1),
                         "GBs": round(nbytes / (ms * 1e-3) / 1e9, 1)}
        else:
            pairs = sum(int(cu[i + 1] - cu[i]) * (int(kvl[i]) - int(cu[i + 1] - cu[i])) +
                        int(cu[i + 1] - cu[i]) * (int(cu[i + 1] - cu[i]) + 1) // 2 for i in range(len(seqs)))
            fl = 4.0 * m.n_heads * m.head_dim * pairs
            out[name] = {"chunks": [int(cu[i + 1] - cu[i]) for i in range(len(seqs))], "us": round(ms * 1e3, 1),
                         "TFLOPs": round(fl / (ms * 1e-3) / 1e12, 1)}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
