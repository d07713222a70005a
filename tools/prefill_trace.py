"""Per-CTA timeline of the prefill attention kernel (measurement build, build.py --variant=trace):
runs one layer's prefill attention of a config's tick, and reports SM occupancy over the kernel's
span, the MMA issuer's wait cycles by cause (Q / K / V tiles, P from the softmax), and the tail.

    python -m paper_conf_sc_00090d00l25_b200.build --variant=trace
    GLLM_LIB=$PWD/paper_conf_sc_00090d00l25_b200/libgllm_trace.so python tools/prefill_trace.py --config C3 --tick 500
"""
import argparse
import ctypes as C
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_00090d00l25_b200 import gllm  # noqa: E402
from workloads.configs import MODELS, SCHED  # noqa: E402
from workloads.streams import make_stream  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from attn_bench import subset  # noqa: E402

PF_TR = 20


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C3")
    ap.add_argument("--tick", type=int, default=500)
    a = ap.parse_args()
    m = MODELS[a.config].with_layers(2)
    sp = SCHED[a.config].with_(pp_depth=1, num_blocks=60000 if a.config == "C1" else SCHED[a.config].num_blocks)
    s = gllm.Sched(sp)
    s.add_stream(make_stream(a.config, m.vocab))
    for _ in range(a.tick):
        s.build_batch()
    full = s.build_batch().to_numpy()
    NP = full["num_prefill_seqs"]
    st = gllm.Stage(m, 1, 2, sp.num_blocks, sp.maxp + sp.max_seqs + 64, sp.max_seqs)
    st.fill_warm_kv(np.arange(full["num_seqs"]), full["kv_len"], full["block_table"])
    x = torch.randn((sp.maxp + sp.max_seqs + 64, m.hidden), device="cuda")
    d, keep = gllm.desc_from_arrays(subset(full, list(range(NP))))
    for _ in range(3):
        st.forward(d, x.data_ptr(), x.data_ptr(), 0, 0)
    st.sync()
    buf = torch.zeros(PF_TR * (1 << 18), dtype=torch.int64, device="cuda")
    L = gllm.lib()
    L.gllm_prefill_trace_arm.argtypes = [C.c_void_p]
    L.gllm_prefill_trace_arm(buf.data_ptr())
    st.forward(d, x.data_ptr(), x.data_ptr(), 0, 0)
    st.sync()
    L.gllm_prefill_trace_arm(None)
    rec = buf.cpu().numpy().astype(np.int64)
    n = int((rec.reshape(-1, PF_TR)[:, 2] > 0).sum())
    r = rec[: n * PF_TR].reshape(n, PF_TR)
    t0 = r[:, 0].min()
    start, mma_end, end = (r[:, 0] - t0) / 1e3, (r[:, 1] - t0) / 1e3, (r[:, 2] - t0) / 1e3
    span = end.max()
    sms = np.unique(r[:, 3])
    busy = np.zeros(len(sms))
    for i, smid in enumerate(sms):
        sel = r[:, 3] == smid
        busy[i] = (end[sel] - start[sel]).sum()
    waits = r[:, 4:8].sum(0)
    dur_cyc = None
    out = {"ctas": n, "sms_used": int(len(sms)), "span_us": round(float(span), 1),
           "sm_busy_frac": round(float(busy.sum() / (len(sms) * span)), 3),
           "cta_us_mean": round(float((end - start).mean()), 2), "cta_us_max": round(float((end - start).max()), 2),
           "last_cta_start_us": round(float(start.max()), 1),
           "mma_wait_share_cycles": {k: round(float(v / max(waits.sum(), 1)), 3) for k, v in zip("qkvp", waits)},
           "mma_wait_mcycles_per_cta": round(float(waits.sum() / n / 1e6), 4),
           "key_tiles_per_cta_mean": round(float(r[:, 8].mean()), 2),
           "epilogue_us_mean": round(float((end - mma_end).mean()), 2)}
    # softmax phases (cycles per key tile, warps 4 / 8): wait for S, TMEM load, max, exp + P store + arrive
    for x, nm in ((0, "softmax_A"), (1, "softmax_B")):
        ph = r[:, 10 + 5 * x: 15 + 5 * x].astype(np.float64)
        it = ph[:, 4].sum()
        if it > 0:
            out[nm] = {k: round(float(ph[:, i].sum() / it), 1) for i, k in enumerate(["wait_s", "tmem_ld", "max", "exp_store"])}
    print(json.dumps(out))


if __name__ == "__main__":
    main()
