"""Pipeline-bubble evaluation of Token Throttling vs Sarathi-Serve on measured B200 stage times
(the paper's central claim, §2.4-2.5, Fig. 15).

One GPU runs stage `--stage` of a `--pp`-stage split of config C* (the per-stage work of a PP
deployment: same layer count, same micro-batches as the PP scheduler produces) over a window of
ticks, timing every micro-batch's stage forward with CUDA events.  A discrete-event model then
replays the window through PP identical stages with the pipeline's two dependencies -- micro-batch
k enters stage s when stage s-1 finished k and stage s finished k-1, and enters stage 0 only
after k-PP left the last stage (at most PP in flight, L179) -- giving the bubble fraction
1 - busy / (PP * makespan) and tokens/s for each policy.

    python tools/pipeline_model.py --config C2 --pp 4 --stage 1 --ticks 200
"""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_00090d00l25_b200 import gllm  # noqa: E402
from paper_conf_sc_00090d00l25_b200.runtime import fill_warm, split_layers  # noqa: E402
from workloads.configs import MODELS, SCHED, STREAMS  # noqa: E402
from workloads.streams import make_stream  # noqa: E402


def measure(config, pp, stage_idx, policy, preroll, ticks, kv_blocks=None, host_us=0.0, **sched_kw):
    m = MODELS[config]
    sp = SCHED[config].with_(pp_depth=pp, policy=policy, token_budget=2048,
                             num_blocks=kv_blocks or SCHED[config].num_blocks, **sched_kw)
    lb, le = split_layers(m.n_layers, pp)[stage_idx]
    max_tokens = max(sp.maxp, sp.token_budget) + sp.max_seqs + 64
    st = gllm.Stage(m, lb, le, sp.num_blocks, max_tokens, sp.max_seqs)
    fill_warm(st, sp, make_stream(config, m.vocab).warm)
    s = gllm.Sched(sp)
    s.add_stream(make_stream(config, m.vocab))
    dev = torch.device("cuda")
    hin = torch.randn((max_tokens, m.hidden), device=dev)
    hout = torch.empty((max_tokens, m.hidden), device=dev)
    samp = torch.empty((sp.max_seqs,), dtype=torch.int32, device=dev)
    stream = torch.cuda.current_stream()
    first, last = stage_idx == 0, le == m.n_layers

    def fwd(d):
        st.forward(d, 0 if first else hin.data_ptr(), 0 if last else hout.data_ptr(),
                   samp.data_ptr() if last else 0, stream.cuda_stream)

    for _ in range(preroll):
        d = s.build_batch()
        if d.num_tokens:
            fwd(d)
    torch.cuda.synchronize()
    pre0 = s.stats()["preemptions"]
    times, toks, pre, dec = [], [], [], []
    samples = []   # per tick: request ids whose next token is sampled (prompt completions + decodes)
    k0 = s.stats()["tick"]
    for _ in range(ticks):
        d = s.build_batch()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        if d.num_tokens:
            fwd(d)
        e1.record()
        torch.cuda.synchronize()
        times.append(e0.elapsed_time(e1) if d.num_tokens else 0.0)
        toks.append(d.num_tokens)
        pre.append(d.num_prefill_tokens)
        dec.append(d.num_decode_tokens)
        a = d.to_numpy()
        cu, rid = a["cu_q"], a["seq_req_ids"]
        seq_of = np.searchsorted(cu, a["sample_idx"], side="right") - 1 if d.num_tokens else np.zeros(0, int)
        samples.append([int(rid[i]) for i in seq_of])
    preempt = s.stats()["preemptions"] - pre0
    st.close()
    arrivals = {r.req_id: r.arrival_tick - k0 for r in make_stream(config, m.vocab).requests}
    return np.array(times), np.array(toks), np.array(pre), np.array(dec), samples, arrivals, preempt


def latencies(samples, arrivals, start, fin):
    """Tick-based serving proxies on the simulated pipeline (§4.6's metrics, Fig. 16): TTFT =
    finish of the micro-batch that completes a prompt - start of the tick the request arrived in;
    TPOT = mean gap between a request's consecutive sampled tokens.  Only requests arriving inside
    the measured window count for TTFT."""
    first, last, gaps = {}, {}, []
    for k, ids in enumerate(samples):
        for r in ids:
            if r not in first:
                first[r] = k
            elif r in last:
                gaps.append(fin[k] - fin[last[r]])
            last[r] = k
    ttft = [fin[k] - start[arrivals[r]] for r, k in first.items()
            if r in arrivals and 0 <= arrivals[r] < len(start) and k >= arrivals[r]]
    return (float(np.mean(ttft)) if ttft else None, float(np.mean(gaps)) if gaps else None, len(ttft))


def simulate(t_ms, pp, host_ms=0.05):
    """Identical stages taking t_ms[k] for micro-batch k; returns (makespan ms, bubble fraction)."""
    n = len(t_ms)
    fin = np.zeros((pp, n))
    for k in range(n):
        for s in range(pp):
            start = 0.0
            if s > 0:
                start = max(start, fin[s - 1, k])
            if k > 0:
                start = max(start, fin[s, k - 1])
            if s == 0 and k >= pp:  # at most PP micro-batches in flight: k waits for k-PP's retire
                start = max(start, fin[pp - 1, k - pp] + host_ms)
            fin[s, k] = start + t_ms[k]
    makespan = fin[pp - 1, n - 1]
    busy = pp * float(np.sum(t_ms))
    start0 = fin[0] - t_ms   # when micro-batch k entered stage 0
    return makespan, 1.0 - busy / (pp * makespan), start0, fin[pp - 1]


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--pp", type=int, default=4)
    ap.add_argument("--stage", type=int, default=1)
    ap.add_argument("--ticks", type=int, default=160)
    ap.add_argument("--preroll", type=int, default=None)
    ap.add_argument("--policies", default="0,1",
                    help="0 token throttling, 1 Sarathi-Serve (w/ CK), 2 w/o WT, 3 w/o UT (PAPER.md §4.5), "
                         "4 context-aware throttling (R21, L354)")
    ap.add_argument("--ctx-a", type=int, default=20000,
                    help="policy 4 (context-aware throttling, R21): attention pairs per token-equivalent")
    ap.add_argument("--sweep", default="",
                    help="hyperparameter sensitivity (PAPER.md §4.6, Fig. 16) under token throttling, e.g. "
                         "'iterp=1,2,4,8,16' or 'maxp=512,1024,2048' or 'kvthresh_num=0,1,2' (den 20)")
    a = ap.parse_args()
    preroll = a.preroll if a.preroll is not None else int(STREAMS[a.config].get("window", (400, None))[0])
    out = {"config": a.config, "pp": a.pp, "stage": a.stage, "ticks": a.ticks, "preroll": preroll}
    names = {0: "token_throttling", 1: "sarathi_serve", 2: "no_wt", 3: "no_ut", 4: "context_aware"}
    runs = [(names[int(p)], int(p), {"attn_pairs_per_token": a.ctx_a} if int(p) == 4 else {})
            for p in a.policies.split(",") if p != ""]
    if a.sweep:
        key, vals = a.sweep.split("=")
        runs = [(f"{key}={v}", 0, {key: int(v)}) for v in vals.split(",")]
        out["sweep"] = key
    for name, pol, kw in runs:
        t, toks, pre, dec, samples, arrivals, preempt = measure(a.config, a.pp, a.stage, pol, preroll, a.ticks, **kw)
        mk, bub, start0, fin_last = simulate(t, a.pp)
        ttft, tpot, n_ttft = latencies(samples, arrivals, start0, fin_last)
        out[name] = {"tokens_per_s": round(float(toks.sum()) / (mk * 1e-3), 1), "bubble_fraction": round(bub, 4),
                     "preemptions": int(preempt), "ttft_ms": round(ttft, 2) if ttft is not None else None,
                     "ttft_requests": n_ttft, "tpot_ms": round(tpot, 3) if tpot is not None else None,
                     "stage_ms_mean": round(float(t.mean()), 3), "stage_ms_cv": round(float(t.std() / t.mean()), 3),
                     "tokens_mean": round(float(toks.mean()), 1), "tokens_cv": round(float(toks.std() / toks.mean()), 3),
                     "prefill_mean": round(float(pre.mean()), 1), "decode_mean": round(float(dec.mean()), 1)}
        print(name, json.dumps(out[name]), flush=True)
    print(json.dumps(out))
