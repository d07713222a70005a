#!/usr/bin/env python
"""bench.py -- mixed-batch tokens/s of the gLLM per-stage forward on B200 (BASELINE.json metric).

Workload (SURVEY.md §8(d) "PP sweep" row): Llama-3-8B-shaped random-init weights (O4),
the C1 synthetic stream (ShareGPT-like lengths, 6 req/tick, token budget #MaxP 2048,
Token Throttling defaults of PAPER.md L248), PP = --gpus stages, one process per GPU.

A step = one tick of the pipeline: the micro-batch chosen by Token Throttling goes
through every stage (all §8(a) rows).  The stream is first pre-rolled (untimed) for
`--preroll` ticks so the timed window sits in the steady state (window start 400).

  value  : device throughput.  W + K batches are scheduled and their metadata staged in HBM
           (gllm_stage_prepare) before the timed region; the region runs K forwards back to
           back.  tokens / (max over ranks of the CUDA-event time).
  e2e    : the serving loop through the public API with host buffers: build_batch on the
           host, stage_forward (metadata H2D inside), D2H of the sampled ids, retire of
           batch k-PP before batch k is built.
  --impl reference : the oracle (oracle/, CPU) timed on this host on bounded samples.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from workloads.configs import MODELS, SCHED  # noqa: E402
from workloads.streams import make_stream  # noqa: E402

METRIC = "mixed-batch tokens/s at PP=1/2/4/8 B200; bubble fraction; stage roofline %"
UNIT = "tokens/s"
FALLBACK_PEAKS = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1400.0}
# The driver's MEASURED_PEAKS.json of this round's pool, as copied into BASELINE.md §2 (the file
# itself is git-ignored and driver-written; a re-created container may not have it).
RECORDED_PEAKS = {"hbm_gbs": 6546.6, "bf16_tflops": 1626.2, "bf16_tflops_sustained": 1344.0}


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return d, "measured"
    if os.path.exists(os.path.join(ROOT, "BASELINE.md")):
        return RECORDED_PEAKS, "measured (MEASURED_PEAKS.json as recorded in BASELINE.md §2)"
    return FALLBACK_PEAKS, "fallback"


def kv_blocks_for(config, pp):
    # C1 uses 100000 blocks at PP=2 (~105 GB/stage); at PP=1 all 32 layers share one GPU -> 60000.
    # C2-C4 keep SURVEY §8(d)'s pools (their stages hold 8-12 layers).
    if config == "C1":
        return 60000 if pp == 1 else 100000
    return SCHED[config].num_blocks


def pp_of(args):
    return args.pp or args.gpus


def workload_config(args, sp):
    m = MODELS[args.config]
    PP = pp_of(args)
    emulated = args.gpus == 1 and PP > 1
    w = f"{args.config}: {m.name}-shaped random-init (O4), {args.config} stream, PP={PP}"
    if emulated:
        w += f", stage {args.stage} of {PP} run alone on 1 GPU (synthetic hidden_in)"
    return {"workload": w, "model": f"{m.name}-shape", "pp": PP, "parallelism": f"pp{PP}",
            "seq_len": f"mixed (stream {args.config})", "kv_blocks": sp.num_blocks,
            "emulated_stage": args.stage if emulated else None}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""

    def __init__(self, index):
        self.index = index
        self.p = None

    def __enter__(self):
        q = ("clocks.sm,clocks.max.sm,clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
             "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")
        try:
            self.p = subprocess.Popen(["nvidia-smi", "-i", str(self.index), f"--query-gpu={q}",
                                       "--format=csv,noheader,nounits", "-lms", "100"],
                                      stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
        except OSError:
            self.p = None
        return self

    def __exit__(self, *a):
        if self.p is not None:
            time.sleep(0.25)
            self.p.terminate()
            out, _ = self.p.communicate(timeout=5)
            self.lines = [l for l in out.splitlines() if l.strip()]

    def summary(self):
        if self.p is None or not getattr(self, "lines", None):
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        sm, mx, reasons = [], [], set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for l in self.lines:
            f = [x.strip() for x in l.split(",")]
            try:
                sm.append(float(f[0]))
                mx.append(float(f[1]))
            except ValueError:
                continue
            for n, v in zip(names, f[2:]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        return {"sm_mhz": float(np.median(sm)) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": sorted(reasons), "samples": len(sm)}


# ---------------------------------------------------------------------------- work model
def batch_work(m, a, n_layers, is_last):
    """Algorithmic (FLOPs, bytes) of one micro-batch per kernel category.

    GEMM bytes = weights read once + activations in + outputs out; whichever of FLOPs / Pi
    and bytes / beta is larger decides the bound (T below the ridge ~205 tokens -> HBM)."""
    T = int(a["num_tokens"])
    H, qd, kd, I, V = m.hidden, m.q_dim, m.kv_dim, m.intermediate, m.vocab
    ns = int(np.asarray(a["sample_idx"]).shape[0])
    NP = int(a["num_prefill_seqs"])
    cu, kvl = np.asarray(a["cu_q"], np.int64), np.asarray(a["kv_len"], np.int64)
    kvb = 2 * m.n_kv_heads * m.head_dim * 2          # K+V bytes per token per layer
    pairs = 0
    for i in range(NP):
        c = int(cu[i + 1] - cu[i])
        s = int(kvl[i]) - c
        pairs += c * s + c * (c + 1) // 2
    dec_keys = int(kvl[NP:].sum()) if kvl.shape[0] > NP else 0
    pre_keys = int(kvl[:NP].sum())                    # each prefill chunk reads its context once
    tp = int(cu[NP]) if NP else 0                     # prefill tokens
    nd = kvl.shape[0] - NP
    L = n_layers

    def gemm(M, N, K, out_bytes):
        return (2.0 * M * N * K * L, float((N * K * 2 + M * K * 2 + M * N * out_bytes) * L))
    w = {
        "qkv_gemm": gemm(T, qd + 2 * kd, H, 2),
        "o_gemm": gemm(T, H, qd, 8),            # fp32 residual read + write
        "gate_up_gemm": gemm(T, 2 * I, H, 1),   # bf16 SiLU*up output is half the columns
        "down_gemm": gemm(T, H, I, 8),
        "prefill_attn": (4.0 * m.n_heads * m.head_dim * pairs * L, float((pre_keys * kvb + tp * qd * 2 * 2) * L)),
        "decode_attn": (4.0 * m.n_heads * m.head_dim * dec_keys * L, float((dec_keys * kvb + nd * qd * 2 * 2) * L)),
        "rope_kv_append": (0.0, float(T * ((qd + 2 * kd) * 2 + qd * 2 + kvb) * L)),
        # fused RMSNorm: one statistics pass at stage entry (x fp32 in, bf16 x + fp32 sum of squares
        # out); the per-layer norms are GEMM epilogues.  Unfused (A/B): 2 passes per layer.
        "rmsnorm": ((0.0, float(T * H * (4 + 2) + T * 4)) if os.environ.get("GLLM_UNFUSED_NORM", "0") != "1"
                    else (0.0, float(2 * T * H * (4 + 2) * L))),
    }
    if is_last:
        w["lm_head"] = (2.0 * ns * H * V, float(V * H * 2 + ns * H * 2))
    return w


def roofline_report(timing_ms, work, launches, pk):
    """Per category: roofline time = max(FLOPs / Pi, bytes / beta) decides the bound; achieved is
    in the bound's unit.  The dominant (largest-time) kernel is the headline."""
    kern = {}
    pi = float(pk.get("bf16_tflops_sustained", pk["bf16_tflops"])) * 1e12
    beta = float(pk["hbm_gbs"]) * 1e9
    for name, ms in timing_ms.items():
        if name in ("total", "other", "attention_span") or name not in work or ms <= 0 or name.endswith("_overlapped"):
            continue
        flops, nbytes = work[name]
        sec = ms * 1e-3
        if flops / pi >= nbytes / beta:
            bound, ach, peak, unit = "tensor", flops / sec / 1e12, pi / 1e12, "TFLOP/s"
        else:
            bound, ach, peak, unit = "hbm", nbytes / sec / 1e9, beta / 1e9, "GB/s"
        kern[name] = {"bound": bound, "achieved": round(ach, 1), "peak": round(peak, 1), "unit": unit,
                      "frac": round(ach / peak, 4), "ms": round(ms, 3),
                      "share": round(ms / max(timing_ms.get("total", ms), 1e-9), 4)}
        if name + "_overlapped" in timing_ms:
            kern[name]["timing"] = "attribution pass (attention kernels in series); timed steps overlap them"
            kern[name]["ms_span_in_timed_steps"] = round(timing_ms[name + "_overlapped"], 3)
    dom = max(kern, key=lambda k: kern[k]["ms"]) if kern else None
    return dom, kern


def stage_roofline(timing_ms, work, pk):
    """Per-stage roofline %: sum over the step's kernels of max(FLOPs/Pi, bytes/beta)
    divided by the measured stage time.  Prefill and decode attention run concurrently (tensor
    pipe vs HBM): their joint bound is max(prefill FLOPs/Pi, (prefill + decode bytes)/beta)."""
    pi = float(pk.get("bf16_tflops_sustained", pk["bf16_tflops"])) * 1e12
    beta = float(pk["hbm_gbs"]) * 1e9
    t = 0.0
    w = dict(work)
    if "rope_kv_append" in w:  # fused into the QKV GEMM epilogue: one kernel, bytes add up
        rf, rb = w.pop("rope_kv_append")
        qf, qb = w.get("qkv_gemm", (0.0, 0.0))
        w["qkv_gemm"] = (qf + rf, qb + rb)
    for name, (fl, by) in w.items():
        if name in ("prefill_attn", "decode_attn"):
            continue
        t += max(fl / pi, by / beta)
    pf, pb = work.get("prefill_attn", (0.0, 0.0))
    df, db = work.get("decode_attn", (0.0, 0.0))
    t += max((pf + df) / pi, (pb + db) / beta)
    total = timing_ms.get("total", 0.0) * 1e-3
    return {"roofline_ms": round(t * 1e3, 3), "measured_ms": round(total * 1e3, 3),
            "frac": round(t / total, 4) if total > 0 else None,
            "attention_span_ms": round(timing_ms.get("attention_span", 0.0), 3)}


# ---------------------------------------------------------------------------- our arm
def run_ours(args):
    import torch
    import torch.distributed as dist

    from paper_conf_sc_00090d00l25_b200 import gllm
    from paper_conf_sc_00090d00l25_b200.runtime import (GpuExecutor, NcclTransport, Pipeline, fill_warm, pack_desc,
                                                        split_layers, unpack_desc)
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    N = args.gpus
    assert world == N, f"--gpus {N} but WORLD_SIZE {world}"
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    meta = None
    if world > 1:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        dist.init_process_group("gloo", rank=rank, world_size=world)
        meta = dist.group.WORLD
    m = MODELS[args.config]
    PP = pp_of(args)
    emulate = world == 1 and PP > 1          # one stage of a PP-stage deployment on this GPU
    assert emulate or PP == N, "--pp must equal --gpus unless emulating one stage on one GPU"
    sidx = args.stage if emulate else rank
    sp = SCHED[args.config].with_(pp_depth=PP, num_blocks=args.kv_blocks or kv_blocks_for(args.config, PP))
    lb, le = split_layers(m.n_layers, PP)[sidx]
    max_tokens = sp.maxp + -(-sp.max_seqs // PP) + 64
    stage = gllm.Stage(m, lb, le, sp.num_blocks, max_tokens, sp.max_seqs, device=local)
    ex = GpuExecutor(stage, dev, max_tokens, m.hidden, pp=PP)
    if emulate and sidx > 0:
        for b in ex.hin:
            b.normal_()                       # synthetic activations arriving from stage sidx-1
    stream = make_stream(args.config, m.vocab)
    fill_warm(stage, sp, stream.warm)         # C4 warm-start decode set: its cache pages hold the O4 values
    tr = None
    if world > 1:
        if args.handoff == "peer":   # fused hand-off over NVLink peer memory (gllm_peer_*)
            from paper_conf_sc_00090d00l25_b200.runtime import PeerTransport
            tr = PeerTransport(ex, rank, world, meta)
        else:
            uid = [gllm.get_unique_id() if rank == 0 else None]
            dist.broadcast_object_list(uid, 0)
            stage.comm_init(uid[0], rank, world)
            nccl_info = stage.comm_size()
            print(f"[bench] rank {rank}: NCCL communicator nranks={nccl_info[0]} rank={nccl_info[1]}",
                  file=sys.stderr, flush=True)
            assert nccl_info == (world, rank), nccl_info
            tr = NcclTransport(ex, rank, world)
    sched = None
    if rank == 0:
        sched = gllm.Sched(sp)
        sched.add_stream(stream)
    pipe = Pipeline(rank, world, ex, tr, sched, meta, pp=PP, stage=sidx if emulate else None)

    def barrier():
        torch.cuda.synchronize(dev)
        if world > 1:
            dist.barrier()

    # ---- pre-roll into the steady-state window (untimed, full pipeline)
    t0 = time.time()
    for _ in range(args.preroll):
        pipe.tick()
    pipe.drain()
    barrier()
    preroll_s = time.time() - t0

    # ---- value: W + K batches scheduled and staged in HBM up front, then K forwards timed
    batches = []
    sched_s = []   # host time of each Token-Throttling build_batch (the paper's 0.045 ms/iteration, L212)
    for _ in range(args.warmup + args.steps):
        buf = None
        if rank == 0:
            # teacher-forced schedule (R17): the sampled ids never change the schedule
            t_b = time.perf_counter()
            d = sched.build_batch()
            sched_s.append(time.perf_counter() - t_b)
            buf = pack_desc(d)
        batches.append(unpack_desc(pipe._bcast(buf)))
    handles = [ex.prepare(a) if a["num_tokens"] > 0 else None for a in batches]
    barrier()
    for a, h in zip(batches[: args.warmup], handles[: args.warmup]):
        pipe.run_batch(a, h)
    barrier()
    # timed pass: the K staged batches with no per-kernel events (they cost 1-10% of a step)
    stage.set_profiling(False)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    launches = 0
    with Clocks(local) as clk:
        barrier()
        torch.cuda.nvtx.range_push("timed")   # ncu --nvtx --nvtx-include timed/ selects this region
        ev0.record(ex.compute)
        for a, h in zip(batches[args.warmup:], handles[args.warmup:]):
            pipe.run_batch(a, h)
            launches += stage.last_launches()
        ev1.record(ex.compute)
        barrier()
        torch.cuda.nvtx.range_pop()
    ms_local = ev0.elapsed_time(ev1)
    # profiled pass (untimed): the same K batches, same launches and stream overlap, with CUDA
    # events around every kernel category on its own stream -> per-kernel durations and the
    # stage's busy time (bubble fraction)
    stage.set_profiling(True)
    stage.last_timing()  # reset accumulation
    pv0, pv1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    barrier()
    pv0.record(ex.compute)
    for a, h in zip(batches[args.warmup:], handles[args.warmup:]):
        pipe.run_batch(a, h)
    pv1.record(ex.compute)
    barrier()
    stage.set_profiling(False)
    ms_prof = pv0.elapsed_time(pv1)
    timing = stage.last_timing()
    # attribution pass (untimed): the same K batches again with the prefill and decode attention
    # kernels in series, so each one's events bracket that kernel alone (in the timed steps they
    # share the SMs on two streams and the side stream's span is the whole attention step)
    stage.set_profiling(2)
    stage.last_timing()
    for a, h in zip(batches[args.warmup:], handles[args.warmup:]):
        pipe.run_batch(a, h)
    barrier()
    serial = stage.last_timing()
    stage.set_profiling(False)
    for kname in ("prefill_attn", "decode_attn"):
        timing[kname + "_overlapped"] = timing.get(kname, 0.0)
        timing[kname] = serial.get(kname, 0.0)
    for h in handles:
        if h is not None:
            ex.release(h)
    t = torch.tensor([ms_local], dtype=torch.float64)
    if world > 1:
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
    ms = float(t[0])
    timed = batches[args.warmup:]
    tokens = sum(int(a["num_tokens"]) for a in timed)
    value = tokens / (ms * 1e-3)
    # stage busy time vs span -> bubble fraction (device): 1 - busy/span per stage, max over stages
    busy = torch.tensor([timing["total"]], dtype=torch.float64)
    bubble_local = max(0.0, 1.0 - timing["total"] / ms_prof) if ms_prof > 0 else 0.0
    bub = torch.tensor([bubble_local], dtype=torch.float64)
    if world > 1:
        allb = [torch.zeros(1, dtype=torch.float64) for _ in range(world)]
        dist.all_gather(allb, bub)
        bubbles = [float(x[0]) for x in allb]
    else:
        bubbles = [bubble_local]

    # roofline of this rank's dominant kernel (rank 0 reports its own stage)
    work = {}
    for a in timed:
        for kname, (fl, by) in batch_work(m, a, le - lb, le == m.n_layers).items():
            f0, b0 = work.get(kname, (0.0, 0.0))
            work[kname] = (f0 + fl, b0 + by)
    pk, pk_src = peaks()
    dom, kern = roofline_report(timing, work, launches, pk)
    stage_rl = stage_roofline(timing, work, pk)
    traffic = None
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    if dom and os.path.exists(tp):
        traffic = json.load(open(tp)).get(f"{args.config}-pp{N}", {}).get(dom)

    # ---- e2e: serving loop through the public API (host scheduler, H2D metadata, D2H ids)
    # the value-phase batches were scheduled directly (teacher forcing, R17) and retire without
    # sampled ids: forget their sample bookkeeping so no rank waits for ids nobody sends
    pipe.pending_samples.clear()
    pipe._expect.clear()
    # replay the SAME window: a fresh scheduler is fast-forwarded on the host to the value phase's
    # first tick (the cache pages then hold earlier values, which does not change the work), W
    # serving ticks warm up, and the K timed ticks are exactly the value phase's timed ticks
    if rank == 0:
        sched = gllm.Sched(sp)
        sched.add_stream(stream)
        for _ in range(int(batches[0]["tick"])):
            sched.build_batch()
        pipe.sched = sched
    for _ in range(args.warmup):
        pipe.tick()
    h2d = d2h = 0
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e2e_tokens = 0
    barrier()
    e0.record(ex.compute)
    for _ in range(args.steps):
        a = pipe.tick()
        e2e_tokens += int(a["num_tokens"])
        T, S = int(a["num_tokens"]), int(a["num_seqs"])
        h2d += 4 * (2 * T + (S + 1) + S + int(np.asarray(a["block_table"]).size) + int(a["sample_idx"].shape[0]))
        d2h += 4 * int(a["sample_idx"].shape[0])
    pipe.drain()
    if rank == 0 and world == 1:
        # the last tick's sampled ids are read back too (its retire happens at the next build)
        k = int(a["tick"])
        if a["sample_idx"].shape[0]:
            ex.sampled(k, int(a["sample_idx"].shape[0]))
    e1.record(ex.compute)
    barrier()
    te = torch.tensor([e0.elapsed_time(e1)], dtype=torch.float64)
    if world > 1:
        dist.all_reduce(te, op=dist.ReduceOp.MAX)
    e2e_value = e2e_tokens / (float(te[0]) * 1e-3)

    if rank == 0:
        cpu = (cpu_baseline(args, m, timed[0], le - lb, le == m.n_layers)
               if (N == 1 and not args.no_cpu_baseline) else None)
        clocks = clk.summary()
        out = {
            "metric": METRIC, "value": round(value, 1), "unit": UNIT, "n_gpus": N, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms / args.steps, 3), "higher_is_better": True,
            "scaling": "strong", "vs_baseline": None, "dtype": "bf16", "data": "synthetic",
            "config": {**workload_config(args, sp), "layers_per_stage": le - lb,
                       "global_batch": round(tokens / args.steps, 1),
                       "token_budget": sp.maxp, "preroll_ticks": args.preroll,
                       "handoff": args.handoff if N > 1 else None,
                       "window_ticks": [int(timed[0]["tick"]), int(timed[-1]["tick"])],
                       "l2": f"inputs > L2: every step streams all {le - lb} layers' weights (GBs >> 126 MB L2)"},
            "e2e": {"value": round(e2e_value, 1), "unit": UNIT, "h2d_bytes_per_step": int(h2d / args.steps),
                    "d2h_bytes_per_step": int(d2h / args.steps)},
            "gpu_launches": int(launches),
            "roofline": ({"kernel": dom, "bound": kern[dom]["bound"], "achieved": kern[dom]["achieved"],
                          "peak": kern[dom]["peak"], "unit": kern[dom]["unit"], "frac": kern[dom]["frac"],
                          "traffic": traffic, "peak_source": pk_src + (" sustained" if kern[dom]["bound"] == "tensor" else "")}
                         if dom else None),
            "kernels": kern,
            "stage_roofline": stage_rl,
            "bubble_fraction": {"per_stage": [round(b, 4) for b in bubbles], "max": round(max(bubbles), 4),
                                "mean": round(float(np.mean(bubbles)), 4)},
            "cpu_baseline": cpu,
            "sched": {"build_batch_us_per_tick": round(float(np.mean(sched_s)) * 1e6, 1) if sched_s else None,
                      "build_batch_us_max": round(float(np.max(sched_s)) * 1e6, 1) if sched_s else None,
                      "ticks": len(sched_s), "paper_us_per_iter": 45.0},
            "clocks": clocks,
            "preroll_s": round(preroll_s, 1),
        }
        print(json.dumps(out))
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


# ---------------------------------------------------------------------------- oracle (CPU)
def _cpu_model():
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def _blas_threads():
    try:
        from threadpoolctl import threadpool_info
        return max((p.get("num_threads", 1) for p in threadpool_info()), default=os.cpu_count())
    except Exception:
        return os.cpu_count()


def _oracle_layer_time(m, a, W, layer=0):
    """Wall time of ONE decoder layer of oracle.model.stage_forward on batch `a` at full width (the
    embedding rows are the stage input; no LM head).  Returns seconds, measured."""
    from oracle import model as om

    class B:
        pass
    b = B()
    for k in ("token_ids", "positions", "slot_mapping", "cu_q", "kv_len", "block_table", "sample_idx"):
        setattr(b, k, np.asarray(a[k]))
    b.num_tokens = int(a["num_tokens"])
    cache = om.PagedCache(m, 16, np.float32)
    # the pages this batch reads from earlier ticks: the O4 warm-KV values of each sequence (the oracle's
    # arithmetic does not depend on them; they make the sample self-contained)
    from oracle.weights import warm_kv
    for i, (row, n) in enumerate(zip(np.asarray(a["block_table"]), np.asarray(a["kv_len"]))):
        k, v = warm_kv(m.weight_seed, i, int(n), layer, m.n_kv_heads, m.head_dim)
        cache.fill_warm(layer, row, k, v)
    W.layer(layer)  # weights generated outside the timed region
    x = W.embed_rows(b.token_ids)
    t0 = time.perf_counter()
    om.stage_forward(m, W, cache, b, layer, layer + 1, hidden_in=x)
    return time.perf_counter() - t0


def _layer_flops(m, T):
    return 2.0 * T * (m.hidden * (m.q_dim + 2 * m.kv_dim) + m.q_dim * m.hidden + 3 * m.hidden * m.intermediate)


def cpu_baseline(args, m, a, n_layers=None, with_lm_head=True):
    """The oracle as it stands on a bounded sample: ONE decoder layer of the first timed tick's whole
    batch, timed for real with all BLAS threads and with one thread, then expressed in the metric's
    unit for the stage (time x layers, + the LM head's FLOP share)."""
    from oracle.weights import Weights
    n_layers = n_layers or m.n_layers
    W = Weights(m)
    T = int(a["num_tokens"])
    lm = (2.0 * int(np.asarray(a["sample_idx"]).shape[0]) * m.hidden * m.vocab if with_lm_head else 0.0)
    scale = n_layers + lm / _layer_flops(m, T)
    sec = _oracle_layer_time(m, a, W)
    sec1 = None
    try:
        from threadpoolctl import threadpool_limits
        with threadpool_limits(limits=1):
            sec1 = _oracle_layer_time(m, a, W)
    except Exception:
        pass
    return {"value": round(T / (sec * scale), 2), "unit": UNIT, "cores": int(_blas_threads()), "kind": "oracle",
            "sample": f"measured: oracle fp32 forward of 1 decoder layer on the first timed tick's whole batch "
                      f"(T={T}): {sec:.2f} s on {_blas_threads()} threads; value = T / (that time x {scale:.2f} "
                      f"layer-equivalents of the stage)",
            "one_thread": ({"value": round(T / (sec1 * scale), 3), "layer_s": round(sec1, 2)} if sec1 else None),
            "layer_s": round(sec, 3), "cpu_model": _cpu_model(), "host_cpus": os.cpu_count()}


def run_reference(args):
    """--impl reference: the oracle as it stands on the host cores.  Each step is a bounded sample of
    that tick's workload: one decoder layer over the tick's whole batch, timed for real; ms_per_step
    is that measured time, `value` expresses it for the whole model (x layers + LM-head share)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle.scheduler import Scheduler
    from oracle.weights import Weights
    m = MODELS[args.config]
    N = args.gpus
    sp = SCHED[args.config].with_(pp_depth=pp_of(args), num_blocks=args.kv_blocks or kv_blocks_for(args.config, pp_of(args)))
    st = make_stream(args.config, m.vocab)
    s = Scheduler(sp, st.requests, st.warm)
    for _ in range(args.preroll):
        s.build_batch()
    W = Weights(m)
    W.layer(0)
    tot_tokens, tot_equiv, tot_meas = 0, 0.0, 0.0
    t_start = time.perf_counter()
    for i in range(args.warmup + args.steps):
        b = s.build_batch()
        a = dict(token_ids=b.token_ids, positions=b.positions, slot_mapping=b.slot_mapping, cu_q=b.cu_q,
                 kv_len=b.kv_len, block_table=b.block_table, sample_idx=b.sample_idx, num_tokens=b.num_tokens)
        if b.num_tokens == 0 or i < args.warmup:   # (the oracle has nothing to warm up)
            continue
        sec = _oracle_layer_time(m, a, W)
        T = b.num_tokens
        scale = m.n_layers + 2.0 * len(b.sample_idx) * m.hidden * m.vocab / _layer_flops(m, T)
        if i >= args.warmup:
            tot_tokens += T
            tot_meas += sec
            tot_equiv += sec * scale
    wall = time.perf_counter() - t_start
    v = tot_tokens / tot_equiv if tot_equiv > 0 else 0.0
    sample = (f"per step: the oracle's fp32 forward of 1 of {m.n_layers} decoder layers over that tick's whole batch, "
              f"measured ({tot_meas / max(args.steps, 1):.2f} s/step); value = tokens / (measured time x layers + "
              f"LM-head share)")
    out = {"impl": "reference", "metric": METRIC, "value": round(v, 2), "unit": UNIT, "n_gpus": N,
           "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(tot_meas / max(args.steps, 1) * 1e3, 1),
           "ms_per_step_model_equivalent": round(tot_equiv / max(args.steps, 1) * 1e3, 1),
           "wall_s": round(wall, 1),
           "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": workload_config(args, sp),
           "cpu_baseline": {"value": round(v, 2), "unit": UNIT, "cores": int(_blas_threads()), "kind": "oracle",
                            "sample": sample, "cpu_model": _cpu_model()},
           "e2e": {"value": round(v, 2), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default="C1")
    ap.add_argument("--preroll", type=int, default=None,
                    help="ticks run before the window (default: the config's window start)")
    ap.add_argument("--pp", type=int, default=0, help="pipeline depth (default --gpus)")
    ap.add_argument("--stage", type=int, default=0, help="with --gpus 1 --pp N: which stage to run")
    ap.add_argument("--kv-blocks", type=int, default=0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--handoff", default="peer", choices=["nccl", "peer"],
                    help="N > 1: the fused peer-memory hand-off (default; flags + slot credits over NVLink) or "
                         "NCCL P2P send/recv")
    args = ap.parse_args()
    if args.preroll is None:
        from workloads.configs import STREAMS
        args.preroll = int(STREAMS[args.config].get("window", (400, None))[0])
    if args.warmup < 3:
        args.warmup = 3
    if args.impl == "reference":
        run_reference(args)
    else:
        run_ours(args)


if __name__ == "__main__":
    main()
