"""Fused stage hand-off over peer memory (a12; include/gllm.h gllm_peer_*).

Two processes share the one GPU (CUDA IPC works between processes on the same device): the
sender holds layer 0 of the C0 model (stage 0 of 2), the receiver layer 1 + the LM head (stage 1).
The sender's last residual-add GEMM epilogue stores its output rows straight into the receiver's
ring slot and raises the slot flag; the receiver's stream waits on the flag and reads the slot as
hidden_in.  The receiver's hidden states and greedy ids must match the oracle's two-layer forward
(north_star bars), tick by tick over the C0 stream and a C1-shaped prefix (stream-K and whole-tile
schedules of the last GEMM).

The free-running variant removes the lockstep: the sender enqueues every tick back to back with a
2-slot ring while the receiver sleeps before each tick, so only the slot credits (the receiver's
stage-entry kernel releases each slot; the sender's stream waits for the credit before overwriting)
keep the sender from overwriting slots the receiver has not read."""
import multiprocessing as mp
import os

import numpy as np
import pytest

from workloads.configs import MODELS, SCHED, SchedParams
from workloads.streams import make_stream

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _cases():
    return {
        "C0": (MODELS["C0"], SCHED["C0"], ("C0", None), 2, 256, 4),
        # 2 layers of Llama-3-8B shape: ticks with T in the hundreds to ~2000 (whole-tile epilogue)
        "C1": (MODELS["C1"].with_layers(2), SchedParams(pp_depth=2, num_blocks=3000), ("C1", 60), 2, 2600, 6),
    }


def _sender(case, lockstep, q_handle, q_credit, q_desc, q_done):
    import sys
    sys.path.insert(0, ROOT)
    import torch
    from paper_conf_sc_00090d00l25_b200 import gllm
    m, cfg, (sname, n), depth, mt, ticks = _cases()[case]
    st = make_stream(sname, m.vocab, n=n) if n else make_stream(sname, m.vocab)
    stage = gllm.Stage(m, 0, 1, cfg.num_blocks, mt, min(cfg.max_seqs, mt))
    sched = gllm.Sched(cfg)
    sched.add_stream(st)
    q_credit.put(stage.peer_ring_open(q_handle.get(timeout=120)))
    s = torch.cuda.current_stream().cuda_stream
    for k in range(ticks):
        d = sched.build_batch()
        a = d.to_numpy()
        q_desc.put(a)
        if d.num_tokens:
            h = stage.prepare(d, s)
            stage.forward_prepared_peer(h, int(a["tick"]), 0, s)
            if lockstep:
                torch.cuda.synchronize()
            stage.release(h)   # (a prepared slot is reused only after its forward completed)
        if lockstep:
            assert q_done.get(timeout=300) == k    # the receiver consumed tick k
    torch.cuda.synchronize()
    if not lockstep:
        for k in range(ticks):   # keep the credit memory alive until the receiver is done
            assert q_done.get(timeout=600) == k
    stage.close()


def _receiver(case, lockstep, q_handle, q_credit, q_desc, q_done, q_out):
    import sys
    sys.path.insert(0, ROOT)
    import torch
    from paper_conf_sc_00090d00l25_b200 import gllm
    m, cfg, _, depth, mt, ticks = _cases()[case]
    stage = gllm.Stage(m, 1, 2, cfg.num_blocks, mt, min(cfg.max_seqs, mt))
    q_handle.put(stage.peer_ring_create(depth))
    stage.peer_credit_open(q_credit.get(timeout=120))
    dev = torch.device("cuda", 0)
    s = torch.cuda.current_stream().cuda_stream
    for k in range(ticks):
        a = q_desc.get(timeout=300)
        if not lockstep:
            import time
            time.sleep(0.3)      # let the sender run ahead by more than the ring depth
        T = int(a["num_tokens"])
        res = {"tick": int(a["tick"]), "T": T}
        if T:
            d, keep = gllm.desc_from_arrays(a)
            h = stage.prepare(d, s)
            slot = stage.peer_ring_recv(int(a["tick"]), s)
            hout = torch.empty((T, m.hidden), dtype=torch.float32, device=dev)
            samp = torch.full((max(d.num_samples, 1),), -1, dtype=torch.int32, device=dev)
            stage.forward_prepared(h, slot, hout.data_ptr(), samp.data_ptr(), s)
            torch.cuda.synchronize()
            stage.release(h)
            res["hidden"] = hout.cpu().numpy()
            res["sampled"] = samp.cpu().numpy()[: d.num_samples]
        q_out.put(res)
        q_done.put(k)
    stage.close()


@pytest.mark.timeout(900)
@pytest.mark.parametrize("case,lockstep", [("C0", True), ("C1", True), ("C1", False)])
def test_peer_handoff_two_processes_one_gpu(case, lockstep):
    from tests.gpu_harness import OracleRun, TOL_HIDDEN, greedy_ok, row_rel_err
    m, cfg, (sname, n), depth, mt, ticks = _cases()[case]
    ctx = mp.get_context("spawn")
    q_handle, q_credit, q_desc, q_done, q_out = ctx.Queue(), ctx.Queue(), ctx.Queue(), ctx.Queue(), ctx.Queue()
    ps = [ctx.Process(target=_sender, args=(case, lockstep, q_handle, q_credit, q_desc, q_done)),
          ctx.Process(target=_receiver, args=(case, lockstep, q_handle, q_credit, q_desc, q_done, q_out))]
    for p in ps:
        p.start()
    outs = [q_out.get(timeout=600) for _ in range(ticks)]
    for p in ps:
        p.join(timeout=120)
        assert p.exitcode == 0, f"worker exit code {p.exitcode}"
    st = make_stream(sname, m.vocab, n=n) if n else make_stream(sname, m.vocab)
    orc = OracleRun(m, cfg, st, 0, 2)
    checked = 0
    for r in outs:
        o = orc.step()
        assert int(o["batch"].tick) == r["tick"] and o["batch"].num_tokens == r["T"]
        if not r["T"]:
            continue
        err = row_rel_err(r["hidden"], o["hidden"])
        assert err.max() <= TOL_HIDDEN, (r["tick"], err.max())
        if len(o["batch"].sample_idx):
            assert greedy_ok(r["sampled"], o["logits"]).mean() >= 0.99
        checked += r["T"]
    assert checked > 0
