"""Pipeline host protocol with world_size 2 on gloo (CPU): metadata broadcast from the driver,
hidden-state hand-off stage 0 -> 1, sampled ids back to the driver, retire of batch k-PP before
batch k.  The stage executor here is the oracle (test-only),
so the 2-stage pipeline must reproduce the 1-process oracle exactly."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

from paper_conf_sc_00090d00l25_b200.runtime import pack_desc, split_layers, unpack_desc
from workloads.configs import MODELS, SCHED
from workloads.streams import make_stream


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class OracleExecutor:
    def __init__(self, m, lb, le, block_size):
        from oracle import model as om
        from oracle.weights import Weights
        self.om, self.m, self.lb, self.le = om, m, lb, le
        self.W = Weights(m)
        self.cache = om.PagedCache(m, block_size)
        self.hin, self.hout, self.samp = {}, {}, {}

    def prepare(self, a):
        class B:
            pass
        b = B()
        for k in ("token_ids", "positions", "slot_mapping", "cu_q", "kv_len", "block_table", "sample_idx"):
            setattr(b, k, np.asarray(a[k]))
        b.num_tokens = int(a["num_tokens"])
        return b

    def release(self, h):
        pass

    def forward(self, b, k, T, is_first, is_last, ns):
        r = self.om.stage_forward(self.m, self.W, self.cache, b, self.lb, self.le, self.hin.pop(k, None))
        self.hout[k] = r["hidden"]
        if is_last:
            self.samp[k] = r.get("sampled", np.zeros(0, np.int32))

    def sampled(self, k, ns):
        return self.samp[k][:ns]


class GlooTransport:
    def __init__(self, ex, rank, group):
        self.ex, self.rank, self.group = ex, rank, group

    def recv(self, k, T):
        import torch
        import torch.distributed as dist
        t = torch.empty((T, self.ex.m.hidden), dtype=torch.float32)
        dist.recv(t, self.rank - 1, group=self.group)
        self.ex.hin[k] = t.numpy()

    def send(self, k, T):
        import torch
        import torch.distributed as dist
        dist.send(torch.from_numpy(np.ascontiguousarray(self.ex.hout.pop(k), np.float32)), self.rank + 1,
                  group=self.group)


def _worker(rank, world, port, ticks, q):
    import torch.distributed as dist

    from paper_conf_sc_00090d00l25_b200 import gllm
    from paper_conf_sc_00090d00l25_b200.runtime import Pipeline
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    m = MODELS["C0"].with_layers(4)
    sp = SCHED["C0"].with_(pp_depth=world, num_blocks=256, iterp=2, maxp=96, minp=8)
    lb, le = split_layers(m.n_layers, world)[rank]
    ex = OracleExecutor(m, lb, le, sp.block_size)
    sched = None
    if rank == 0:
        sched = gllm.Sched(sp)
        sched.add_stream(make_stream("C1", m.vocab, n=24))
    pipe = Pipeline(rank, world, ex, GlooTransport(ex, rank, dist.group.WORLD), sched, dist.group.WORLD)
    out = {}
    for _ in range(ticks):
        a = pipe.tick()
        if rank == world - 1:
            out[int(a["tick"])] = (ex.samp.get(int(a["tick"]), np.zeros(0, np.int32)).tolist(),)
    pipe.drain()
    if rank == world - 1:
        q.put(out)
    if rank == 0:
        q.put({"stats": sched.stats()})
    dist.barrier()
    dist.destroy_process_group()


def _bench_flow_worker(rank, world, port, q):
    """bench.py's multi-rank sequence: preroll ticks, drain, W+K batches scheduled up front and run
    from prepared handles (three times: timed, profiled, attribution), bookkeeping reset, e2e serving
    ticks, drain."""
    import torch.distributed as dist

    from paper_conf_sc_00090d00l25_b200 import gllm
    from paper_conf_sc_00090d00l25_b200.runtime import Pipeline, pack_desc, unpack_desc
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    m = MODELS["C0"].with_layers(2)
    sp = SCHED["C0"].with_(pp_depth=world, num_blocks=256, iterp=2, maxp=64, minp=8)
    lb, le = split_layers(m.n_layers, world)[rank]
    ex = OracleExecutor(m, lb, le, sp.block_size)
    sched = None
    if rank == 0:
        sched = gllm.Sched(sp)
        sched.add_stream(make_stream("C1", m.vocab, n=40))
    pipe = Pipeline(rank, world, ex, GlooTransport(ex, rank, dist.group.WORLD), sched, dist.group.WORLD)
    for _ in range(6):
        pipe.tick()
    pipe.drain()
    batches = []
    for _ in range(5):
        buf = pack_desc(sched.build_batch()) if rank == 0 else None
        batches.append(unpack_desc(pipe._bcast(buf)))
    handles = [ex.prepare(a) for a in batches]
    for a, h in zip(batches, handles):
        pipe.run_batch(a, h)
    for _ in range(2):   # bench's untimed profiled and attribution passes re-run the same batches
        for a, h in zip(batches, handles):
            pipe.run_batch(a, h)
    pipe.pending_samples.clear()
    pipe._expect.clear()
    # e2e leg: a fresh scheduler fast-forwarded to the value window replays the same ticks
    if rank == 0:
        sched = gllm.Sched(sp)
        sched.add_stream(make_stream("C1", m.vocab, n=40))
        for _ in range(int(batches[0]["tick"])):
            sched.build_batch()
        pipe.sched = sched
    replay = [pipe.tick() for _ in range(5)]
    pipe.drain()
    for a, b in zip(replay, batches):
        assert int(a["tick"]) == int(b["tick"]) and int(a["num_tokens"]) == int(b["num_tokens"])
        for key in ("token_ids", "positions", "cu_q", "kv_len", "slot_mapping", "block_table", "sample_idx"):
            if key in a:
                np.testing.assert_array_equal(np.asarray(a[key]), np.asarray(b[key]))
    dist.barrier()
    q.put(rank)
    dist.destroy_process_group()


@pytest.mark.timeout(600)
def test_bench_multi_rank_sequence_does_not_deadlock():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_bench_flow_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    done = sorted(q.get(timeout=500) for _ in range(2))
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert done == [0, 1]


def test_pack_unpack_roundtrip():
    from oracle.scheduler import Scheduler
    st = make_stream("C1", 1000, n=50)
    s = Scheduler(SCHED["C1"].with_(num_blocks=3000), st.requests)
    for _ in range(30):
        b = s.build_batch()
        a = dict(tick=b.tick, P=b.P, D=b.D, num_tokens=b.num_tokens, num_seqs=len(b.cu_q) - 1 if len(b.cu_q) else 0,
                 num_prefill_seqs=len(b.chunks), token_ids=b.token_ids, positions=b.positions,
                 slot_mapping=b.slot_mapping, cu_q=b.cu_q, kv_len=b.kv_len, block_table=b.block_table,
                 sample_idx=b.sample_idx, seq_req_ids=b.seq_req_ids)
        u = unpack_desc(pack_desc(a))
        for k in ("token_ids", "positions", "slot_mapping", "kv_len", "sample_idx", "seq_req_ids"):
            assert np.array_equal(u[k], a[k]), k
        if a["num_seqs"]:
            assert np.array_equal(u["cu_q"], a["cu_q"]) and np.array_equal(u["block_table"], a["block_table"])
        assert u["tick"] == b.tick and u["num_tokens"] == b.num_tokens


def test_split_layers():
    assert split_layers(32, 1) == [(0, 32)]
    assert split_layers(32, 8)[3] == (12, 16)
    assert split_layers(10, 3) == [(0, 4), (4, 7), (7, 10)]


@pytest.mark.timeout(600)
def test_two_stage_pipeline_matches_single_process_oracle():
    ticks = 14
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, 2, port, ticks, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = [q.get(timeout=500) for _ in range(2)]
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    out = next(r for r in res if "stats" not in r)
    # single-process oracle over the same schedule (PP=2 scheduling semantics)
    from oracle import model as om
    from oracle.scheduler import Scheduler
    from oracle.weights import Weights
    m = MODELS["C0"].with_layers(4)
    sp = SCHED["C0"].with_(pp_depth=2, num_blocks=256, iterp=2, maxp=96, minp=8)
    s = Scheduler(sp, make_stream("C1", m.vocab, n=24).requests)
    W = Weights(m)
    cache = om.PagedCache(m, sp.block_size)
    n_checked = 0
    for _ in range(ticks):
        b = s.build_batch()
        if b.num_tokens == 0:
            continue
        r = om.stage_forward(m, W, cache, b, 0, m.n_layers)
        assert out[b.tick][0] == r["sampled"].tolist(), b.tick
        n_checked += len(b.sample_idx)
    assert n_checked > 0
