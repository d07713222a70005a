"""Pipeline-parallel driver: one process per stage (P1).

Rank 0 is the driver worker: it owns the Token-Throttling scheduler and the page tables
(L198) and publishes each micro-batch's metadata to every stage before the activations
move (dual-phase transmission, L204).  Every rank runs its layers; hidden states move
stage to stage through `Transport` (NCCL P2P over NVLink in production, gloo in the CPU
tests); the last stage returns the sampled ids to the driver, which retires batch k-PP
before building batch k (at most PP micro-batches in flight, L179).

The executor/transport objects are injected so the host protocol can be tested on CPU
with world_size 2 (tests/test_runtime_gloo.py); the product executor is `GpuExecutor`
(libgllm.so) and the product transport `NcclTransport` (gllm_send_hidden / recv_hidden).
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import gllm

HDR = 10  # tick, P, D, T, S, NP, maxblk, ns, num_prefill_tokens, reserved


def split_layers(n_layers: int, world: int):
    """Equal contiguous layer ranges [lb, le) per stage."""
    base, rem = divmod(n_layers, world)
    out, b = [], 0
    for s in range(world):
        e = b + base + (1 if s < rem else 0)
        out.append((b, e))
        b = e
    return out


def fill_warm(stage, sched_cfg, warm) -> None:
    """Warm-start KV of a warm decode set (C4, O4 values): the blocks each warm sequence holds are
    those the scheduler allocates at add_warm (lowest first, in list order, before any request), so a
    scheduler holding only the warm set reproduces them on every rank."""
    if not warm:
        return
    s = gllm.Sched(sched_cfg)
    for w in warm:
        s.add_warm(w.req_id, w.context_len, w.remaining_out, w.token_ids)
    rows = [s.seq_blocks(w.req_id) for w in warm]
    bt = np.full((len(rows), max(len(r) for r in rows)), -1, np.int32)
    for i, r in enumerate(rows):
        bt[i, :len(r)] = r
    stage.fill_warm_kv([w.req_id for w in warm], [w.context_len for w in warm], bt)


def pack_desc(d) -> np.ndarray:
    """Flatten a BatchDesc (or its to_numpy() dict) into one int32 buffer for the broadcast."""
    a = d.to_numpy() if hasattr(d, "to_numpy") else d
    T, S = int(a["num_tokens"]), int(a["num_seqs"])
    bt = np.asarray(a["block_table"], np.int32).reshape(S, -1) if S else np.zeros((0, 0), np.int32)
    ns = int(np.asarray(a["sample_idx"]).shape[0])
    npt = int(a["cu_q"][a["num_prefill_seqs"]]) if S else 0
    hdr = np.array([a["tick"], a.get("P", 0), a.get("D", 0), T, S, a["num_prefill_seqs"], bt.shape[1] if S else 0,
                    ns, npt, 0], np.int64).astype(np.int32)
    parts = [hdr, a["token_ids"], a["positions"], a["slot_mapping"], a["cu_q"] if S else np.zeros(0, np.int32),
             a["kv_len"], bt.ravel(), a["sample_idx"],
             np.asarray(a["seq_req_ids"], np.int64).view(np.int32)]
    return np.concatenate([np.asarray(p, np.int32).ravel() for p in parts])


def unpack_desc(buf: np.ndarray) -> dict:
    buf = np.asarray(buf, np.int32)
    tick, P, D, T, S, NP, maxblk, ns, npt, _ = [int(v) for v in buf[:HDR]]
    o = HDR

    def take(n):
        nonlocal o
        r = buf[o:o + n]
        o += n
        return r
    ids, pos, slots = take(T), take(T), take(T)
    cu = take(S + 1) if S else np.zeros(0, np.int32)
    kvl = take(S)
    bt = take(S * maxblk).reshape(S, maxblk) if S else np.zeros((0, 0), np.int32)
    samp = take(ns)
    seq = take(2 * S).copy().view(np.int64)
    return dict(tick=tick, P=P, D=D, num_tokens=T, num_seqs=S, num_prefill_seqs=NP, token_ids=ids,
                positions=pos, slot_mapping=slots, cu_q=cu, kv_len=kvl, block_table=bt, sample_idx=samp,
                seq_req_ids=seq)


class GpuExecutor:
    """Product executor: a gllm.Stage on this rank's GPU; buffers are torch CUDA tensors."""

    def __init__(self, stage: "gllm.Stage", device, max_tokens, hidden, pp=1):
        import torch
        self.torch = torch
        self.stage = stage
        self.dev = device
        self.compute = torch.cuda.Stream(device=device)
        self.comm = torch.cuda.Stream(device=device)
        self.hin = [torch.empty((max_tokens, hidden), dtype=torch.float32, device=device) for _ in range(2)]
        self.hout = [torch.empty((max_tokens, hidden), dtype=torch.float32, device=device) for _ in range(2)]
        # sampled ids of batch k are read PP-1 (last stage, world > 1) or PP (one-GPU emulation) ticks
        # later, so the ring holds more than PP batches
        self.nsamp = max(4, 2 * pp + 2)
        self.samp = [torch.empty((max(stage.max_seqs, 1),), dtype=torch.int32, device=device)
                     for _ in range(self.nsamp)]
        self.samp_host = [torch.empty((max(stage.max_seqs, 1),), dtype=torch.int32, pin_memory=True)
                          for _ in range(self.nsamp)]
        self.samp_ev = [torch.cuda.Event() for _ in range(self.nsamp)]
        self.fwd_ev = [torch.cuda.Event() for _ in range(2)]
        self.recv_ev = [torch.cuda.Event() for _ in range(2)]
        self.send_ev = [torch.cuda.Event() for _ in range(2)]
        self.keep = {}

    def prepare(self, a: dict) -> int:
        desc, keep = gllm.desc_from_arrays(a)
        h = self.stage.prepare(desc, self.compute.cuda_stream)
        self.keep[h] = keep
        return h

    def release(self, h):
        self.stage.release(h)
        self.keep.pop(h, None)

    peer_in = False    # hidden_in arrives in this stage's peer ring (PeerTransport)
    peer_out = False   # hidden_out goes straight into the next stage's peer ring

    def forward(self, h, k, T, is_first, is_last, ns):
        i = k & 1
        cs = self.compute.cuda_stream
        hin = 0
        if not is_first:
            if self.peer_in:   # stream waits for the sender's release flag of tick k
                hin = self.stage.peer_ring_recv(k, cs)
            else:
                self.compute.wait_event(self.recv_ev[i])
                hin = self.hin[i].data_ptr()
        if not is_last and self.peer_out:
            self.stage.forward_prepared_peer(h, k, hin, cs)
        else:
            if not is_last:
                self.compute.wait_event(self.send_ev[i])   # send k-2 finished reading hout[i]
            j = k % self.nsamp
            self.stage.forward_prepared(h, hin, 0 if is_last else self.hout[i].data_ptr(),
                                        self.samp[j].data_ptr() if is_last else 0, cs)
        self.fwd_ev[i].record(self.compute)
        if is_last and ns:
            j = k % self.nsamp
            with self.torch.cuda.stream(self.compute):
                self.samp_host[j][:ns].copy_(self.samp[j][:ns], non_blocking=True)
            self.samp_ev[j].record(self.compute)

    def sampled(self, k, ns) -> np.ndarray:
        j = k % self.nsamp
        self.samp_ev[j].synchronize()
        return self.samp_host[j][:ns].numpy().copy()


class NcclTransport:
    """Hidden-state hand-off through gllm_send_hidden / gllm_recv_hidden (NCCL P2P over NVLink)."""

    def __init__(self, ex: GpuExecutor, rank, world):
        self.ex, self.rank, self.world = ex, rank, world

    def recv(self, k, T):
        ex = self.ex
        i = k & 1
        ex.comm.wait_event(ex.fwd_ev[i])      # forward k-2 finished reading hin[i]
        ex.stage.recv_hidden(ex.hin[i].data_ptr(), T, self.rank - 1, ex.comm.cuda_stream)
        ex.recv_ev[i].record(ex.comm)

    def send(self, k, T):
        ex = self.ex
        i = k & 1
        ex.comm.wait_event(ex.fwd_ev[i])
        ex.stage.send_hidden(ex.hout[i].data_ptr(), T, self.rank + 1, ex.comm.cuda_stream)
        ex.send_ev[i].record(ex.comm)


class PeerTransport:
    """Fused hand-off over peer memory (include/gllm.h gllm_peer_*): stage s+1 exports a ring of
    receive slots, stage s maps it and its last residual GEMM writes into the slot; ready flags
    (sender -> receiver) and slot credits (receiver -> sender) make the hand-off stream-ordered and
    flow-controlled on the devices, so recv/send are no-ops here.  depth = 2 PP slots.

    Handle exchange over the (gloo) metadata group: rank s+1 sends its ring handle to rank s; rank s
    maps it and sends back the handle of its slot credits, which rank s+1 maps."""

    def __init__(self, ex: GpuExecutor, rank, world, group, pp=None):
        import torch
        import torch.distributed as dist
        self.ex, self.rank, self.world = ex, rank, world
        depth = 2 * (pp or world)

        def send(b: bytes, dst):
            dist.send(torch.frombuffer(bytearray(b), dtype=torch.uint8), dst, group=group)

        def recv(src) -> bytes:
            t = torch.empty(128, dtype=torch.uint8)
            dist.recv(t, src, group=group)
            return bytes(t.numpy().tobytes())
        if rank > 0:
            send(ex.stage.peer_ring_create(depth), rank - 1)
            ex.peer_in = True
        if rank < world - 1:
            send(ex.stage.peer_ring_open(recv(rank + 1)), rank + 1)
            ex.peer_out = True
        if rank > 0:
            ex.stage.peer_credit_open(recv(rank - 1))

    def recv(self, k, T):
        pass

    def send(self, k, T):
        pass


class _NullTransport:
    """Stage emulation on one GPU: the hidden input buffers keep synthetic data, nothing is sent."""

    def recv(self, k, T):
        pass

    def send(self, k, T):
        pass


class Pipeline:
    """The per-rank tick loop.  `meta` is a torch.distributed group (gloo) for metadata and
    sampled ids; None when world == 1."""

    def __init__(self, rank, world, executor, transport=None, sched=None, meta=None, pp=None, stage=None):
        """`stage` (emulation, world == 1): run only pipeline stage `stage` of `pp` on this GPU, with
        synthetic hidden inputs -- the per-stage work of a PP=pp deployment measured on one GPU."""
        self.rank, self.world = rank, world
        self.ex, self.tr, self.sched, self.meta = executor, transport, sched, meta
        self.pp = pp or world
        s, n = (rank, world) if stage is None else (stage, self.pp)
        self.is_first, self.is_last = s == 0, s == n - 1
        if self.tr is None and not (self.is_first and self.is_last) and world == 1:
            self.tr = _NullTransport()
        self.pending_samples = {}   # tick -> ns (last stage)
        self._expect = {}           # tick -> ns (driver): sampled ids owed by the last stage
        self.tokens = 0
        self.samples = 0

    # ---- metadata phase ---------------------------------------------------------
    def _bcast(self, buf: np.ndarray | None) -> np.ndarray:
        if self.world == 1:
            return buf
        import torch
        import torch.distributed as dist
        n = torch.tensor([0 if buf is None else buf.shape[0]], dtype=torch.int64)
        dist.broadcast(n, 0, group=self.meta)
        t = torch.from_numpy(buf) if self.rank == 0 else torch.empty(int(n[0]), dtype=torch.int32)
        dist.broadcast(t, 0, group=self.meta)
        return t.numpy()

    def build_and_publish(self):
        """Driver builds the next micro-batch (after retiring k-PP) and publishes it to every stage."""
        buf = None
        if self.rank == 0:
            k = self.sched.stats()["tick"]
            j = k - self.pp
            if j >= 0 and j in self._expect:
                ns = self._expect.pop(j)
                self.sched.retire_batch(j, self._recv_sampled(j, ns))
            d = self.sched.build_batch()
            buf = pack_desc(d)
            self._expect[int(d.tick)] = int(d.num_samples)
        return unpack_desc(self._bcast(buf))

    def _recv_sampled(self, j, ns):
        if ns == 0:
            return np.zeros(0, np.int32)
        if self.world == 1:
            return self.ex.sampled(j, ns) if self.is_last else None
        import torch
        import torch.distributed as dist
        t = torch.empty(ns, dtype=torch.int32)
        dist.recv(t, self.world - 1, group=self.meta)
        return t.numpy()

    def _send_sampled_upto(self, k):
        """Last stage: return sampled ids of batch j = k - PP + 1 to the driver (after its tick-k work)."""
        j = k - self.pp + 1
        if self.world == 1 or j < 0 or j not in self.pending_samples:
            return
        ns = self.pending_samples.pop(j)
        if ns == 0:
            return
        import torch
        import torch.distributed as dist
        dist.send(torch.from_numpy(self.ex.sampled(j, ns)), 0, group=self.meta)

    # ---- activation phase ---------------------------------------------------------
    def run_batch(self, a: dict, handle=None):
        k, T, ns = int(a["tick"]), int(a["num_tokens"]), int(np.asarray(a["sample_idx"]).shape[0])
        own = handle is None
        if T > 0:
            h = self.ex.prepare(a) if own else handle
            if not self.is_first:
                self.tr.recv(k, T)
            self.ex.forward(h, k, T, self.is_first, self.is_last, ns)
            if not self.is_last:
                self.tr.send(k, T)
            if own:
                self.ex.release(h)
        self.tokens += T
        if self.is_last:
            self.pending_samples[k] = ns if T > 0 else 0
            self.samples += ns
        return k

    def tick(self):
        """One serving tick: schedule + publish (rank 0), then this rank's stage work."""
        a = self.build_and_publish()
        k = self.run_batch(a)
        if self.is_last and self.world > 1:
            self._send_sampled_upto(k)
        return a

    def drain(self):
        """After the last tick t: the driver collects (and records) the sampled ids of batch
        t - PP + 1 that the last stage already sent, so no send is left unmatched."""
        if self.world == 1:
            return
        if self.rank == 0:
            t = self.sched.stats()["tick"] - 1
            j = t - self.pp + 1
            if j >= 0 and j in self._expect:
                ns = self._expect.pop(j)
                self.sched.retire_batch(j, self._recv_sampled(j, ns))
