"""Stream/event ordering of the product executor + NCCL transport (runtime.GpuExecutor,
runtime.NcclTransport) on CPU, with a recording fake stage and fake CUDA streams/events.

The hand-off double-buffers hidden_in / hidden_out (2 buffers each) across the compute and comm
streams; every read and write of a buffer must be ordered after the previous use of that buffer
(activations move stage to stage; L179: up to PP micro-batches in flight).
The fake records each device operation with a vector clock; happens-before follows stream order
and event record -> wait edges exactly as CUDA defines them (a wait captures the event's most
recent record).  The check fails if any wait_event of the executor or transport is dropped."""
import numpy as np
import pytest

from paper_conf_sc_00090d00l25_b200 import runtime


class Clock:
    def __init__(self, n):
        self.v = [0] * n

    def merge(self, o):
        self.v = [max(a, b) for a, b in zip(self.v, o.v)]

    def copy(self):
        c = Clock(len(self.v))
        c.v = list(self.v)
        return c


class FakeStream:
    all = []

    def __init__(self, n_streams=2):
        self.id = len(FakeStream.all)
        FakeStream.all.append(self)
        self.clock = Clock(8)
        self.cuda_stream = 1000 + self.id

    def op(self):
        self.clock.v[self.id] += 1
        return self.clock.copy()

    def wait_event(self, ev):
        if ev.snap is not None:
            self.clock.merge(ev.snap)


class FakeEvent:
    def __init__(self):
        self.snap = None

    def record(self, stream):
        self.snap = stream.op()

    def synchronize(self):
        pass


def hb(a, b):
    """operation a happens before operation b (vector clocks)."""
    return all(x <= y for x, y in zip(a.v, b.v)) and a.v != b.v


class Buf:
    n = 0

    def __init__(self):
        Buf.n += 1
        self.ptr = Buf.n * 4096

    def data_ptr(self):
        return self.ptr


class FakeStage:
    """Records (op, buffer, access, clock) for every device operation the runtime enqueues."""

    def __init__(self):
        self.log = []
        self.max_seqs = 8

    def _stream(self, handle):
        return next(s for s in FakeStream.all if s.cuda_stream == handle)

    def forward_prepared(self, h, hin, hout, samp, cs):
        c = self._stream(cs).op()
        self.log.append(("fwd", h, hin, hout, c))

    def recv_hidden(self, ptr, T, src, cs):
        self.log.append(("recv", ptr, self._stream(cs).op()))

    def send_hidden(self, ptr, T, dst, cs):
        self.log.append(("send", ptr, self._stream(cs).op()))


def make_executor(stage):
    ex = object.__new__(runtime.GpuExecutor)
    ex.stage = stage
    ex.compute, ex.comm = FakeStream(), FakeStream()
    ex.hin = [Buf(), Buf()]
    ex.hout = [Buf(), Buf()]
    ex.nsamp = 4
    ex.samp = [Buf() for _ in range(4)]
    ex.fwd_ev = [FakeEvent() for _ in range(2)]
    ex.recv_ev = [FakeEvent() for _ in range(2)]
    ex.send_ev = [FakeEvent() for _ in range(2)]
    ex.samp_ev = [FakeEvent() for _ in range(4)]
    return ex


def accesses(stage):
    """(clock, buffer, 'r'|'w', label) per device operation."""
    out = []
    for e in stage.log:
        if e[0] == "fwd":
            _, h, hin, hout, c = e
            if hin:
                out.append((c, hin, "r", f"fwd{h}"))
            if hout:
                out.append((c, hout, "w", f"fwd{h}"))
        elif e[0] == "recv":
            out.append((e[2], e[1], "w", "recv"))
        else:
            out.append((e[2], e[1], "r", "send"))
    return out


def check_no_races(stage):
    acc = accesses(stage)
    n = 0
    for i in range(len(acc)):
        for j in range(i + 1, len(acc)):
            ci, bi, mi, li = acc[i]
            cj, bj, mj, lj = acc[j]
            if bi != bj or (mi == "r" and mj == "r"):
                continue
            # program order issued i before j: the device must order them the same way
            assert hb(ci, cj), f"race on buffer {bi}: {li} ({mi}) vs {lj} ({mj})"
            n += 1
    return n


@pytest.mark.parametrize("role", ["first", "middle", "last"])
def test_nccl_transport_orders_every_buffer_reuse(role):
    FakeStream.all = []
    stage = FakeStage()
    ex = make_executor(stage)
    tr = runtime.NcclTransport(ex, rank=1, world=3)
    is_first, is_last = role == "first", role == "last"
    for k in range(9):   # the Pipeline.run_batch order: recv, forward, send
        if not is_first:
            tr.recv(k, 100)
        ex.forward(k, k, 100, is_first, is_last, 0)
        if not is_last:
            tr.send(k, 100)
    pairs = check_no_races(stage)
    assert pairs >= 8
    # and the producer -> consumer edges themselves
    log = stage.log
    for k in range(9):
        fwd = next(e for e in log if e[0] == "fwd" and e[1] == k)
        if not is_first:
            rcv = [e for e in log if e[0] == "recv"][k]
            assert rcv[1] == fwd[2] and hb(rcv[2], fwd[4])        # recv(k) -> forward(k)
        if not is_last:
            snd = [e for e in log if e[0] == "send"][k]
            assert snd[1] == fwd[3] and hb(fwd[4], snd[2])        # forward(k) -> send(k)


def test_checker_catches_a_dropped_wait():
    # the same loop with the transport's wait on the forward event removed must be flagged
    FakeStream.all = []
    stage = FakeStage()
    ex = make_executor(stage)
    tr = runtime.NcclTransport(ex, rank=1, world=3)
    orig = ex.comm.wait_event
    ex.comm.wait_event = lambda ev: None
    with pytest.raises(AssertionError):
        for k in range(6):
            tr.recv(k, 100)
            ex.forward(k, k, 100, False, False, 0)
            tr.send(k, 100)
        check_no_races(stage)
    ex.comm.wait_event = orig
