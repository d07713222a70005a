"""Hand-worked scheduler traces under tests/golden/ (W1, P1, P2, S1, WS1) and their setups.

Each golden file was derived by hand from the readings R1-R21 and PAPER.md
(Eq.3 L169 + threshold L165, Eq.4, paged KV L136, preemption L127/L165/L325, the
Sarathi-Serve comparator L81/L125/L310); none was written by a program.  The files carry the
derivation in their headers.  `compare()` checks a canonical trace (oracle.scheduler.trace_bytes
layout == gllm_sched_trace) against a golden row, so the same goldens pin the oracle
(tests/test_oracle_scheduler.py) and the C++ scheduler (tests/test_sched_parity.py).
"""
import os

import numpy as np

from workloads.configs import SchedParams
from workloads.streams import Request, Stream, WarmSeq

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def _req(rid, arrival, prompt, out):
    return Request(rid, arrival, prompt, out, (np.arange(prompt + out - 1, dtype=np.int32) * 7 + rid) % 500)


def _warm(rid, ctx, rem):
    return WarmSeq(rid, ctx, rem, (np.arange(ctx + rem, dtype=np.int32) * 3 + rid) % 500)


SMALL = dict(pp_depth=1, block_size=4, num_blocks=4, iterp=1, maxp=64, minp=1, kvthresh_num=0,
             kvthresh_den=4, max_seqs=8)

CASES = {
    "w1_trace.txt": (SchedParams(iterp=2, maxp=16, minp=2, kvthresh_num=1, kvthresh_den=4, pp_depth=2,
                                 num_blocks=16, block_size=4),
                     Stream("W1", [_req(0, 0, 12, 3), _req(1, 1, 5, 2)])),
    "p1_preempt_order.txt": (SchedParams(**SMALL),
                             Stream("P1", [_req(0, 0, 4, 3), _req(1, 0, 2, 3), _req(2, 0, 2, 3), _req(3, 0, 2, 3)])),
    "p2_preempt_inflight.txt": (SchedParams(**{**SMALL, "pp_depth": 2}),
                                Stream("P2", [_req(0, 0, 3, 4), _req(1, 0, 2, 4), _req(2, 0, 2, 4),
                                              _req(3, 0, 2, 4)])),
    "s1_sarathi.txt": (SchedParams(policy=1, token_budget=6, pp_depth=2, block_size=4, num_blocks=16,
                                   kvthresh_num=0, kvthresh_den=4, max_seqs=8),
                       Stream("S1", [_req(0, 0, 8, 3), _req(1, 0, 3, 2), _req(2, 3, 9, 2)])),
    "ws1_warm.txt": (SchedParams(pp_depth=2, block_size=4, num_blocks=8, iterp=1, maxp=64, minp=1,
                                 kvthresh_num=1, kvthresh_den=4, max_seqs=8),
                     Stream("WS1", [_req(2, 0, 6, 2)], warm=[_warm(0, 5, 2), _warm(1, 8, 1)])),
}


def parse(name):
    rows = []
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            cols = [x.strip() for x in line.split("|")]
            if len(cols) == 6:       # W1 predates the victims column
                cols.insert(5, "-")
            tick, pd, ch, dec, slots, vic, free = cols
            P, D = map(int, pd.split())
            rows.append(dict(
                tick=int(tick), P=P, D=D,
                chunks=[] if ch == "-" else [tuple(map(int, c.split(":"))) for c in ch.split(",")],
                decodes=[] if dec == "-" else [tuple(map(int, d.split(":"))) for d in dec.split(",")],
                slots=[] if slots == "-" else list(map(int, slots.split(","))),
                victims=[] if vic == "-" else list(map(int, vic.split(","))),
                free=int(free)))
    return rows


def decode_trace(buf: bytes) -> dict:
    """Fields of one canonical trace record (DESIGN.md §3 layout)."""
    v = np.frombuffer(buf, np.int64)
    tick, P, D, _rd, _wp, _f0, f1, nc, nd, npre, nal, T, ns = (int(x) for x in v[:13])
    o = 13
    ch = [tuple(int(x) for x in v[o + 3 * i:o + 3 * i + 3]) for i in range(nc)]
    o += 3 * nc
    dec = [tuple(int(x) for x in v[o + 2 * i:o + 2 * i + 2]) for i in range(nd)]
    o += 2 * nd
    vic = [int(x) for x in v[o:o + npre]]
    o += npre + 2 * nal
    slots = [int(x) for x in v[o:o + T]]
    return dict(tick=tick, P=P, D=D, chunks=ch, decodes=dec, slots=slots, victims=vic, free=f1)


def compare(traces, name):
    gold = parse(name)
    got = [decode_trace(t) for t in traces]
    assert len(got) == len(gold), (name, len(got), len(gold))
    for g, e in zip(got, gold):
        assert g == e, f"{name} tick {e['tick']}:\n got  {g}\n want {e}"
