"""Seeded synthetic request streams (shapes after PAPER.md L234-L236).

Arrivals are in scheduler ticks (reading R4), lengths are drawn in order
(prompt lengths, output lengths, inter-arrival gaps) from
`numpy.random.default_rng(seed)`.  Token ids of request r are drawn from
`default_rng([seed, 7, r])` uniformly in [0, vocab).  Each request carries
prompt_len + output_len - 1 ids: the prompt followed by the teacher-forced
output tokens t1..t_{out-1} (reading R17), so that the id at any position p is
`token_ids[p]`.
"""
from __future__ import annotations

from dataclasses import dataclass, field

import numpy as np

from .configs import STREAMS


@dataclass
class Request:
    req_id: int
    arrival_tick: int
    prompt_len: int
    output_len: int
    token_ids: np.ndarray  # int32 [prompt_len + output_len - 1]


@dataclass
class WarmSeq:
    """A sequence already in decode with `context_len` cached tokens (C4 warm start)."""
    req_id: int
    context_len: int
    remaining_out: int
    token_ids: np.ndarray  # int32 [context_len + remaining_out]


@dataclass
class Stream:
    name: str
    requests: list[Request]
    warm: list[WarmSeq] = field(default_factory=list)
    window: tuple[int, int | None] = (0, None)

    @property
    def last_arrival(self) -> int:
        return max((r.arrival_tick for r in self.requests), default=0)


def _ids(seed: int, req_id: int, n: int, vocab: int) -> np.ndarray:
    rng = np.random.default_rng([seed, 7, req_id])
    return rng.integers(0, vocab, size=n, dtype=np.int64).astype(np.int32)


def _lognormal(rng, n, median, sigma, lo, hi):
    x = rng.lognormal(mean=np.log(median), sigma=sigma, size=n)
    return np.clip(np.rint(x), lo, hi).astype(np.int64)


def _req(seed, rid, arrival, p, o, vocab):
    return Request(rid, int(arrival), int(p), int(o), _ids(seed, rid, int(p) + int(o) - 1, vocab))


def make_stream(name: str, vocab: int, n: int | None = None) -> Stream:
    """Build stream `name` (C0, C0b, C1..C4).  `n` truncates the request count."""
    rec = STREAMS[name]
    kind = rec["kind"]
    if kind == "handmade_c0":
        # tick 0: 8 prompts hitting block edges, output 2; tick 1: one 64-token prompt, output 1
        lens = [1, 15, 16, 17, 31, 32, 33, 100]
        reqs = [_req(0, i, 0, p, 2, vocab) for i, p in enumerate(lens)]
        reqs.append(_req(0, 8, 1, 64, 1, vocab))
        return Stream(name, reqs)
    if kind == "handmade_c0b":
        return Stream(name, [_req(0, 0, 0, 104, 2, vocab)])
    seed = rec["seed"]
    count = rec["n"] if n is None else min(n, rec["n"])
    rng = np.random.default_rng(seed)
    pm, ps, plo, phi = rec["prompt"]
    om, osg, olo, ohi = rec["output"]
    prompts = _lognormal(rng, rec["n"], pm, ps, plo, phi)
    outputs = _lognormal(rng, rec["n"], om, osg, olo, ohi)
    gaps = rng.exponential(1.0 / rec["rate"], size=rec["n"])
    arrivals = np.floor(np.cumsum(gaps)).astype(np.int64)
    warm = []
    base = 0
    if "warm" in rec:
        w = rec["warm"]
        wr = np.random.default_rng([seed, 11])
        ctx = wr.integers(w["context"][0], w["context"][1] + 1, size=w["n"])
        rem = wr.integers(w["remaining"][0], w["remaining"][1] + 1, size=w["n"])
        for i in range(w["n"]):
            warm.append(WarmSeq(i, int(ctx[i]), int(rem[i]),
                                _ids(seed, i, int(ctx[i]) + int(rem[i]), vocab)))
        base = w["n"]
    reqs = [_req(seed, base + i, arrivals[i], prompts[i], outputs[i], vocab) for i in range(count)]
    return Stream(name, reqs, warm, rec.get("window", (0, None)))
