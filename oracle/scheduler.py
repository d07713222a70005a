"""ORACLE (test infrastructure only) -- canonical Token-Throttling scheduler + block manager.

Follows PAPER.md step by step, under the readings R1-R18 listed in DESIGN.md §3
(= SURVEY.md §8(c) O1):

  * Eq.3 + threshold (L165-L169 §3.1.3): prefill token count #P, computed in
    exact integer arithmetic (R10):
        P = 0                                   if WP == 0 or KV_free < KV_thresh
        P = min(max(min(WP // T, cap), MinP), WP)
        cap = MaxP * (free*den - num*N) // (N * (den - num))
  * Eq.4 (L179-L183 §3.2.1): #D = ceil(RD / PP_depth) (R6); schedule all ready
    decodes if fewer remain, else exactly #D.
  * Decoupled merge (L125 §2.5, L131-L143 §3): #P and #D are chosen
    independently and merged into one micro-batch, prefill chunks first (R15).
  * Chunked prefill + CPP (L81, L92, L212): FCFS chunks; a prompt may have
    chunks in several in-flight micro-batches (R13).
  * Paged KV (L136 Fig.6): blocks allocated at schedule time, lowest free
    block first (R8), decode allocation before prefill (R9); freed when the
    request finishes at retire (R3); at most PP_depth micro-batches in flight
    (R1, L179); preemption by recompute only when a decode finds no free block
    (R14, L127/L165).
  * slot(t) = block_table[seq(t)][pos // bs] * bs + pos % bs (O2).

Pinned by (tests/test_oracle_scheduler.py): the hand-worked Eq.3/Eq.4 values
E1-E9 and the full trace W1 (tests/golden/w1_trace.txt), the C0 / C0b traces
(SURVEY.md §8(d), Appendix A.2), and invariants (sum of #P = prompt tokens,
live-slot uniqueness, blocks freed exactly once, KV_free bookkeeping).
"""
from __future__ import annotations

import heapq
import struct
from dataclasses import dataclass, field

import numpy as np


def throttle_prefill(cfg, wp: int, free: int) -> int:
    """#P by Eq.3 with the L165 threshold, exact integer reading R10.

    Ablations of §4.5 (L305-L310, Fig. 15): policy 2 "w/o WT" drops the #WP/#T term of Eq.3
    (R19); policy 3 "w/o UT" is Eq.1 (L153) with the L165 threshold kept (R20)."""
    n, num, den = cfg.num_blocks, cfg.kvthresh_num, cfg.kvthresh_den
    if wp == 0 or free * den < num * n:          # KV_free < KV_thresh: suspend prefill (L165)
        return 0
    cap = (cfg.maxp * (free * den - num * n)) // (n * (den - num))   # MaxP*(KVfree-th)/(1-th)
    policy = getattr(cfg, "policy", 0)
    if policy == 2:                              # w/o WT: max(MaxP*(KVfree-th)/(1-th), MinP)
        return min(max(cap, cfg.minp), wp)
    if policy == 3:                              # w/o UT: Eq.1 = min(max(WP/T, MinP), MaxP)
        return min(max(wp // cfg.iterp, cfg.minp), cfg.maxp, wp)
    return min(max(min(wp // cfg.iterp, cap), cfg.minp), wp)         # Eq.3, capped by WP (R11)


def chunk_cost(s: int, c: int, a: int) -> int:
    """Reading R21 (policy 4, context-aware Token Throttling; PAPER.md L354 future work): the
    token-equivalent cost of a prefill chunk of c tokens at offset s = its c tokens of linear
    work plus its causal (query, key) pairs c*s + c(c+1)/2 (query s+j sees keys 0..s+j), in units
    of `a` pairs per token, rounded down."""
    pairs = sum(s + j + 1 for j in range(c))
    return c + pairs // a


def throttle_decode(cfg, rd: int) -> int:
    """#D = ceil(#RD / #PP_depth) (Eq.4; ceil per reading R6)."""
    return -(-rd // cfg.pp_depth)


@dataclass
class _Req:
    req_id: int
    arrival: int
    orig_len: int
    output_len: int
    ids: np.ndarray
    prefill_len: int = 0
    sched_prompt: int = 0
    done_prompt: int = 0
    gen: int = 0
    blocks: list = field(default_factory=list)
    inflight: int = 0
    ready_tick: int = 0
    finished: bool = False

    @property
    def decode_phase(self) -> bool:
        return (not self.finished) and self.done_prompt == self.prefill_len

    @property
    def waiting(self) -> bool:
        return (not self.finished) and self.sched_prompt < self.prefill_len


@dataclass
class Batch:
    """Oracle mirror of `gllm_batch_desc` (include/gllm.h)."""
    tick: int
    P: int
    D: int
    chunks: list            # (req_id, start, length, completes_prompt)
    decodes: list           # (req_id, pos)
    token_ids: np.ndarray
    positions: np.ndarray
    slot_mapping: np.ndarray
    cu_q: np.ndarray
    kv_len: np.ndarray
    block_table: np.ndarray  # [S, max_blocks_per_seq], -1 padded
    sample_idx: np.ndarray
    seq_req_ids: np.ndarray
    preempted: list
    allocs: list             # (req_id, block) in allocation order
    stats: tuple             # (RD, WP, free_before, free_after)

    @property
    def num_tokens(self) -> int:
        return int(self.token_ids.shape[0])

    @property
    def num_prefill_tokens(self) -> int:
        return int(sum(c[2] for c in self.chunks))


class Scheduler:
    """Canonical scheduler; `build_batch()` is one tick (R1-R18)."""

    def __init__(self, cfg, requests=(), warm=()):
        if not (0 <= cfg.kvthresh_num < cfg.kvthresh_den):
            raise ValueError("KV_thresh must be in [0, 1)")
        self.cfg = cfg
        self.tick = 0
        self.free = list(range(cfg.num_blocks))
        heapq.heapify(self.free)
        self.pending = sorted(requests, key=lambda r: (r.arrival_tick, r.req_id))
        self.next_arrival = 0
        self.admitted: list[_Req] = []
        self.inflight: dict[int, Batch] = {}
        self.finished: list[_Req] = []
        self.preemptions = 0
        self.sampled: dict[int, list] = {}
        for w in warm:
            self._add_warm(w)

    # -- block pool ------------------------------------------------------
    def _alloc(self, r, allocs):
        b = heapq.heappop(self.free)          # lowest-numbered free block (R8)
        r.blocks.append(b)
        allocs.append((r.req_id, b))

    def _release(self, r):
        for b in r.blocks:
            heapq.heappush(self.free, b)
        r.blocks = []

    def _add_warm(self, w):
        # warm decode sequence: context_len cached tokens, next decode at pos context_len
        r = _Req(w.req_id, -1, w.context_len, w.remaining_out + 1, w.token_ids)
        r.prefill_len = r.sched_prompt = r.done_prompt = w.context_len
        r.gen = 1
        bs = self.cfg.block_size
        for _ in range(-(-w.context_len // bs)):
            self._alloc(r, [])
        self.admitted.append(r)

    # -- retire (R1-R3) --------------------------------------------------------
    def _retire(self, b: Batch, sampled=None):
        touched = []
        by_id = {r.req_id: r for r in self.admitted}
        for (rid, start, c, _done) in b.chunks:
            r = by_id[rid]
            r.done_prompt += c
            r.inflight -= 1
            if r.done_prompt == r.prefill_len:   # prompt completes: first output token (R2)
                r.gen += 1
                r.ready_tick = self.tick
            touched.append(r)
        for (rid, _pos) in b.decodes:
            r = by_id[rid]
            r.gen += 1
            r.inflight -= 1
            r.ready_tick = self.tick
            touched.append(r)
        if sampled is not None:
            self.sampled[b.tick] = list(sampled)
        for r in touched:
            if not r.finished and r.gen >= r.output_len:   # fixed output length (R3)
                r.finished = True
                self._release(r)
                self.finished.append(r)
        self.admitted = [r for r in self.admitted if not r.finished]

    def retire(self, tick, sampled=None):
        b = self.inflight.pop(tick, None)
        if b is not None:
            self._retire(b, sampled)

    # -- preemption (R14) ------------------------------------------------------
    def _preempt_victim(self, exclude):
        cands = [r for r in self.admitted
                 if r.blocks and r.inflight == 0 and r.req_id not in exclude]
        if not cands:
            return None
        v = max(cands, key=lambda r: (r.arrival, r.req_id))
        self._release(v)
        v.prefill_len = v.orig_len + v.gen
        v.sched_prompt = v.done_prompt = 0
        self.preemptions += 1
        return v

    # -- one tick ----------------------------------------------------------------
    def build_batch(self, auto_retire=True) -> Batch:
        cfg, bs, k = self.cfg, self.cfg.block_size, self.tick
        if auto_retire:
            self.retire(k - cfg.pp_depth)                       # R1
        while (self.next_arrival < len(self.pending)
               and self.pending[self.next_arrival].arrival_tick <= k):   # R4
            q = self.pending[self.next_arrival]
            r = _Req(q.req_id, q.arrival_tick, q.prompt_len, q.output_len, q.token_ids)
            r.prefill_len = q.prompt_len
            self.admitted.append(r)
            self.next_arrival += 1
        # stats (R5)
        rd = sum(1 for r in self.admitted if r.decode_phase)
        wp = sum(r.prefill_len - r.sched_prompt for r in self.admitted if r.waiting)
        free0 = len(self.free)
        allocs, preempted, selected = [], [], set()
        # decode selection (Eq.4, R6-R9, R14)
        if cfg.policy == 1:   # Sarathi-Serve: every ready decode
            d_cnt = rd
        else:
            d_cnt = throttle_decode(cfg, rd)
        ready = sorted((r for r in self.admitted if r.decode_phase and r.inflight == 0),
                       key=lambda r: (r.ready_tick, r.arrival, r.req_id))
        decodes = []
        for r in ready[:min(d_cnt, len(ready))]:
            if not r.decode_phase:          # preempted earlier in this tick
                continue
            pos = r.orig_len + r.gen - 1
            if len(r.blocks) * bs <= pos:
                if not self.free:
                    v = self._preempt_victim(selected | {r.req_id})
                    if v is None:
                        continue
                    preempted.append(v.req_id)
                self._alloc(r, allocs)
            decodes.append((r, pos))
            selected.add(r.req_id)
        # prefill count (Eq.3 + L165, R10-R12)
        if cfg.policy == 1:
            p_cnt = min(max(cfg.token_budget - len(decodes), 0), wp)
        else:
            p_cnt = throttle_prefill(cfg, wp, free0)
        # prefill selection (R13)
        running = sum(1 for r in self.admitted if r.blocks or r.sched_prompt > 0)
        p_left = p_cnt
        chunks = []
        for r in sorted((r for r in self.admitted if r.waiting),
                        key=lambda r: (r.arrival, r.req_id)):
            if p_left == 0:
                break
            fresh = not r.blocks and r.sched_prompt == 0
            if fresh and running >= cfg.max_seqs:
                continue
            remaining = r.prefill_len - r.sched_prompt
            capacity = (len(r.blocks) + len(self.free)) * bs - r.sched_prompt
            if cfg.policy == 4:
                # R21: the longest chunk whose cost fits the budget left (linear scan from 0)
                a, s0 = cfg.attn_pairs_per_token, r.sched_prompt
                c, pairs = 0, 0
                while c < min(remaining, capacity):
                    nxt = pairs + (s0 + c + 1)  # query s0+c attends keys 0..s0+c
                    if (c + 1) + nxt // a > p_left:
                        break
                    c, pairs = c + 1, nxt
                if c == 0 and not chunks and capacity > 0:
                    c, pairs = 1, s0 + 1        # progress: at least one token per tick
                cost = c + pairs // a
            else:
                c = min(remaining, p_left, capacity)
                cost = c
            if c <= 0:
                break
            need = -(-(r.sched_prompt + c) // bs) - len(r.blocks)
            for _ in range(need):
                self._alloc(r, allocs)
            if fresh:
                running += 1
            chunks.append((r, r.sched_prompt, c))
            r.sched_prompt += c
            p_left = max(p_left - cost, 0)
            if c < remaining:                   # budget spent or KV capacity reached (R13)
                break
        # layout (R15): prefill chunks first, then decodes
        tok, pos_l, slot, cu, kvl, samp, seq_ids, rows = [], [], [], [0], [], [], [], []
        chunk_rec = []
        for (r, s, c) in chunks:
            for p in range(s, s + c):
                tok.append(int(r.ids[p]))
                pos_l.append(p)
                slot.append(r.blocks[p // bs] * bs + p % bs)     # O2
            cu.append(cu[-1] + c)
            kvl.append(s + c)
            completes = (s + c == r.prefill_len)
            if completes:
                samp.append(cu[-1] - 1)
            seq_ids.append(r.req_id)
            rows.append(list(r.blocks[: -(-(s + c) // bs)]))
            chunk_rec.append((r.req_id, s, c, completes))
            r.inflight += 1
        dec_rec = []
        for (r, p) in decodes:
            tok.append(int(r.ids[p]))
            pos_l.append(p)
            slot.append(r.blocks[p // bs] * bs + p % bs)
            cu.append(cu[-1] + 1)
            kvl.append(p + 1)
            samp.append(cu[-1] - 1)
            seq_ids.append(r.req_id)
            rows.append(list(r.blocks[: -(-(p + 1) // bs)]))
            dec_rec.append((r.req_id, p))
            r.inflight += 1
        maxblk = max((len(x) for x in rows), default=0)
        bt = np.full((len(rows), maxblk), -1, dtype=np.int32)
        for i, x in enumerate(rows):
            bt[i, :len(x)] = x
        b = Batch(k, p_cnt, d_cnt, chunk_rec, dec_rec,
                  np.array(tok, np.int32), np.array(pos_l, np.int32), np.array(slot, np.int32),
                  np.array(cu, np.int32), np.array(kvl, np.int32), bt,
                  np.array(samp, np.int32), np.array(seq_ids, np.int64),
                  preempted, allocs, (rd, wp, free0, len(self.free)))
        self.inflight[k] = b
        self.tick += 1
        return b

    def done(self) -> bool:
        # every request finished; remaining in-flight batches are then empty
        return self.next_arrival >= len(self.pending) and not self.admitted

    def kv_used(self) -> int:
        return self.cfg.num_blocks - len(self.free)


def trace_bytes(b: Batch) -> bytes:
    """Canonical per-tick trace (little-endian int64), identical in layout to gllm_sched_trace."""
    rd, wp, free0, free1 = b.stats
    v = [b.tick, b.P, b.D, rd, wp, free0, free1, len(b.chunks), len(b.decodes),
         len(b.preempted), len(b.allocs), b.num_tokens, int(b.sample_idx.shape[0])]
    for (rid, s, c, _d) in b.chunks:
        v += [rid, s, c]
    for (rid, p) in b.decodes:
        v += [rid, p]
    v += list(b.preempted)
    for (rid, blk) in b.allocs:
        v += [rid, blk]
    v += [int(x) for x in b.slot_mapping]
    v += [int(x) for x in b.sample_idx]
    return struct.pack("<%dq" % len(v), *v)


def run(cfg, stream, max_ticks=None, until_done=True):
    """Drive the scheduler over a stream; returns the list of batches (traces)."""
    s = Scheduler(cfg, stream.requests, stream.warm)
    out = []
    while True:
        if max_ticks is not None and s.tick >= max_ticks:
            break
        if until_done and s.done():
            break
        out.append(s.build_batch())
    return s, out
