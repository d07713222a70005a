"""Pins for the oracle scheduler (oracle/scheduler.py) -- CPU only.

Pinned against: hand-worked values of Eq.3 + threshold (L165)
and Eq.4 (L181), the hand-worked trace
W1 (tests/golden/w1_trace.txt), the hand-built C0 / C0b streams whose slots
follow from the closed form slot = bt[pos//16]*16 + pos%16, and invariants.
"""
import os

import numpy as np
import pytest

from oracle.scheduler import Scheduler, run, throttle_decode, throttle_prefill
from workloads.configs import SCHED, SchedParams
from workloads.streams import Request, Stream, make_stream

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
DEF = SchedParams(num_blocks=1000)   # #T=8, MaxP=2048, MinP=32, thresh=1/20 (L248)


@pytest.mark.parametrize("wp,free,expect", [
    (10000, 1000, 1250),   # E1: WP/T = 1250 < cap 2048
    (10000, 500, 970),     # E2: cap = floor(2048*9000/19000)
    (100, 1000, 32),       # E3: floor(12.5) -> MinP
    (20, 1000, 20),        # E4: MinP capped by WP (R11)
    (10000, 49, 0),        # E5: KV_free 0.049 < 0.05 -> suspended (L165)
    (10000, 50, 32),       # E6: equality uses Eq.3 (L167 ">="): cap 0 -> MinP
    (0, 1000, 0),          # E7: nothing waiting
    (20000, 1000, 2048),   # E8: MaxP
    (3000, 300, 375),      # E9: cap 538 > 375
])
def test_eq3_examples(wp, free, expect):
    assert throttle_prefill(DEF, wp, free) == expect


def test_eq3_matches_exact_rational_floor():
    # floor is monotone, so the integer reading equals floor(Eq.3) evaluated in exact rationals.
    from fractions import Fraction as F
    rng = np.random.default_rng(0)
    for _ in range(2000):
        n = int(rng.integers(1, 5000))
        cfg = SchedParams(iterp=int(rng.integers(1, 17)), maxp=int(rng.integers(1, 4096)),
                          minp=int(rng.integers(0, 64)), kvthresh_num=int(rng.integers(0, 5)),
                          kvthresh_den=int(rng.integers(5, 40)), num_blocks=n)
        wp = int(rng.integers(0, 50000))
        free = int(rng.integers(0, n + 1))
        kvf, th = F(free, n), F(cfg.kvthresh_num, cfg.kvthresh_den)
        if wp == 0 or kvf < th:
            ref = 0
        else:
            eq3 = max(min(F(wp, cfg.iterp), cfg.maxp * (kvf - th) / (1 - th)), cfg.minp)
            ref = min(int(eq3), wp)      # int() == floor for non-negative rationals
        assert throttle_prefill(cfg, wp, free) == ref


def test_eq1_eq2_special_cases():
    # thresh = 0 and KV fully free: Eq.3 reduces to Eq.1 (WT only)
    cfg = SchedParams(kvthresh_num=0, kvthresh_den=20, num_blocks=100)
    for wp in [1, 31, 32, 33, 255, 256, 1000, 16384, 16385, 99999]:
        eq1 = min(max(wp // 8, 32), 2048)
        assert throttle_prefill(cfg, wp, 100) == min(eq1, wp)
    # WP huge: Eq.3 reduces to Eq.2 with KV_free rescaled over the threshold
    for free in [0, 1, 5, 50, 99, 100]:
        eq2 = max((2048 * free) // 100, 32)
        assert throttle_prefill(cfg, 10 ** 9, free) == (eq2 if free > 0 else 32)


NO_WT, NO_UT = DEF.with_(policy=2), DEF.with_(policy=3)


@pytest.mark.parametrize("cfg,wp,free,expect", [
    # "w/o WT" (R19): max(MaxP*(KV_free-th)/(1-th), MinP), capped by WP
    (NO_WT, 10000, 1000, 2048),   # KV fully free -> MaxP (WP/T = 1250 no longer caps it)
    (NO_WT, 10000, 500, 970),     # floor(2048*9000/19000)
    (NO_WT, 100, 1000, 100),      # capped by WP (R11)
    (NO_WT, 10000, 49, 0),        # threshold kept (L165)
    (NO_WT, 10000, 50, 32),       # cap 0 -> MinP
    # "w/o UT" (R20): Eq.1 = min(max(WP/T, MinP), MaxP) with the L165 threshold
    (NO_UT, 10000, 500, 1250),    # KV pressure ignored: WP/T
    (NO_UT, 20000, 60, 2048),     # MaxP even with 6% free
    (NO_UT, 100, 1000, 32),       # MinP
    (NO_UT, 20, 1000, 20),        # capped by WP
    (NO_UT, 10000, 49, 0),        # threshold kept
])
def test_ablation_examples(cfg, wp, free, expect):
    assert throttle_prefill(cfg, wp, free) == expect


def test_ablations_match_eq1_eq2_exact_rationals():
    # policy 2 is floor(Eq.2 rescaled over the threshold), policy 3 is floor(Eq.1) (L153, L161),
    # both behind the L165 threshold and capped by #WP (R11), in exact rationals
    from fractions import Fraction as F
    rng = np.random.default_rng(1)
    for _ in range(2000):
        n = int(rng.integers(1, 5000))
        base = SchedParams(iterp=int(rng.integers(1, 17)), maxp=int(rng.integers(1, 4096)),
                           minp=int(rng.integers(0, 64)), kvthresh_num=int(rng.integers(0, 5)),
                           kvthresh_den=int(rng.integers(5, 40)), num_blocks=n)
        wp, free = int(rng.integers(0, 50000)), int(rng.integers(0, n + 1))
        kvf, th = F(free, n), F(base.kvthresh_num, base.kvthresh_den)
        off = wp == 0 or kvf < th
        eq2 = max(base.maxp * (kvf - th) / (1 - th), base.minp)
        eq1 = min(max(F(wp, base.iterp), base.minp), base.maxp)
        assert throttle_prefill(base.with_(policy=2), wp, free) == (0 if off else min(int(eq2), wp))
        assert throttle_prefill(base.with_(policy=3), wp, free) == (0 if off else min(int(eq1), wp))


def test_eq4_examples():
    c4 = SchedParams(pp_depth=4)
    assert throttle_decode(c4, 1000) == 250
    assert throttle_decode(c4, 10) == 3          # ceil (R6)
    assert throttle_decode(c4, 0) == 0
    assert throttle_decode(SchedParams(pp_depth=1), 7) == 7


def test_eq4_steady_pattern_and_ready_cap():
    # RD=10 at PP=4, decode-only, long outputs: per-tick decode counts 3,3,3,1 repeating (Fig.8)
    cfg = SchedParams(pp_depth=4, num_blocks=4096, iterp=1, maxp=4096, minp=1)
    reqs = [Request(i, 0, 16, 1000, np.zeros(16 + 999, np.int32)) for i in range(10)]
    s = Scheduler(cfg, reqs)
    counts = [len(s.build_batch().decodes) for _ in range(24)]
    steady = counts[8:20]
    assert steady == [3, 3, 3, 1] * 3, counts
    # RD=10 but only 2 ready -> 2 (L183 "schedule all of them")
    cfg2 = SchedParams(pp_depth=4, num_blocks=4096)
    s2 = Scheduler(cfg2)
    for i in range(10):
        s2.admitted.append(_warm_req(s2, i))
    for r in s2.admitted[2:]:
        r.inflight = 1
    assert len(s2.build_batch(auto_retire=False).decodes) == 2


def _warm_req(s, i):
    from oracle.scheduler import _Req
    r = _Req(i, 0, 20, 50, np.zeros(80, np.int32))
    r.prefill_len = r.sched_prompt = r.done_prompt = 20
    r.gen = 1
    s._alloc(r, [])
    s._alloc(r, [])
    return r


def _parse_w1():
    rows = []
    with open(os.path.join(GOLDEN, "w1_trace.txt")) as f:
        for line in f:
            if line.startswith("#") or not line.strip():
                continue
            tick, pd, ch, dec, slots, free = [x.strip() for x in line.split("|")]
            P, D = map(int, pd.split())
            chunks = [] if ch == "-" else [tuple(map(int, c.split(":"))) for c in ch.split(",")]
            decs = [] if dec == "-" else [tuple(map(int, d.split(":"))) for d in dec.split(",")]
            sl = [] if slots == "-" else list(map(int, slots.split(",")))
            rows.append((int(tick), P, D, chunks, decs, sl, int(free)))
    return rows


def test_w1_full_trace():
    cfg = SchedParams(iterp=2, maxp=16, minp=2, kvthresh_num=1, kvthresh_den=4,
                      pp_depth=2, num_blocks=16, block_size=4)
    st = Stream("W1", [Request(0, 0, 12, 3, np.zeros(14, np.int32)),
                       Request(1, 1, 5, 2, np.zeros(6, np.int32))])
    s, batches = run(cfg, st)
    gold = _parse_w1()
    assert len(batches) == len(gold)
    for b, (tick, P, D, chunks, decs, sl, free) in zip(batches, gold):
        assert b.tick == tick
        assert (b.P, b.D) == (P, D), tick
        assert [(c[0], c[1], c[2]) for c in b.chunks] == chunks, tick
        assert list(b.decodes) == decs, tick
        assert list(b.slot_mapping) == sl, tick
        assert b.stats[3] == free, tick
    assert sorted(s.free) == list(range(16))


def test_c0_trace():
    cfg = SCHED["C0"]
    st = make_stream("C0", 512)
    s = Scheduler(cfg, st.requests)
    b0 = s.build_batch()
    assert b0.P == 245 and b0.num_tokens == 245 and len(b0.chunks) == 8
    assert cfg.num_blocks - len(s.free) == 19
    b1 = s.build_batch()
    assert b1.stats[2] == 45                      # free after retire
    assert [(c[0], c[1], c[2]) for c in b1.chunks] == [(8, 0, 64)]
    assert len(b1.decodes) == 8 and b1.num_tokens == 72
    assert list(b1.slot_mapping[64:]) == [1, 31, 304, 65, 111, 320, 177, 292]
    assert cfg.num_blocks - len(s.free) == 25
    # decodes sit on block edges 15/16/17, 31/32/33
    assert [p for (_, p) in b1.decodes] == [1, 15, 16, 17, 31, 32, 33, 100]
    assert list(b1.sample_idx) == [63] + list(range(64, 72))


def test_c0b_trace():
    st = make_stream("C0b", 512)
    s, bs = run(SCHED["C0b"], st)
    assert [[(c[1], c[2]) for c in b.chunks] for b in bs[:3]] == [[(0, 40)], [(40, 38)], [(78, 26)]]
    # tick-1 UT cap: floor(40*(61*20-64)/(64*19)) = 38  (Eq.3 UT term, L169)
    assert bs[1].P == 38 and bs[1].stats[2] == 61
    assert bs[3].decodes == [(0, 104)] and list(bs[3].slot_mapping) == [104]


def _check_invariants(cfg, st, max_ticks=None):
    s = Scheduler(cfg, st.requests, st.warm)
    live = {}       # slot -> (req, pos)
    total_p = 0
    while not s.done() and (max_ticks is None or s.tick < max_ticks):
        b = s.build_batch()
        total_p += b.num_prefill_tokens
        # live slots unique within a batch
        assert len(set(b.slot_mapping.tolist())) == b.num_tokens
        # block tables: no block held by two live requests
        owners = {}
        for r in s.admitted:
            for blk in r.blocks:
                assert blk not in owners, "block double-allocated"
                owners[blk] = r.req_id
        assert len(owners) + len(s.free) == cfg.num_blocks
        assert len(set(s.free)) == len(s.free)
        # slots of this batch lie in blocks owned by the token's request
        for t, slot in enumerate(b.slot_mapping):
            seq = np.searchsorted(b.cu_q, t, side="right") - 1
            assert owners[int(slot) // cfg.block_size] == int(b.seq_req_ids[seq])
        # KV_free bookkeeping: free after build == free before - allocations + preemption releases
        assert b.stats[3] == len(s.free)
        assert b.num_tokens <= cfg.maxp + -(-max(b.stats[0], 1) // cfg.pp_depth) or cfg.policy == 1
    return s, total_p


def test_invariants_and_prompt_conservation_small_stream():
    st = make_stream("C1", 1024, n=300)
    cfg = SchedParams(pp_depth=2, num_blocks=2000)
    s, total_p = _check_invariants(cfg, st)
    assert s.done()
    assert total_p == sum(r.prompt_len for r in st.requests) + 0 * s.preemptions
    assert sorted(s.free) == list(range(cfg.num_blocks))
    assert all(r.gen == r.output_len for r in s.finished)


def test_preemption_recompute_tiny_pool():
    # pool so small that decodes run out of blocks -> preemption by recompute (R14)
    st = make_stream("C1", 1024, n=60)
    cfg = SchedParams(pp_depth=2, num_blocks=120, kvthresh_num=0, kvthresh_den=20)
    s, total_p = _check_invariants(cfg, st)
    assert s.done()
    assert s.preemptions > 0
    # every prompt token prefilled at least once; recompute adds the regenerated tokens
    assert total_p >= sum(r.prompt_len for r in st.requests)
    assert sorted(s.free) == list(range(cfg.num_blocks))
    assert all(r.gen == r.output_len for r in s.finished)


def test_decode_fairness_once_per_pp_ticks():
    # with enough KV, every decode-phase request is scheduled at least once every PP..2PP ticks
    st = make_stream("C1", 1024, n=150)
    cfg = SchedParams(pp_depth=4, num_blocks=5000)
    s = Scheduler(cfg, st.requests)
    last = {}
    while not s.done():
        b = s.build_batch()
        for (rid, _p) in b.decodes:
            if rid in last:
                assert b.tick - last[rid] >= cfg.pp_depth
            last[rid] = b.tick


# ---- R21: context-aware Token Throttling (policy 4; PAPER.md L354 future work) ----------------

def test_chunk_cost_closed_form_and_examples():
    from oracle.scheduler import chunk_cost
    # pairs of a chunk of c tokens at offset s = c*s + c(c+1)/2 (query s+j sees keys 0..s+j)
    for s0 in (0, 1, 17, 1000):
        for c in (0, 1, 2, 15, 64):
            for a in (1, 7, 100, 10 ** 9):
                assert chunk_cost(s0, c, a) == c + (c * s0 + c * (c + 1) // 2) // a
    # hand-worked (R21): a = 100
    assert chunk_cost(0, 164, 100) == 164 + 13530 // 100 == 299
    assert chunk_cost(0, 165, 100) == 301
    assert chunk_cost(164, 47, 100) == 47 + (7708 + 1128) // 100 == 135
    assert chunk_cost(164, 48, 100) == 138


def test_ctx_policy_hand_worked_trace():
    # one 300-token prompt, #T = 1, PP = 1, a = 100 pairs/token; Eq.3 gives the budget P = WP each tick
    cfg = SchedParams(iterp=1, maxp=2048, minp=1, pp_depth=1, num_blocks=64, policy=4, attn_pairs_per_token=100)
    st = Stream("ctx", [Request(0, 0, 300, 2, np.zeros(301, np.int32))])
    s, bs = run(cfg, st)
    # tick 0: budget 300 -> c = 164 (cost 299; 165 would cost 301)
    # tick 1: budget 136 at offset 164 -> c = 47 (cost 135; 48 would cost 138)
    assert [(b.P, [(c[1], c[2]) for c in b.chunks]) for b in bs[:2]] == [(300, [(0, 164)]), (136, [(164, 47)])]
    # every tick takes the longest chunk whose cost fits its budget; when not even one token fits,
    # one token is taken anyway (progress rule of R21)
    from oracle.scheduler import chunk_cost
    for b in bs:
        for (_rid, s0, c, _d) in b.chunks:
            assert chunk_cost(s0, c, 100) <= b.P or c == 1
            assert c == 300 - s0 or chunk_cost(s0, c + 1, 100) > b.P
    assert sum(c[2] for b in bs for c in b.chunks) == 300


def test_ctx_policy_reduces_to_token_throttling_for_large_a():
    # a -> infinity: every chunk costs its token count, so the trace equals policy 0 byte for byte
    from oracle.scheduler import trace_bytes
    st = make_stream("C1", 1024, n=150)
    base = SchedParams(pp_depth=2, num_blocks=3000)
    s0 = Scheduler(base, st.requests)
    s4 = Scheduler(base.with_(policy=4, attn_pairs_per_token=2 ** 31 - 1), st.requests)
    while not s0.done():
        assert trace_bytes(s0.build_batch()) == trace_bytes(s4.build_batch())
    assert s4.done()


def test_ctx_policy_invariants_and_long_prompts():
    # C3-like long prompts: chunks deep into a prompt get fewer tokens than Eq.3's count
    st = make_stream("C3", 1024, n=12)
    cfg = SCHED["C3"].with_(num_blocks=6000, pp_depth=4, policy=4, attn_pairs_per_token=4096)
    s, total_p = _check_invariants(cfg, st, max_ticks=None)
    assert s.done() and total_p == sum(r.prompt_len for r in st.requests)
    assert sorted(s.free) == list(range(cfg.num_blocks))


@pytest.mark.parametrize("name", ["w1_trace.txt", "p1_preempt_order.txt", "p2_preempt_inflight.txt",
                                  "s1_sarathi.txt", "ws1_warm.txt"])
def test_hand_worked_goldens(name):
    # hand-worked traces (tests/golden/, derivations in their headers): preemption victim order and
    # in-flight exclusion (R14, L127/L165/L325), Sarathi-Serve (L81/L125/L310), warm start (C4)
    from oracle.scheduler import trace_bytes
    from tests.golden_traces import CASES, compare
    cfg, st = CASES[name]
    s, batches = run(cfg, st)
    compare([trace_bytes(b) for b in batches], name)
    assert sorted(s.free) == list(range(cfg.num_blocks))
