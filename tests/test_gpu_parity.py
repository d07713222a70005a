"""GPU parity: the CUDA path (through the C ABI) vs the oracle on the same seeded inputs.

Bars (BASELINE north_star): weights, slot mapping and scheduler decisions
bit-exact; hidden states per-row inf-norm relative error <= 2e-2 (stage-local); greedy
ids tolerance-aware (logit_ref[u] >= max - 2e-2 |logit_ref|_inf) on >= 99% of rows."""
import numpy as np
import pytest
import torch

from tests.gpu_harness import GpuRun, OracleRun, TOL_HIDDEN, greedy_ok, row_rel_err
from oracle.weights import Weights
from workloads.configs import MODELS, SCHED, ModelShape, SchedParams
from workloads.streams import Request, Stream, make_stream

pytestmark = pytest.mark.gpu

GQA_GPU = ModelShape("gqa-bias-gpu", 2, 256, 4, 2, 64, 512, 512, 1e-5, 10000.0, True, 77)


def _run_pair(shape, cfg, stream, lb=0, le=None, max_ticks=None, kv_blocks=None, check_kv=True, tick_hook=None):
    g = GpuRun(shape, cfg, stream, lb, le, kv_blocks=kv_blocks)
    o = OracleRun(shape, cfg, stream, lb, le)
    n_rows, errs, greedy = 0, [], []
    ticks = 0
    while not o.sched.done() and (max_ticks is None or ticks < max_ticks):
        # stage-local parity for lb > 0: any fp32 input works; both sides get the batch's embedding rows
        ob = o.step(hin_fn=(lambda b: o.W.embed_rows(b.token_ids)) if lb > 0 else None)
        gb = g.step(ob.get("hidden_in"))
        ticks += 1
        b = ob["batch"]
        if tick_hook is not None:
            tick_hook(g, o, b)
        d = gb["desc"]
        assert np.array_equal(d["slot_mapping"], b.slot_mapping)
        if b.num_tokens == 0:
            continue
        assert np.array_equal(gb["slots_dev"], b.slot_mapping), "device slot mapping != oracle"
        e = row_rel_err(gb["hidden"], ob["hidden"])
        errs.append(e)
        n_rows += b.num_tokens
        if "sampled" in gb and len(b.sample_idx):
            greedy.append(greedy_ok(gb["sampled"], ob["logits"]))
        if check_kv:
            for l in range(g.lb, g.le):
                k, v = g.stage.read_kv(l, b.slot_mapping)
                kr = np.stack([o.cache.k[l][s // 16][s % 16] for s in b.slot_mapping])
                vr = np.stack([o.cache.v[l][s // 16][s % 16] for s in b.slot_mapping])
                assert np.max(row_rel_err(k.reshape(len(k), -1), kr.reshape(len(k), -1))) < 2e-2
                assert np.max(row_rel_err(v.reshape(len(v), -1), vr.reshape(len(v), -1))) < 2e-2
    errs = np.concatenate(errs)
    return n_rows, errs, (np.concatenate(greedy) if greedy else np.ones(0, bool))


def test_weights_bit_exact_c0():
    m = MODELS["C0"]
    g = GpuRun(m, SCHED["C0"], make_stream("C0", m.vocab))
    W = Weights(m)
    for l in range(m.n_layers):
        w = W.layer(l)
        for name in ("wq", "wk", "wv", "wo", "wg", "wu", "wd"):
            ref = w[name]
            got = g.stage.read_weight(l, name, 0, ref.shape[0], ref.shape[1])
            assert np.array_equal(got, ref), (l, name)
    E = W.embed_rows(np.arange(m.vocab))
    assert np.array_equal(g.stage.read_weight(0, "embed", 0, m.vocab, m.hidden), E)
    assert np.array_equal(g.stage.read_weight(0, "lm_head", 0, m.vocab, m.hidden), W.lm_head())


def test_weights_bit_exact_bias_and_c1_rows():
    m = GQA_GPU
    g = GpuRun(m, SchedParams(num_blocks=64), Stream("x", []))
    w = Weights(m).layer(1)
    for name, n in (("bq", m.q_dim), ("bk", m.kv_dim), ("bv", m.kv_dim)):
        assert np.array_equal(g.stage.read_weight(1, name, 0, 1, n)[0], w[name])
    # full-width C1 shapes: sampled rows of every tensor of layer 0 (interleaved gate|up layout)
    c1 = MODELS["C1"].with_layers(1)
    from oracle.weights import gen, layer_tid, scale_for
    st = GpuRun(c1, SchedParams(num_blocks=16, maxp=128, max_seqs=64), Stream("x", []), kv_blocks=16,
                max_tokens=256, max_seqs=64)
    for name, rows, cols in (("wq", 4096, 4096), ("wk", 1024, 4096), ("wg", 14336, 4096), ("wu", 14336, 4096),
                             ("wd", 4096, 14336), ("wo", 4096, 4096)):
        for r0 in (0, 127, 128, rows - 1):
            got = st.stage.read_weight(0, name, r0, 1, cols)[0]
            ref = gen(c1.weight_seed, layer_tid(0, name), cols, scale_for("proj", 4096 if name != "wd" else 14336),
                      start=r0 * cols)
            assert np.array_equal(got, ref), (name, r0)


def test_c0_mixed_batch_parity():
    # tick 0: 8 prompts (245 tokens); tick 1: one 64-token prefill chunk + 8 decode tokens (C0)
    m = MODELS["C0"]
    n, errs, greedy = _run_pair(m, SCHED["C0"], make_stream("C0", m.vocab))
    assert n == 245 + 72
    assert errs.max() <= TOL_HIDDEN, errs.max()
    assert greedy.mean() >= 0.99 and len(greedy) == 8 + 1 + 8


def test_c0b_chunked_prefill_parity():
    m = MODELS["C0"]
    n, errs, greedy = _run_pair(m, SCHED["C0b"], make_stream("C0b", m.vocab))
    assert errs.max() <= TOL_HIDDEN, errs.max()
    assert greedy.all()


@pytest.mark.parametrize("chunk", [1, 7, 16, 64, 200])
def test_gqa_bias_chunk_sizes(chunk):
    ids = make_stream("C0", 512).requests[7].token_ids
    st = Stream("x", [Request(0, 0, 70, 4, ids[:73]), Request(1, 0, 23, 3, ids[:25]),
                      Request(2, 1, 150, 2, np.concatenate([ids, ids])[:151])])
    cfg = SchedParams(iterp=1, maxp=chunk, minp=1, pp_depth=1, num_blocks=64)
    n, errs, greedy = _run_pair(GQA_GPU, cfg, st)
    assert errs.max() <= TOL_HIDDEN, errs.max()
    assert greedy.mean() >= 0.99


def test_c1_full_width_first_stage_layer():
    # Llama-3-8B shapes at full width, one layer of stage 0, on a C1 stream prefix (prefill + decode mix,
    # ragged T, several GEMM tiles, split-KV decode): hidden after layer 0 vs the oracle.
    m = MODELS["C1"].with_layers(4)
    st = make_stream("C1", m.vocab, n=120)
    cfg = SCHED["C1"].with_(num_blocks=4000)
    n, errs, _ = _run_pair(m, cfg, st, lb=0, le=1, max_ticks=40, kv_blocks=4000, check_kv=False)
    assert n > 1000
    assert errs.max() <= TOL_HIDDEN, errs.max()


def test_c1_stream_long_chunk_continuation():
    # the first 40 ticks of the full C1 stream at PP=1 include a 984-token chunk continuing a prompt at
    # offset 1402 (kv 2386 keys, 38 key tiles): the tcgen05 prefill kernel's lazy O rescale and
    # long causal tails, at full Llama-3-8B width (one layer, stage-local)
    m = MODELS["C1"].with_layers(4)
    st = make_stream("C1", m.vocab)
    cfg = SCHED["C1"].with_(num_blocks=20000, pp_depth=1)
    n, errs, _ = _run_pair(m, cfg, st, lb=0, le=1, max_ticks=40, kv_blocks=20000, check_kv=False)
    assert n > 40000
    assert errs.max() <= TOL_HIDDEN, errs.max()


@pytest.mark.parametrize("cfg_name,n_req,ticks,kvb", [("C2", 60, 14, 3000), ("C4", 30, 10, 3000)])
def test_full_width_other_shapes_stage_local(cfg_name, n_req, ticks, kvb):
    # C2 = Qwen2.5-14B shapes (H 5120, GQA group 5, q/k/v bias, theta 1e6); C4 = Llama-3-70B shapes
    # (H 8192, I 28672, GQA group 8): one middle-stage layer fed the batch's embedding rows
    # (stage-local parity), on a stream prefix of the config.
    m = MODELS[cfg_name].with_layers(4)
    st = make_stream("C1", m.vocab, n=n_req)          # cold stream of C1 lengths (C4's warm set is separate)
    cfg = SCHED[cfg_name].with_(num_blocks=kvb, pp_depth=2)
    n, errs, _ = _run_pair(m, cfg, st, lb=1, le=2, max_ticks=ticks, kv_blocks=kvb, check_kv=False)
    assert n > 300
    assert errs.max() <= TOL_HIDDEN, errs.max()


def test_c3_long_prompt_chunks_stage_local():
    # Qwen2.5-32B shapes (GQA group 5, bias): the C3 long-prompt stream at PP=1 prefills ~4k-token
    # prompts in Token-Throttled chunks, so later chunks sit at offsets of thousands of keys (many
    # 128-key tiles, both Q tiles of the warp-specialised prefill kernel, causal tails that end in
    # different key tiles for the two tiles)
    m = MODELS["C3"].with_layers(4)
    st = make_stream("C3", m.vocab, n=4)
    cfg = SCHED["C3"].with_(num_blocks=3000, pp_depth=1)
    # ticks 3-5: chunks of 1563, 1977 and 1751 tokens at offsets 0, 1563 and 3540
    n, errs, _ = _run_pair(m, cfg, st, lb=1, le=2, max_ticks=6, kv_blocks=3000, check_kv=False)
    assert n == 5291
    assert errs.max() <= TOL_HIDDEN, errs.max()


def test_c1_last_stage_full_vocab_lm_head():
    # last stage of a 2-layer Llama-3-8B-shaped model: layer 1 + final norm + 128256-wide LM head with the
    # fused argmax epilogue (501 N tiles) -> greedy ids tolerance-aware vs the oracle's fp32 logits
    m = MODELS["C1"].with_layers(2)
    st = make_stream("C1", m.vocab, n=40)
    cfg = SCHED["C1"].with_(num_blocks=2000, pp_depth=1)
    n, errs, greedy = _run_pair(m, cfg, st, lb=1, le=2, max_ticks=12, kv_blocks=2000, check_kv=False)
    assert errs.max() <= TOL_HIDDEN, errs.max()
    assert len(greedy) > 50 and greedy.mean() >= 0.99, (len(greedy), greedy.mean())


def test_invalid_batch_is_einval_not_ub():
    from paper_conf_sc_00090d00l25_b200 import gllm
    m = MODELS["C0"]
    g = GpuRun(m, SCHED["C0"], make_stream("C0", m.vocab))
    d = g.sched.build_batch().to_numpy()
    bad = dict(d)
    bad["block_table"] = d["block_table"].copy()
    bad["block_table"][0, 0] = 10 ** 6
    desc, keep = gllm.desc_from_arrays(bad)
    x = torch.empty((d["num_tokens"], m.hidden), device="cuda")
    with pytest.raises(gllm.GllmError) as ei:
        g.stage.forward(desc, 0, x.data_ptr(), 0, 0)
    assert ei.value.code == -1


def _warm_kv_bit_exact(g, o, shape, warm, layers, n_seq=4):
    # the warm cache itself: GPU bf16 pages == the oracle's O4 values, bit for bit, through the blocks
    from oracle.weights import warm_kv
    blocks = {r.req_id: r.blocks for r in o.sched.admitted}
    for w in warm[:n_seq]:
        pos = np.arange(w.context_len)
        bl = np.asarray(blocks[w.req_id], np.int64)
        slots = (bl[pos // 16] * 16 + pos % 16).astype(np.int32)
        for l in layers:
            k, v = g.stage.read_kv(l, slots)
            kr, vr = warm_kv(shape.weight_seed, w.req_id, w.context_len, l, shape.n_kv_heads, shape.head_dim)
            assert np.array_equal(k, kr) and np.array_equal(v, vr), (w.req_id, l)


def test_c4_warm_start_decode_near_full_kv_last_stage():
    # C4 (Llama-3-70B shapes: H 8192, I 28672, GQA group 8) warm start as the bench runs it, scaled to
    # 64 warm decode sequences with contexts U[1536, 2560] whose O4 warm K/V fill >= 90% of the pool,
    # plus the C4 arrivals (prefill throttled near KV_thresh, Eq.3 UT term / L165).  Last stage: two
    # layers + final norm + the 128256-wide LM head, so the greedy ids are checked too.
    m = MODELS["C4"].with_layers(4)
    full = make_stream("C4", m.vocab, n=12)
    warm = full.warm[:64]
    used = sum(-(-w.context_len // 16) for w in warm)
    nb = int(used / 0.92)
    st = Stream("C4w", full.requests, warm)
    cfg = SCHED["C4"].with_(num_blocks=nb, pp_depth=2)
    kv, ctx = [], []

    def hook(g, o, b):
        if b.tick == 0:
            _warm_kv_bit_exact(g, o, m, warm, (2, 3))
        kv.append(o.sched.kv_used() / nb)
        ctx.extend(int(x) for x in b.kv_len[len(b.chunks):])
    n, errs, greedy = _run_pair(m, cfg, st, lb=2, le=4, max_ticks=6, kv_blocks=nb, check_kv=True, tick_hook=hook)
    assert min(kv) >= 0.9, kv
    assert max(ctx) >= 2400 and len(ctx) >= 6 * 32, (max(ctx), len(ctx))
    assert errs.max() <= TOL_HIDDEN, errs.max()
    assert len(greedy) >= 6 * 32 and greedy.mean() >= 0.99, (len(greedy), greedy.mean())


def test_c3_long_context_decode_stage_local():
    # C3 (Qwen2.5-32B shapes, GQA group 5, q/k/v bias): 40 decode rows at the C3 window's ~4.8k-token
    # contexts (decode ctx ~4.8k), warm-started from O4 K/V, all in one micro-batch
    # (PP=1): long split-KV decode work items merged across splits, vs the oracle, one middle layer.
    from workloads.streams import WarmSeq
    m = MODELS["C3"].with_layers(4)
    rng = np.random.default_rng(33)
    ctxs = rng.integers(4096, 5633, size=40)
    warm = [WarmSeq(i, int(c), 3, rng.integers(0, m.vocab, size=int(c) + 3).astype(np.int32))
            for i, c in enumerate(ctxs)]
    nb = sum(-(-int(c) // 16) for c in ctxs) + 64
    st = Stream("C3w", [], warm)
    cfg = SCHED["C3"].with_(num_blocks=nb, pp_depth=1)

    def hook(g, o, b):
        if b.tick == 0:
            _warm_kv_bit_exact(g, o, m, warm, (1,), n_seq=2)
    n, errs, _ = _run_pair(m, cfg, st, lb=1, le=2, max_ticks=2, kv_blocks=nb, check_kv=True, tick_hook=hook)
    assert n == 80
    assert errs.max() <= TOL_HIDDEN, errs.max()
