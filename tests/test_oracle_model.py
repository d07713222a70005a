"""Pins for the oracle forward (oracle/model.py) -- CPU only.

Independent pins: textbook closed forms (RMSNorm, SiLU, 2-D rotation),
fp64 brute-force attention written as explicit loops, torch's
scaled_dot_product_attention, HF transformers Llama / Qwen2 fp32 forward on the
same weights [ext], and the exactness of paging / chunking / batching
(chunked == unchunked, decode == full recompute).
"""
import math

import numpy as np
import pytest
import torch

from oracle import model as om
from oracle.scheduler import Scheduler, run
from oracle.weights import Weights
from workloads.configs import MODELS, SCHED, ModelShape, SchedParams
from workloads.streams import Request, Stream, make_stream

GQA = ModelShape("tiny-gqa-bias", 2, 128, 4, 2, 32, 256, 300, 1e-5, 10000.0, True, 7)


def test_rmsnorm_closed_form():
    x = np.full((3, 64), 2.0)
    g = np.linspace(0.5, 1.5, 64)
    y = om.rmsnorm(x, g, 1e-5)
    assert np.allclose(y, 2.0 / math.sqrt(4.0 + 1e-5) * g, rtol=1e-14)
    x = np.array([[3.0, 4.0]])
    assert np.allclose(om.rmsnorm(x, np.ones(2), 0.0), [[3 / math.sqrt(12.5), 4 / math.sqrt(12.5)]])


def test_silu_values():
    assert om.silu(np.array([0.0]))[0] == 0.0
    assert abs(om.silu(np.array([1.0]))[0] - 1.0 / (1.0 + math.exp(-1.0))) < 1e-15
    assert abs(om.silu(np.array([40.0]))[0] - 40.0) < 1e-12


def test_rope_is_2d_rotation_and_relative():
    # d = 2: a plain rotation of (x1, x2) by angle pos * theta^0 = pos
    x = np.array([[[1.0, 0.0]], [[0.3, -0.7]]])
    pos = np.array([0.5, 2.0])
    y = om.rope(x, pos, 10000.0)
    for t in range(2):
        c, s = math.cos(pos[t]), math.sin(pos[t])
        x1, x2 = x[t, 0]
        assert np.allclose(y[t, 0], [x1 * c - x2 * s, x2 * c + x1 * s], atol=1e-15)
    # <rope(q, m), rope(k, n)> depends only on m - n; norms preserved
    rng = np.random.default_rng(0)
    q, k = rng.standard_normal((1, 1, 64)), rng.standard_normal((1, 1, 64))
    dots = [np.sum(om.rope(q, [m + 7], 1e4) * om.rope(k, [m], 1e4)) for m in (0, 5, 100, 3000)]
    assert np.allclose(dots, dots[0], rtol=1e-9)
    assert np.allclose(np.linalg.norm(om.rope(q, [123], 1e4)), np.linalg.norm(q))


def test_rope_matches_hf_rotate_half():
    from transformers.models.llama.modeling_llama import apply_rotary_pos_emb
    rng = np.random.default_rng(1)
    T, H, d = 9, 3, 16
    q = rng.standard_normal((T, H, d))
    pos = np.arange(T) * 37
    inv = 1.0 / (500000.0 ** (np.arange(0, d, 2) / d))
    emb = np.concatenate([np.outer(pos, inv)] * 2, axis=-1)
    qt = torch.from_numpy(q).permute(1, 0, 2)[None]
    qr, _ = apply_rotary_pos_emb(qt, qt, torch.from_numpy(np.cos(emb))[None], torch.from_numpy(np.sin(emb))[None])
    assert np.allclose(om.rope(q, pos, 500000.0), qr[0].permute(1, 0, 2).numpy(), atol=1e-12)


def _brute_attention(q, k, v, qpos, kpos):
    Tq, Hq, d = q.shape
    grp = Hq // k.shape[1]
    out = np.zeros_like(q)
    for t in range(Tq):
        for h in range(Hq):
            kh = h // grp
            scores = []
            for s in range(k.shape[0]):
                if kpos[s] <= qpos[t]:
                    scores.append((s, sum(q[t, h, i] * k[s, kh, i] for i in range(d)) / math.sqrt(d)))
            mx = max(sc for _, sc in scores)
            z = sum(math.exp(sc - mx) for _, sc in scores)
            for s, sc in scores:
                out[t, h] += math.exp(sc - mx) / z * v[s, kh]
    return out


def test_attention_brute_force_fp64():
    rng = np.random.default_rng(2)
    q = rng.standard_normal((5, 4, 8))
    k = rng.standard_normal((9, 2, 8))
    v = rng.standard_normal((9, 2, 8))
    qpos = np.array([4, 5, 6, 7, 8])          # a chunk at offset 4 over 9 keys
    kpos = np.arange(9)
    assert np.allclose(om.attention(q, k, v, qpos, kpos), _brute_attention(q, k, v, qpos, kpos), atol=1e-13)


def test_attention_matches_torch_sdpa():
    rng = np.random.default_rng(3)
    q = rng.standard_normal((12, 8, 16))
    k = rng.standard_normal((12, 2, 16))
    v = rng.standard_normal((12, 2, 16))
    pos = np.arange(12)
    ref = torch.nn.functional.scaled_dot_product_attention(
        torch.from_numpy(q).permute(1, 0, 2), torch.from_numpy(k).permute(1, 0, 2),
        torch.from_numpy(v).permute(1, 0, 2), is_causal=True, enable_gqa=True).permute(1, 0, 2).numpy()
    assert np.allclose(om.attention(q, k, v, pos, pos), ref, atol=1e-12)


def _hf_model(m, W):
    from transformers import LlamaConfig, LlamaForCausalLM, Qwen2Config, Qwen2ForCausalLM
    kw = dict(vocab_size=m.vocab, hidden_size=m.hidden, intermediate_size=m.intermediate,
              num_hidden_layers=m.n_layers, num_attention_heads=m.n_heads,
              num_key_value_heads=m.n_kv_heads, rms_norm_eps=m.rms_eps, rope_theta=m.rope_theta,
              max_position_embeddings=4096, tie_word_embeddings=False)
    if m.qkv_bias:
        hf = Qwen2ForCausalLM(Qwen2Config(**kw))
    else:
        hf = LlamaForCausalLM(LlamaConfig(head_dim=m.head_dim, **kw))
    hf = hf.float().eval()
    sd = {"model.embed_tokens.weight": W.embed_rows(np.arange(m.vocab)),
          "lm_head.weight": W.lm_head(), "model.norm.weight": W.final_norm()}
    for l in range(m.n_layers):
        w = W.layer(l)
        p = f"model.layers.{l}."
        sd.update({p + "self_attn.q_proj.weight": w["wq"], p + "self_attn.k_proj.weight": w["wk"],
                   p + "self_attn.v_proj.weight": w["wv"], p + "self_attn.o_proj.weight": w["wo"],
                   p + "mlp.gate_proj.weight": w["wg"], p + "mlp.up_proj.weight": w["wu"],
                   p + "mlp.down_proj.weight": w["wd"], p + "input_layernorm.weight": w["g1"],
                   p + "post_attention_layernorm.weight": w["g2"]})
        if m.qkv_bias:
            sd.update({p + "self_attn.q_proj.bias": w["bq"], p + "self_attn.k_proj.bias": w["bk"],
                       p + "self_attn.v_proj.bias": w["bv"]})
    hf.load_state_dict({k: torch.from_numpy(np.ascontiguousarray(v)) for k, v in sd.items()}, strict=True)
    return hf


@pytest.mark.parametrize("shape", [MODELS["C0"], GQA], ids=["C0-llama", "gqa-qwen2-bias"])
def test_dense_forward_matches_hf_transformers(shape):
    W = Weights(shape)
    hf = _hf_model(shape, W)
    ids = make_stream("C0", shape.vocab).requests[7].token_ids[:100]
    hs = om.dense_forward(shape, W, ids)
    with torch.no_grad():
        out = hf(torch.from_numpy(ids.astype(np.int64))[None], output_hidden_states=True)
    for l in range(1, shape.n_layers):   # HF's last hidden state is post-final-norm
        ref = out.hidden_states[l][0].numpy()
        assert np.max(np.abs(hs[l] - ref)) / np.max(np.abs(ref)) < 1e-4
    lg = om.logits_of(shape, W, hs[-1])
    ref = out.logits[0].numpy()
    assert np.max(np.abs(lg - ref)) / np.max(np.abs(ref)) < 1e-4


def _check_stage_equals_dense(shape, stream, sched_cfg, dtype=np.float64):
    W = Weights(shape, dtype=dtype)
    s = Scheduler(sched_cfg, stream.requests)
    cache = om.PagedCache(shape, sched_cfg.block_size, dtype)
    by_id = {r.req_id: r for r in stream.requests}
    dense = {}
    n_rows = 0
    while not s.done():
        b = s.build_batch()
        if b.num_tokens == 0:
            continue
        out = om.stage_forward(shape, W, cache, b, 0, shape.n_layers)
        for i in range(len(b.cu_q) - 1):
            rid = int(b.seq_req_ids[i])
            if rid not in dense:
                r = by_id[rid]
                dense[rid] = om.dense_forward(shape, W, r.token_ids)[-1]
            for t in range(int(b.cu_q[i]), int(b.cu_q[i + 1])):
                ref = dense[rid][int(b.positions[t])]
                err = np.max(np.abs(out["hidden"][t] - ref)) / np.max(np.abs(ref))
                assert err < (1e-10 if dtype == np.float64 else 2e-5), (b.tick, rid, t, err)
                n_rows += 1
        if len(b.sample_idx):
            ref_lg = om.logits_of(shape, W, out["hidden"][b.sample_idx])
            assert np.array_equal(out["sampled"], om.greedy(ref_lg))
    return n_rows


def test_c0_paged_mixed_batches_equal_dense():
    # tick 0: 8 prompts; tick 1: one 64-token chunk + 8 decodes on block edges (decode == recompute)
    n = _check_stage_equals_dense(MODELS["C0"], make_stream("C0", 512), SCHED["C0"])
    assert n == 245 + 72


def test_c0b_chunked_equals_unchunked():
    # chunks [0:40], [40:78], [78:104] at non-block-aligned offsets, then a decode
    _check_stage_equals_dense(MODELS["C0"], make_stream("C0b", 512), SCHED["C0b"])


@pytest.mark.parametrize("chunk", [1, 7, 16, 64, 200])
def test_chunk_sizes_gqa_bias(chunk):
    st = Stream("x", [Request(0, 0, 70, 3, make_stream("C0", 300).requests[7].token_ids[:72]),
                      Request(1, 0, 23, 2, make_stream("C0", 300).requests[6].token_ids[:24])])
    cfg = SchedParams(iterp=1, maxp=chunk, minp=1, pp_depth=1, num_blocks=64)
    _check_stage_equals_dense(GQA, st, cfg)


def test_fp32_paged_equals_fp32_dense():
    n = _check_stage_equals_dense(MODELS["C0"], make_stream("C0", 512), SCHED["C0"], dtype=np.float32)
    assert n > 0


def test_warm_start_decode_reads_the_warm_cache():
    # A warm sequence's first decode (pos = context_len) attends the O4 warm K/V of positions
    # [0, context_len) plus its own new key: stage_forward through the paged cache (blocks from the
    # scheduler's warm allocation) == the same layer computed on dense concatenated arrays.
    from oracle.weights import warm_kv
    from workloads.streams import WarmSeq
    shape = GQA.with_layers(1)
    W = Weights(shape, dtype=np.float64)
    ids = np.arange(200, dtype=np.int32) % shape.vocab
    warm = [WarmSeq(0, 37, 3, ids[:40]), WarmSeq(1, 64, 2, ids[:66]), WarmSeq(2, 5, 2, ids[:7])]
    cfg = SchedParams(pp_depth=1, num_blocks=32, block_size=16)
    s = Scheduler(cfg, [], warm)
    cache = om.PagedCache(shape, 16, np.float64)
    for r in s.admitted:
        k, v = warm_kv(shape.weight_seed, r.req_id, r.orig_len, 0, shape.n_kv_heads, shape.head_dim)
        cache.fill_warm(0, r.blocks, k, v)
    b = s.build_batch()
    assert [p for (_, p) in b.decodes] == [37, 64, 5]
    out = om.stage_forward(shape, W, cache, b, 0, 1)
    w = W.layer(0)
    for t, (rid, p) in enumerate(b.decodes):
        x = W.embed_rows(ids[p:p + 1])
        h = om.rmsnorm(x, w["g1"], shape.rms_eps)
        q, k, v = om._qkv(shape, w, h, np.array([p]))
        kw, vw = warm_kv(shape.weight_seed, rid, p, 0, shape.n_kv_heads, shape.head_dim)
        kk, vv = np.concatenate([kw, k]), np.concatenate([vw, v])
        a = om.attention(q, kk, vv, np.array([p]), np.arange(p + 1)).reshape(1, shape.q_dim)
        ref = om._mlp(shape, w, x + a @ w["wo"].T)
        assert np.max(np.abs(out["hidden"][t] - ref[0])) / np.max(np.abs(ref)) < 1e-12
