"""Kernel-level parity of the tcgen05 GEMM (gllm_op_gemm, include/gllm_ops.h) against the plain
definition Y = A W^T computed in fp64 with numpy on the same bf16 values, for ragged M (TMA
out-of-bounds rows, partial tiles), stream-K (few tiles) and every epilogue."""
import numpy as np
import pytest
import torch

from paper_conf_sc_00090d00l25_b200 import gllm

pytestmark = pytest.mark.gpu


@pytest.fixture(params=[1, 2, 0], ids=["cta1", "cta2", "auto"], autouse=True)
def variant(request):
    # every test runs with the 1-CTA kernel, the CTA-pair (cta_group::2) kernel and the automatic choice
    gllm.op_set_gemm_variant(request.param)
    yield request.param
    gllm.op_set_gemm_variant(0)


def _bf16(shape, scale, seed):
    g = torch.Generator().manual_seed(seed)
    return (torch.randn(shape, generator=g) * scale).to(torch.bfloat16)


def _ref(A, W):
    return A.double().numpy() @ W.double().numpy().T


@pytest.mark.parametrize("M", [1, 7, 128, 129, 1000, 2094])
@pytest.mark.parametrize("N,K", [(768, 256), (4096, 4096), (6144, 4096), (1024, 14336)])
def test_store_bf16_with_bias(M, N, K):
    A, W = _bf16((M, K), 1.0, 1), _bf16((N, K), K ** -0.5, 2)
    bias = torch.randn(N, generator=torch.Generator().manual_seed(3)) * 0.02
    dA, dW, db = A.cuda(), W.cuda(), bias.cuda()
    out = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
    gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, N, K, 0, out.data_ptr(), db.data_ptr())
    torch.cuda.synchronize()
    ref = _ref(A, W) + bias.double().numpy()
    got = out.float().cpu().numpy()
    err = np.abs(got - ref).max(-1) / np.abs(ref).max(-1)
    assert err.max() < 1e-2, err.max()


@pytest.mark.parametrize("M", [1, 33, 300, 2094])
@pytest.mark.parametrize("N,K", [(4096, 4096), (8192, 28672), (5120, 5120)])
def test_residual_add_f32(M, N, K):
    # covers whole-tile and stream-K (below one wave of tiles: fp32 vector reductions) schedules
    A, W = _bf16((M, K), 1.0, 4), _bf16((N, K), K ** -0.5, 5)
    x0 = torch.randn((M, N), generator=torch.Generator().manual_seed(6))
    dA, dW, x = A.cuda(), W.cuda(), x0.clone().cuda()
    gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, N, K, 1, x.data_ptr())
    torch.cuda.synchronize()
    ref = x0.double().numpy() + _ref(A, W)
    err = np.abs(x.cpu().double().numpy() - ref).max()
    assert err < 1e-3, err


@pytest.mark.parametrize("M,N,K", [(900, 5120, 5120), (900, 5120, 27648), (1100, 4096, 4096), (2094, 5120, 5120),
                                   (626, 5120, 13824), (300, 5120, 5120)])
def test_residual_add_f32_hybrid_tail(M, N, K):
    # CTA-pair tiles whose last wave is mostly empty (C3's O / down GEMMs at T ~ 900: 80 tiles of
    # 256 x 256 on 74 pairs): whole tiles first, the tail tiles' k-blocks spread over every pair
    # and reduced into the residual (Jobs mode 2); below one wave (C2's O / down at T ~ 626: 60 tiles
    # on 74 pairs, whole tiles since they fill >= 75% of the pairs) every tile's k-blocks are spread
    # over all pairs
    A, W = _bf16((M, K), 1.0, 14), _bf16((N, K), K ** -0.5, 15)
    x0 = torch.randn((M, N), generator=torch.Generator().manual_seed(16))
    dA, dW, x = A.cuda(), W.cuda(), x0.clone().cuda()
    gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, N, K, 1, x.data_ptr())
    torch.cuda.synchronize()
    ref = x0.double().numpy() + _ref(A, W)
    err = np.abs(x.cpu().double().numpy() - ref).max()
    assert err < 1e-3, err


@pytest.mark.parametrize("M,N,K", [(9460, 288, 256), (9400, 544, 512), (2094, 2336, 1024)])
def test_residual_add_f32_tma_epilogue_ragged(M, N, K):
    # the CTA-pair residual epilogue through TMA (x chunks loaded ahead into swizzled SMEM, stored
    # back by TMA): a last N tile of one or two 32-column chunks (N % 256 != 0) inside the whole-tile
    # range (74 tiles = one wave for the first two shapes), ragged M (rows past M: zero-filled loads,
    # clipped stores), and a hybrid launch mixing TMA whole tiles with stream-K tail tiles
    A, W = _bf16((M, K), 1.0, 24), _bf16((N, K), K ** -0.5, 25)
    x0 = torch.randn((M, N), generator=torch.Generator().manual_seed(26))
    dA, dW, x = A.cuda(), W.cuda(), x0.clone().cuda()
    gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, N, K, 1, x.data_ptr())
    torch.cuda.synchronize()
    ref = x0.double().numpy() + _ref(A, W)
    err = np.abs(x.cpu().double().numpy() - ref).max()
    assert err < 1e-3, err


@pytest.mark.parametrize("M", [5, 128, 700])
def test_silu_mul_interleaved(M):
    I, K = 1024, 512
    A = _bf16((M, K), 1.0, 7)
    Wg, Wu = _bf16((I, K), K ** -0.5, 8), _bf16((I, K), K ** -0.5, 9)
    W = torch.empty((2 * I, K), dtype=torch.bfloat16)
    for j in range(I // 128):      # interleave blocks of 128 gate rows and 128 up rows
        W[256 * j:256 * j + 128] = Wg[128 * j:128 * j + 128]
        W[256 * j + 128:256 * j + 256] = Wu[128 * j:128 * j + 128]
    dA, dW = A.cuda(), W.cuda()
    out = torch.empty((M, I), dtype=torch.bfloat16, device="cuda")
    gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, 2 * I, K, 2, out.data_ptr())
    torch.cuda.synchronize()
    g, u = _ref(A, Wg), _ref(A, Wu)
    ref = g / (1 + np.exp(-g)) * u
    err = np.abs(out.float().cpu().numpy() - ref).max(-1) / np.abs(ref).max(-1)
    assert err.max() < 1e-2, err.max()


@pytest.mark.parametrize("M,N", [(1, 512), (9, 128256), (200, 152064), (256, 128256), (300, 152064)])
def test_argmax_epilogue(M, N):
    K = 1024
    A, W = _bf16((M, K), 1.0, 10), _bf16((N, K), K ** -0.5, 11)
    dA, dW = A.cuda(), W.cuda()
    out = torch.empty((M,), dtype=torch.int32, device="cuda")
    gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, N, K, 3, out.data_ptr())
    torch.cuda.synchronize()
    ref = _ref(A, W)
    ids = out.cpu().numpy()
    # fp32 accumulation vs fp64: the chosen logit must be the max up to accumulation error
    # (tolerance-aware greedy: several ids are correct when logits tie within rounding)
    assert np.all(ref[np.arange(M), ids] >= ref.max(-1) - 1e-4 * np.abs(ref).max(-1))


def test_bad_shapes_are_einval():
    A = torch.zeros((4, 100), dtype=torch.bfloat16, device="cuda")
    with pytest.raises(gllm.GllmError) as e:
        gllm.op_gemm(A.data_ptr(), A.data_ptr(), 4, 4, 100, 0, A.data_ptr())
    assert e.value.code == -1


@pytest.mark.parametrize("det", [False, True], ids=["default", "deterministic"])
@pytest.mark.parametrize("M,N,K,epi", [(128, 10240, 8192, 0), (96, 8192, 8192, 1), (128, 8192, 28672, 1),
                                       (64, 2048, 4096, 2), (17, 6144, 4096, 0), (900, 5120, 5120, 1)])
def test_small_t_weight_streaming_shapes_deterministic(M, N, K, epi, variant, det):
    # C4's small-T projections (T <= 128: one M tile, few N tiles -> cluster split-K for the
    # non-additive epilogues, k-split partials reduced over DSMEM in rank order; stream-K for the
    # residual add) and C3's O shape (hybrid tail): parity with fp64 in both modes; with
    # gllm_op_set_deterministic two runs are bit-identical for every kernel variant
    gllm.op_set_deterministic(det)
    A = _bf16((M, K), 1.0, 20)
    if epi == 2:
        I = N // 2
        Wg, Wu = _bf16((I, K), K ** -0.5, 21), _bf16((I, K), K ** -0.5, 23)
        W = torch.empty((N, K), dtype=torch.bfloat16)
        for j in range(I // 128):
            W[256 * j:256 * j + 128] = Wg[128 * j:128 * j + 128]
            W[256 * j + 128:256 * j + 256] = Wu[128 * j:128 * j + 128]
    else:
        W = _bf16((N, K), K ** -0.5, 21)
    dA, dW = A.cuda(), W.cuda()
    x0 = torch.randn((M, N), generator=torch.Generator().manual_seed(22))
    outs = []
    for _ in range(2):
        if epi == 1:
            out = x0.clone().cuda()
        elif epi == 2:
            out = torch.empty((M, N // 2), dtype=torch.bfloat16, device="cuda")
        else:
            out = torch.empty((M, N), dtype=torch.bfloat16, device="cuda")
        gllm.op_gemm(dA.data_ptr(), dW.data_ptr(), M, N, K, epi, out.data_ptr())
        torch.cuda.synchronize()
        outs.append(out.float().cpu().numpy())
    if epi == 1:
        assert np.abs(outs[0] - (x0.double().numpy() + _ref(A, W))).max() < 1e-3
    else:
        if epi == 2:
            g, u = _ref(A, Wg), _ref(A, Wu)
            ref = g / (1 + np.exp(-g)) * u
        else:
            ref = _ref(A, W)
        err = np.abs(outs[0] - ref).max(-1) / np.abs(ref).max(-1)
        assert err.max() < 1e-2, err.max()
    gllm.op_set_deterministic(False)
    if det:
        assert np.array_equal(outs[0], outs[1]), "non-deterministic result"
