// Kernel-level entry points (include/gllm_ops.h): the stage's GEMM outside a stage.
#include <cuda_runtime.h>

#include "common.h"
#include "gemm.cuh"
#include "gllm_ops.h"
#include "kernels.cuh"

extern "C" int gllm_op_set_gemm_variant(int32_t cta_group) {
  if (cta_group < 0 || cta_group > 2) return gllm::set_error(GLLM_EINVAL, "gemm variant must be 0, 1 or 2");
  gllm::g_force_cg = cta_group;
  return GLLM_OK;
}

static bool g_op_deterministic = false;

extern "C" int gllm_op_set_deterministic(int32_t on) {
  g_op_deterministic = on != 0;
  return GLLM_OK;
}

extern "C" int gllm_op_gemm(const void* A, const void* W, int32_t M, int32_t N, int32_t K, int32_t epi,
                            const float* bias, void* out, void* stream) {
  if (!A || !W || !out || M < 0 || N <= 0 || K <= 0) return gllm::set_error(GLLM_EINVAL, "op_gemm: bad arguments");
  if (K % 64 || N % 32 || (epi == gllm::EPI_SILU_MUL && N % 256) || epi < 0 || epi > gllm::EPI_ARGMAX)
    return gllm::set_error(GLLM_EINVAL, "op_gemm: unsupported shape/epilogue (M=%d N=%d K=%d epi=%d)", M, N, K, epi);
  if (M == 0) return GLLM_OK;
  cudaStream_t s = reinterpret_cast<cudaStream_t>(stream);
  CUtensorMap ta, tb;
  int rc;
  if ((rc = gllm::make_tmap_bf16(&ta, A, M, K, gllm::GEMM_BM)) || (rc = gllm::make_tmap_bf16(&tb, W, N, K, gllm::GEMM_B_BOX)))
    return rc;
  const int sms = gllm::num_sms_of_current_device();
  gllm::GemmArgs g{};
  g.M = M;
  g.N = N;
  g.K = K;
  g.out = out;
  g.ldo = epi == gllm::EPI_SILU_MUL ? N / 2 : N;
  g.bias = epi == gllm::EPI_STORE_BF16 ? bias : nullptr;
  g.deterministic = g_op_deterministic;
  const int ntn = (N + gllm::GEMM_BN - 1) / gllm::GEMM_BN;
  void* tmp = nullptr;
  const size_t ws_elems = g_op_deterministic ? 0 : gllm::gemm_workspace_elems(M, N, K, epi, sms);
  const size_t part_elems = epi == gllm::EPI_ARGMAX ? (size_t)M * ntn : 0;
  if (ws_elems) {  // stream-K: a process-wide fp32 workspace, zero between calls
    static float* ws = nullptr;
    static size_t ws_cap = 0;
    if (ws_cap < ws_elems) {
      if (ws) cudaFree(ws);
      ws_cap = 0;
      if (cudaMalloc(&ws, ws_elems * 4) != cudaSuccess || cudaMemset(ws, 0, ws_elems * 4) != cudaSuccess)
        return gllm::set_error(GLLM_ENOMEM, "op_gemm: workspace allocation failed");
      ws_cap = ws_elems;
    }
    g.ws = ws;
  }
  if (part_elems) {
    if (cudaMallocAsync(&tmp, 2 * part_elems * 4, s) != cudaSuccess)
      return gllm::set_error(GLLM_ENOMEM, "op_gemm: workspace allocation failed");
    g.part_val = static_cast<float*>(tmp);
    g.part_idx = reinterpret_cast<int32_t*>(g.part_val + part_elems);
  }
  if (epi == gllm::EPI_ARGMAX) g.out = nullptr;
  CUtensorMap tx{};
  if (epi == gllm::EPI_ADD_F32 && (rc = gllm::make_tmap_res_f32(&tx, static_cast<const float*>(out), M, N))) return rc;
  rc = gllm::launch_gemm(ta, tb, static_cast<gllm::GemmEpi>(epi), g, s, sms, epi == gllm::EPI_ADD_F32 ? &tx : nullptr);
  if (rc == GLLM_OK && epi == gllm::EPI_ARGMAX)
    gllm::launch_argmax_reduce(g.part_val, g.part_idx, M, ntn, static_cast<int32_t*>(out), s);
  if (tmp) cudaFreeAsync(tmp, s);
  if (rc) return rc;
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK : gllm::set_error(GLLM_ECUDA, "op_gemm: %s", cudaGetErrorString(e));
}
