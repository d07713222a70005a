/* gllm_ops.h -- kernel-level entry points of libgllm.so, for parity tests and micro-benchmarks
 * of the hot ops outside a stage.  Same conventions as gllm.h (int status, gllm_last_error).
 * All pointers are device pointers of the current CUDA device; `stream` is a cudaStream_t
 * (NULL = legacy default stream); calls are asynchronous. */
#ifndef GLLM_OPS_H
#define GLLM_OPS_H

#include "gllm.h"

#ifdef __cplusplus
extern "C" {
#endif

/* The stage's projection GEMM (tcgen05): Y = A . W^T (a5, a8, a9, a10, a11).
 *   A   bf16 [M, K] row-major (activations), W bf16 [N, K] row-major (weights, nn.Linear layout)
 *   epi 0: out bf16 [M, N]  = Y (+ bias[N] if bias != NULL)
 *       1: out fp32 [M, N] += Y                          (residual add)
 *       2: out bf16 [M, N/2] = silu(Y_gate) * Y_up where W's rows are interleaved in blocks of
 *          128: rows [256j, 256j+128) = gate rows [128j, ...), rows [256j+128, 256j+256) = up rows
 *       3: out int32 [M]     = argmax_n Y[m, n] (lowest n on ties; greedy LM head)
 * Constraints: K % 64 == 0, N % 32 == 0 (N % 256 == 0 for epi 2), M >= 0; rows beyond M are
 * never touched.  A temporary workspace is allocated and freed for epi 3 / stream-K.
 * Returns GLLM_EINVAL on bad shapes, GLLM_ECUDA on launch errors. */
GLLM_API int gllm_op_gemm(const void* A, const void* W, int32_t M, int32_t N, int32_t K, int32_t epi,
                          const float* bias, void* out, void* stream);

/* Testing / tuning knob for every GEMM the library launches afterwards (process-wide):
 * 0 = automatic, 1 = force the 1-CTA 128x256 kernel, 2 = force the CTA-pair 256x256 kernel. */
GLLM_API int gllm_op_set_gemm_variant(int32_t cta_group);

/* gllm_op_gemm calls afterwards (process-wide): 1 = schedules with a fixed reduction order (no
 * stream-K / hybrid atomics; as gllm_stage_set_deterministic), 0 = automatic (default). */
GLLM_API int gllm_op_set_deterministic(int32_t on);

#ifdef __cplusplus
}
#endif
#endif /* GLLM_OPS_H */
