// Launchers of the bandwidth-bound kernels of the stage forward (internal interface).
#pragma once
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace gllm {

// O4 weight generator: logical [rows, cols] tensor `tid` written
// as bf16 at physical row phys(row) of `dst` (row stride = cols).
//   mode 0: phys = row + row_offset          (fused QKV: q, k, v stacked)
//   mode 1: phys = (row/128)*256 + row%128   (gate rows of the interleaved gate|up)
//   mode 2: phys = (row/128)*256 + 128 + row%128   (up rows)
void launch_init_bf16(__nv_bfloat16* dst, int64_t rows, int64_t cols, uint64_t seed, uint64_t tid, float scale,
                      int mode, int64_t row_offset, cudaStream_t s, int tiled = 0);
void launch_init_f32(float* dst, int64_t n, uint64_t seed, uint64_t tid, float scale, cudaStream_t s);
void launch_fill_f32(float* dst, int64_t n, float v, cudaStream_t s);

// per-forward metadata: slot mapping (O2) and the RoPE cos/sin table for the batch positions
void launch_prep(const int32_t* positions, const int32_t* cu_q, const int32_t* block_table, int T, int S,
                 int maxblk, int block_size, int32_t* slots, float2* rope_cs, int head_dim, float rope_theta,
                 cudaStream_t s);

void launch_embed(const __nv_bfloat16* E, const int32_t* ids, float* x, int T, int H, cudaStream_t s);

// y[r] = bf16(x[row(r)] * rsqrt(mean(x^2) + eps) * g); row(r) = rows ? rows[r] : r
void launch_rmsnorm(const float* x, const float* g, __nv_bfloat16* y, const int32_t* rows, int n, int H, float eps,
                    cudaStream_t s);

// Fused-RMSNorm statistics (a4): xb[r] = bf16(x[r]) and ss[r] = sum(x[r]^2) (fp32); the
// consumer GEMM scales its output rows by rsqrt(ss/H + eps).  x_copy (optional) receives x (the
// stage-entry hand-off copy-in); rel_flag (optional): once every CTA has read its rows, the last one
// stores rel_val there with st.release.sys (peer-ring slot credit); rel_ctr = one zeroed counter.
void launch_rms_stats(const float* x, float* x_copy, __nv_bfloat16* xb, float* ss, int n, int H, uint32_t* rel_flag,
                      uint32_t rel_val, unsigned* rel_ctr, cudaStream_t s);

// (RoPE + paged K/V append run in the QKV GEMM epilogue, gemm.cu EPI_QKV_ROPE.)

// sampled[r] = argmax over n-tile partials (lowest id on ties, R18)
void launch_argmax_reduce(const float* part_val, const int32_t* part_idx, int rows, int ntiles, int32_t* out,
                          cudaStream_t s);

// warm-start KV (O4): positions [0, ctx[i]) of warm request req_ids[i] through block-table row i,
// K / V of one layer from tensor ids tid / tid + 1 (device arrays)
void launch_fill_warm_kv(__nv_bfloat16* kc, __nv_bfloat16* vc, const int64_t* req_ids, const int32_t* ctx,
                         const int32_t* bt, int n_seqs, int maxblk, int Hkv, int D, int bs, uint64_t seed,
                         uint64_t tid, cudaStream_t s);

}  // namespace gllm
