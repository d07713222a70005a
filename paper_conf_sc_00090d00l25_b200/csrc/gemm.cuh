// tcgen05 GEMM  Y[M,N] = X[M,K] . W[N,K]^T  with fused epilogues (internal interface).
#pragma once
#include <cuda.h>
#include <cuda_bf16.h>
#include <cuda_runtime.h>
#include <stdint.h>

namespace gllm {

enum GemmEpi : int {
  EPI_STORE_BF16 = 0,  // out bf16 [M, ldo] = acc (+ bias[col] if bias)
  EPI_ADD_F32 = 1,     // out fp32 [M, ldo] += acc          (residual add, a8 / a10)
  EPI_SILU_MUL = 2,    // out bf16 [M, ldo] = silu(gate) * up; W rows interleaved per 128 (a9)
  EPI_ARGMAX = 3,      // per (row, n-tile) max & argmax of acc -> partial buffers (a11)
  EPI_QKV_ROPE = 4,    // fused QKV epilogue (a5+a6): (+bias) RoPE on q -> out, RoPE on k and v -> paged cache
};

struct GemmArgs {
  int M, N, K;
  void* out;
  int ldo;
  const float* bias;
  float* part_val;   // EPI_ARGMAX: [M, num_n_tiles]
  int32_t* part_idx; // EPI_ARGMAX: [M, num_n_tiles]
  int num_m_tiles, num_n_tiles;
  // EPI_QKV_ROPE
  const float2* rope_cs;  // [M, head_dim/2] (cos, sin) of each row's position
  const int32_t* slots;   // [M] cache slot of each row
  __nv_bfloat16* kc;      // [kv_blocks][n_kv_heads][block_size][head_dim]
  __nv_bfloat16* vc;
  int q_dim, kv_dim, head_dim, n_kv_heads, block_size;
  // scheduling (filled by launch_gemm): 0 = one CTA per 128x256 tile (persistent round robin);
  // 1 = stream-K: CTA i owns k-block units [i*units_per_cta, (i+1)*units_per_cta) of the
  // (tile, k-block) space; partial tiles combine with fp32 atomics into `out` (EPI_ADD_F32) or
  // into the fp32 workspace `ws` [M, N], finished by gemm_finish_kernel.
  // 2 = hybrid (CTA pairs, residual add only): whole tiles [0, dp_tiles) round robin, then
  // stream-K over the remaining tiles' k-blocks (units_per_cta per pair), partial tiles reduced.
  // 3 = cluster split-K (CG=1, M <= 128, few tiles): each tile's k-blocks are split evenly over a
  // cluster of split_s CTAs; partial accumulators meet in shared memory and every CTA reduces its
  // share of the tile's column chunks over DSMEM in fixed rank order and runs the epilogue
  // (no atomics, no workspace, no finish pass; deterministic).
  int streamk, units_per_cta, dp_tiles, split_s;
  // B (the weights) is never written by a kernel on the stream: with PDL the producer issues the
  // first ring fill's B tiles before griddepcontrol.wait (stage GEMMs only; gllm_op_gemm leaves 0)
  int b_static;
  // B is stored in the tiled weight layout (weight_tiled_index): each 128-row x 64-column block of
  // the K-major weight is 16 KB contiguous, and the B tensor map is the [blocks * 128, 64] view of
  // it (make_tmap_weight_tiled), so a B box is one contiguous DRAM run (stage weights only)
  int b_tiled;
  float* ws;  // fp32 [M, N] stream-K workspace of non-additive epilogues: zero on entry, left zero
  // 1: a schedule with a fixed reduction order (no stream-K / hybrid fp32 atomics; whole tiles or
  // cluster split-K): bitwise run-to-run reproducible results
  int deterministic;
  // fused RMSNorm (a4).  Consumers (EPI_STORE_BF16 / EPI_QKV_ROPE / EPI_SILU_MUL) read the bf16
  // copy of the residual as A and scale each output row by r = rsqrt(row_ss[row] * inv_h + eps)
  // (the norm gain is folded into W; it is exactly 1 for the O4 weights).  The producer
  // (EPI_ADD_F32, whole tiles) writes xb_out = bf16(x_new) and adds sum(x_new^2) into ss_out.
  const float* row_ss;
  float inv_h, eps;
  __nv_bfloat16* xb_out;
  float* ss_out;
  float* zero_rows;  // consumers: the n-tile-0 epilogue sets zero_rows[row] = 0 (resets the next ss_out)
  // EPI_ADD_F32, whole tiles: the updated residual rows are also stored to out_peer [M, ldo] (the
  // next pipeline stage's receive slot, NVLink peer memory) -- the fused stage hand-off (a12)
  float* out_peer;
  // set by launch_gemm: the CTA-pair residual-add kernel stages its whole tiles' residual through
  // shared memory with TMA (loads of x chunks ahead of the accumulator, stores of x and bf16(x))
  int res_tma;
};

// true if launch_gemm would combine partial tiles (stream-K) for this shape -- then the ADD_F32
// epilogue cannot produce xb_out / ss_out and the caller runs rms_stats instead
bool gemm_uses_streamk(int M, int N, int K, int epi, int num_sms, bool deterministic = false);

// fp32 workspace (elements) launch_gemm may need for a GEMM of this shape/epilogue (0 = none)
size_t gemm_workspace_elems(int M, int N, int K, int epi, int num_sms);

constexpr int GEMM_BM = 128, GEMM_BN = 256, GEMM_BK = 64, GEMM_STAGES = 4;
constexpr size_t GEMM_WS_ELEMS = size_t(8) << 20;  // stream-K fp32 workspace capacity (32 MB)
// TMA box rows of the B (weight) tensor maps: one 128-row half of a 256-wide N tile, so the same
// map serves the 1-CTA kernel (two loads per stage) and the CTA-pair kernel (one per CTA).
constexpr int GEMM_B_BOX = 128;
// testing / tuning: force the 1-CTA (1) or CTA-pair (2) kernel; 0 = automatic
extern int g_force_cg;

// Encodes a 2-D bf16 K-major tensor map (rows x cols, cols contiguous) with a
// (box_rows x 64) box and 128-byte swizzle.  Returns 0 or a GLLM_* error.
int make_tmap_bf16(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols, uint32_t box_rows);

// Tiled weight layout of the stage GEMMs' B operand: element (r, c) of a [rows, cols] K-major
// weight (cols % 64 == 0) lives at block (r / 128, c / 64) -- 128 x 64 row-major, 16 KB -- with the
// blocks of a 128-row slab consecutive along K.  weight_tiled_elems pads rows to a multiple of 128.
inline int64_t weight_tiled_index(int64_t r, int64_t c, int64_t cols) {
  return ((r >> 7) * (cols >> 6) + (c >> 6)) * 8192 + (r & 127) * 64 + (c & 63);
}
inline size_t weight_tiled_elems(int64_t rows, int64_t cols) { return (size_t)((rows + 127) / 128) * 128 * cols; }
// the [blocks * 128, 64] tensor map of a tiled weight (128-row box, 128-byte swizzle)
int make_tmap_weight_tiled(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols);

// Residual-epilogue tensor maps (EPI_ADD_F32): x fp32 [rows, cols] with a 128-row x 32-column box
// and 128-byte swizzle; bf16(x) [rows, cols] with a 128 x 32 box and 64-byte swizzle.
int make_tmap_res_f32(CUtensorMap* map, const float* base, uint64_t rows, uint64_t cols);
int make_tmap_res_bf16(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols);

// Launches the persistent GEMM on `stream`.  A map: box 128 rows; B map: box 256 rows.
// EPI_ADD_F32 needs tm_x (the residual `out`, make_tmap_res_f32) and, when xb_out is set, tm_xb
// (make_tmap_res_bf16 of xb_out); the other epilogues ignore them.
int launch_gemm(const CUtensorMap& a, const CUtensorMap& b, GemmEpi epi, const GemmArgs& args,
                cudaStream_t stream, int num_sms, const CUtensorMap* tm_x = nullptr,
                const CUtensorMap* tm_xb = nullptr);

int num_sms_of_current_device();

}  // namespace gllm
