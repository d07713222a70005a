// Prefill (chunked, causal, paged) attention on tensor cores -- part of a7.
//
//   chunk i: c_i query tokens at offset s_i; token j attends keys [0, s_i + j] of its sequence,
//   read from the paged cache (the chunk's own keys were appended by the QKV epilogue).
//
// CTA = 128 flattened (token, group-head) rows of one chunk x one kv head, 8 warps x 16 rows,
// so the G query heads sharing a kv head reuse every K/V tile.  64-key K/V tiles (4 pages)
// are double-buffered in SMEM with cp.async (XOR-swizzled rows, conflict-free ldmatrix);
// S = Q K^T and O += P V run on mma.sync m16n8k16 (bf16 in, fp32 accumulate) with the online
// softmax in registers.  Q fragments are re-read from SMEM each tile (fewer registers -> two
// CTAs per SM), and 8-key n-tiles / 16-key k-steps entirely above a warp's causal diagonal
// are skipped (their probabilities are exactly 0).
#include <cuda_bf16.h>

#include "attention.cuh"
#include "common.h"
#include "ptx.cuh"

namespace gllm {

namespace {

constexpr float LOG2E_P = 1.4426950408889634f;
constexpr int PF_ROWS = 128;   // flattened rows per CTA
constexpr int PF_WARPS = 8;
constexpr int PF_KEYS = 64;    // keys per tile

template <int D>
__device__ __forceinline__ uint32_t pswz(int row, int chunk) {
  return row * (D * 2) + ((chunk ^ (row & 7)) << 4);
}

template <int D>
struct PfSmem {
  static constexpr int Q_BYTES = PF_ROWS * D * 2;
  static constexpr int T_BYTES = PF_KEYS * D * 2;
  static constexpr int BYTES = Q_BYTES + 4 * T_BYTES;  // Q + 2 x (K, V)
};

template <int D>
__global__ void __launch_bounds__(PF_WARPS * 32, 2)
    prefill_attn_kernel(const AttnArgs a, const PrefillItem* __restrict__ items) {
  constexpr int NCH = D / 8;
  extern __shared__ __align__(128) uint8_t smem[];
  const uint32_t sQ = ptx::smem_u32(smem);
  const uint32_t sKV = sQ + PfSmem<D>::Q_BYTES;  // buffer b: K at sKV + 2b T, V at sKV + (2b+1) T
  constexpr int TB = PfSmem<D>::T_BYTES;

  const PrefillItem it = items[blockIdx.x];
  const int kvh = blockIdx.y;
  const int G = a.Hq / a.Hkv;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int t0 = a.cu_q[it.seq];
  const int c = a.cu_q[it.seq + 1] - t0;
  const int s0 = a.kv_len[it.seq] - c;
  const int nrows = c * G;
  const int max_pos = s0 + min(it.row0 + PF_ROWS - 1, nrows - 1) / G;
  const int n_kt = (max_pos + PF_KEYS) / PF_KEYS;
  const int nblk_seq = (a.kv_len[it.seq] + 15) / 16;
  const int32_t* bt = a.block_table + (size_t)it.seq * a.maxblk;
  const float sl2 = LOG2E_P * rsqrtf((float)D);

  for (int idx = threadIdx.x; idx < PF_ROWS * NCH; idx += blockDim.x) {
    const int r = idx / NCH, ch = idx % NCH;
    const int rr = min(it.row0 + r, nrows - 1);
    const int tok = rr / G, h = kvh * G + rr % G;
    ptx::cp_async16(sQ + pswz<D>(r, ch), a.q + (size_t)(t0 + tok) * a.q_stride + (size_t)h * D + ch * 8, true);
  }
  auto load_kv = [&](int kt, int buf) {
    const uint32_t kb = sKV + 2 * buf * TB, vb = kb + TB;
    for (int idx = threadIdx.x; idx < PF_KEYS * NCH; idx += blockDim.x) {
      const int r = idx / NCH, ch = idx % NCH;
      const int key = kt * PF_KEYS + r;
      const int blk = key >> 4;
      const bool ok = blk < nblk_seq;
      const size_t page = ok ? (size_t)bt[blk] : 0;
      const size_t off = ((page * a.Hkv + kvh) * 16 + (key & 15)) * D + ch * 8;
      ptx::cp_async16(kb + pswz<D>(r, ch), a.kc + off, ok);
      ptx::cp_async16(vb + pswz<D>(r, ch), a.vc + off, ok);
    }
  };
  load_kv(0, 0);
  ptx::cp_async_commit();

  const int g = lane >> 2, tq = lane & 3;
  const int wrow0 = it.row0 + warp * 16;  // first flattened row of this warp
  const bool warp_live = wrow0 < nrows;
  int pos_r[2];
#pragma unroll
  for (int hr = 0; hr < 2; ++hr) pos_r[hr] = s0 + min(wrow0 + g + hr * 8, nrows - 1) / G;
  const int wpos_min = s0 + min(wrow0, nrows - 1) / G;
  const int wpos_max = s0 + min(wrow0 + 15, nrows - 1) / G;

  float o[D / 8][4];
#pragma unroll
  for (int n = 0; n < D / 8; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};

  for (int kt = 0; kt < n_kt; ++kt) {
    if (kt + 1 < n_kt) load_kv(kt + 1, (kt + 1) & 1);
    ptx::cp_async_commit();
    ptx::cp_async_wait<1>();
    __syncthreads();
    const int key0 = kt * PF_KEYS;
    if (warp_live && key0 <= wpos_max) {
      const uint32_t kb = sKV + 2 * (kt & 1) * TB, vb = kb + TB;
      const int n_np = min(4, (wpos_max - key0) / 16 + 1);  // 16-key groups with any visible key
      float s[8][4];
#pragma unroll
      for (int n = 0; n < 8; ++n) s[n][0] = s[n][1] = s[n][2] = s[n][3] = 0.f;
#pragma unroll
      for (int ks = 0; ks < D / 16; ++ks) {
        uint32_t qa[4];
        ptx::ldsm_x4(sQ + pswz<D>(warp * 16 + (lane & 15), ks * 2 + (lane >> 4)), qa[0], qa[1], qa[2], qa[3]);
#pragma unroll
        for (int np = 0; np < 4; ++np) {
          if (np < n_np) {
            uint32_t b0, b1, b2, b3;
            ptx::ldsm_x4(kb + pswz<D>(np * 16 + ((lane >> 4) << 3) + (lane & 7), ks * 2 + ((lane >> 3) & 1)), b0, b1,
                         b2, b3);
            ptx::mma_bf16_16816(s[2 * np], qa, b0, b1);
            ptx::mma_bf16_16816(s[2 * np + 1], qa, b2, b3);
          }
        }
      }
      const bool need_mask = key0 + PF_KEYS - 1 > wpos_min;
#pragma unroll
      for (int n = 0; n < 8; ++n)
#pragma unroll
        for (int e = 0; e < 4; ++e) {
          const int key = key0 + n * 8 + 2 * tq + (e & 1);
          s[n][e] = (need_mask && key > pos_r[e >> 1]) ? -INFINITY : s[n][e] * sl2;
        }
      float corr[2];
#pragma unroll
      for (int hr = 0; hr < 2; ++hr) {
        float mx = -INFINITY;
#pragma unroll
        for (int n = 0; n < 8; ++n) mx = fmaxf(mx, fmaxf(s[n][2 * hr], s[n][2 * hr + 1]));
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
        mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
        const float mn = fmaxf(mrow[hr], mx);
        corr[hr] = exp2f(mrow[hr] - mn);
        mrow[hr] = mn;
        float sum = 0.f;
#pragma unroll
        for (int n = 0; n < 8; ++n) {
          s[n][2 * hr] = exp2f(s[n][2 * hr] - mn);
          s[n][2 * hr + 1] = exp2f(s[n][2 * hr + 1] - mn);
          sum += s[n][2 * hr] + s[n][2 * hr + 1];
        }
        lrow[hr] = lrow[hr] * corr[hr] + sum;
      }
#pragma unroll
      for (int n = 0; n < D / 8; ++n) {
        o[n][0] *= corr[0];
        o[n][1] *= corr[0];
        o[n][2] *= corr[1];
        o[n][3] *= corr[1];
      }
#pragma unroll
      for (int kk = 0; kk < 4; ++kk) {
        if (kk < n_np) {
          uint32_t pa[4];
          pa[0] = ptx::pack_bf16(s[2 * kk][0], s[2 * kk][1]);
          pa[1] = ptx::pack_bf16(s[2 * kk][2], s[2 * kk][3]);
          pa[2] = ptx::pack_bf16(s[2 * kk + 1][0], s[2 * kk + 1][1]);
          pa[3] = ptx::pack_bf16(s[2 * kk + 1][2], s[2 * kk + 1][3]);
#pragma unroll
          for (int dp = 0; dp < D / 16; ++dp) {
            uint32_t b0, b1, b2, b3;
            ptx::ldsm_x4_t(vb + pswz<D>(kk * 16 + (lane & 7) + (((lane >> 3) & 1) << 3), dp * 2 + (lane >> 4)), b0,
                           b1, b2, b3);
            ptx::mma_bf16_16816(o[2 * dp], pa, b0, b1);
            ptx::mma_bf16_16816(o[2 * dp + 1], pa, b2, b3);
          }
        }
      }
    }
    __syncthreads();
  }
  if (!warp_live) return;
#pragma unroll
  for (int hr = 0; hr < 2; ++hr) {
    float lt = lrow[hr];
    lt += __shfl_xor_sync(0xffffffffu, lt, 1);
    lt += __shfl_xor_sync(0xffffffffu, lt, 2);
    const float inv = 1.f / lt;
    const int rr = wrow0 + g + hr * 8;
    if (rr < nrows) {
      const int tok = rr / G, h = kvh * G + rr % G;
      __nv_bfloat16* dst = a.out + (size_t)(t0 + tok) * a.Hq * D + (size_t)h * D;
#pragma unroll
      for (int n = 0; n < D / 8; ++n)
        *reinterpret_cast<uint32_t*>(dst + n * 8 + 2 * tq) = ptx::pack_bf16(o[n][2 * hr] * inv, o[n][2 * hr + 1] * inv);
    }
  }
}

template <int D>
int launch_prefill_d(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s) {
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(prefill_attn_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, PfSmem<D>::BYTES);
    set = true;
  }
  prefill_attn_kernel<D><<<dim3(n_items, a.Hkv), PF_WARPS * 32, PfSmem<D>::BYTES, s>>>(a, items);
  return GLLM_OK;
}

}  // namespace

int prefill_rows_per_item() { return PF_ROWS; }

int launch_prefill_attention(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s) {
  if (n_items <= 0) return GLLM_OK;
  if (a.D == 128)
    launch_prefill_d<128>(a, items, n_items, s);
  else if (a.D == 64)
    launch_prefill_d<64>(a, items, n_items, s);
  else
    return set_error(GLLM_EINVAL, "prefill attention: head_dim %d unsupported", a.D);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK : set_error(GLLM_ECUDA, "prefill attention launch: %s", cudaGetErrorString(e));
}

}  // namespace gllm
