// Varlen paged causal attention (a7): prefill chunks and decode rows, both on tensor cores
// (mma.sync m16n8k16, bf16 in / fp32 accumulate), K/V pages streamed through SMEM with
// cp.async.
//
//   prefill chunk i (c_i tokens at offset s_i): token j attends keys [0, s_i + j]
//   decode row j (position L_j - 1):           attends keys [0, L_j - 1]
//   softmax(q k^T / sqrt(D)) v, GQA: q head h uses kv head h / G, G = Hq / Hkv
//
// Cache layout per layer: K, V each [kv_blocks][Hkv][16][D] bf16, so one
// (block, kv head) page is a contiguous 16 x D tile (4 KB at D = 128).
#include <cuda_bf16.h>

#include "attention.cuh"
#include "common.h"
#include "ptx.cuh"

namespace gllm {

namespace {

constexpr float LOG2E = 1.4426950408889634f;

// swizzled byte offset of (row, 16-byte chunk) in a row-major tile with D bf16 per row:
// chunk' = chunk ^ (row % 8) keeps the 8 rows an ldmatrix reads on distinct banks.
template <int D>
__device__ __forceinline__ uint32_t swz(int row, int chunk) {
  return row * (D * 2) + ((chunk ^ (row & 7)) << 4);
}

// ------------------------------------------------------------------ decode
// Bandwidth-bound: every decode row reads L x 2 x D x 2 bytes of K/V per kv head once.
// CTA = (decode row, key split) x kv head, 4 warps; warp w owns pages w, w+4, ... of the split
// with its own online-softmax state and a private NST-stage cp.async ring (K page + V page per
// stage), merged across warps at the end.  The G query heads of the kv head are the rows of
// a 16-row MMA tile (rows >= G are zero), so Q K^T of a 16-token page is 2 n-tiles x D/16
// k-steps and P V is 1 k-step x D/8 n-tiles -- no shuffles in the dot products.
template <int D>
struct DecodeSmem {
#ifdef GLLM_VARIANT_DEC3
  static constexpr int NST = 3;
#else
  // 2 stages (64 KB per CTA at D = 128): a prefill CTA (96 KB) still fits beside two decode CTAs
  static constexpr int NST = 2;
#endif
  static constexpr int PAGE = 16 * D * 2;
  static constexpr int PER_WARP = NST * 2 * PAGE;
  static constexpr int MERGE = 4 * 16 * D * 4 + 4 * 16 * 2 * 4;
  static constexpr int BYTES = (4 * PER_WARP > MERGE ? 4 * PER_WARP : MERGE);
};

template <int D, int G>
__global__ void __launch_bounds__(128) decode_attn_kernel(const AttnArgs a, const DecodeItem* __restrict__ items) {
  static_assert(G >= 1 && G <= 16, "GQA group must fit one 16-row MMA tile");
  constexpr int NCH = D / 8;
  constexpr int NST = DecodeSmem<D>::NST;
  constexpr int PAGE = DecodeSmem<D>::PAGE;
  extern __shared__ __align__(128) uint8_t smem[];

  const DecodeItem it = items[blockIdx.x];
  const int kvh = blockIdx.y;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, tq = lane & 3;
  const int t = a.cu_q[it.seq];
  const int L = a.kv_len[it.seq];
  const int k0 = it.split * a.split_len;
  const int k1 = min(L, k0 + a.split_len);
  const int nb0 = k0 / 16, nb1 = (k1 + 15) / 16;
  const int n_my = nb1 - nb0 > warp ? (nb1 - nb0 - warp + 3) / 4 : 0;
  const int32_t* bt = a.block_table + (size_t)it.seq * a.maxblk;
  const float sl2 = LOG2E * rsqrtf((float)D);
  uint8_t* ws = smem + warp * DecodeSmem<D>::PER_WARP;
  const uint32_t ws_u32 = ptx::smem_u32(ws);

  auto issue = [&](int i) {
    if (i < n_my) {
      const size_t page = (size_t)bt[nb0 + warp + 4 * i];
      const __nv_bfloat16* kp = a.kc + ((page * a.Hkv + kvh) * 16) * D;
      const __nv_bfloat16* vp = a.vc + ((page * a.Hkv + kvh) * 16) * D;
      const uint32_t st = ws_u32 + (i % NST) * 2 * PAGE;
#pragma unroll
      for (int j = 0; j < 16 * NCH / 32; ++j) {
        const int c = lane + 32 * j;
        const int r = c / NCH, ch = c % NCH;
        ptx::cp_async16(st + swz<D>(r, ch), kp + r * D + ch * 8, true);
        ptx::cp_async16(st + PAGE + swz<D>(r, ch), vp + r * D + ch * 8, true);
      }
    }
    ptx::cp_async_commit();  // always commit (possibly empty) so group counting stays uniform
  };
#pragma unroll
  for (int i = 0; i < NST - 1; ++i) issue(i);

  // Q fragments (rows = the G heads of this kv head; rows >= G are zero)
  uint32_t qa[D / 16][4];
  {
    const __nv_bfloat16* qrow = a.q + (size_t)t * a.q_stride + (size_t)kvh * G * D;
#pragma unroll
    for (int ks = 0; ks < D / 16; ++ks) {
      const int c0 = ks * 16 + 2 * tq;
      qa[ks][0] = g < G ? *reinterpret_cast<const uint32_t*>(qrow + g * D + c0) : 0u;
      qa[ks][1] = g + 8 < G ? *reinterpret_cast<const uint32_t*>(qrow + (g + 8) * D + c0) : 0u;
      qa[ks][2] = g < G ? *reinterpret_cast<const uint32_t*>(qrow + g * D + c0 + 8) : 0u;
      qa[ks][3] = g + 8 < G ? *reinterpret_cast<const uint32_t*>(qrow + (g + 8) * D + c0 + 8) : 0u;
    }
  }
  float o[D / 8][4];
#pragma unroll
  for (int n = 0; n < D / 8; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};

  for (int i = 0; i < n_my; ++i) {
    issue(i + NST - 1);
    ptx::cp_async_wait<NST - 1>();
    __syncwarp();
    const uint32_t kst = ws_u32 + (i % NST) * 2 * PAGE;
    const uint32_t vst = kst + PAGE;
    float s[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
#pragma unroll
    for (int ks = 0; ks < D / 16; ++ks) {
      uint32_t b0, b1, b2, b3;
      ptx::ldsm_x4(kst + swz<D>(((lane >> 4) << 3) + (lane & 7), ks * 2 + ((lane >> 3) & 1)), b0, b1, b2, b3);
      ptx::mma_bf16_16816(s[0], qa[ks], b0, b1);
      ptx::mma_bf16_16816(s[1], qa[ks], b2, b3);
    }
    const int kbase = (nb0 + warp + 4 * i) * 16;
#pragma unroll
    for (int n = 0; n < 2; ++n)
#pragma unroll
      for (int e = 0; e < 4; ++e) s[n][e] = (kbase + n * 8 + 2 * tq + (e & 1) < k1) ? s[n][e] * sl2 : -INFINITY;
    // online softmax with a lazy reference max: O and l are rescaled only when the running max
    // grows by more than 2^8 (exact: p, l and O share the reference), which removes the
    // per-page O rescale from the HBM-bound inner loop
    float corr[2];
    bool rescale = false;
#pragma unroll
    for (int hr = 0; hr < 2; ++hr) {
      float mx = fmaxf(fmaxf(s[0][2 * hr], s[0][2 * hr + 1]), fmaxf(s[1][2 * hr], s[1][2 * hr + 1]));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
      corr[hr] = 1.f;
      if (mx > mrow[hr] + 8.f) {
        corr[hr] = exp2f(mrow[hr] - mx);
        mrow[hr] = mx;
        lrow[hr] *= corr[hr];
        rescale = true;
      }
      const float mn = mrow[hr];
      float sum = 0.f;
#pragma unroll
      for (int n = 0; n < 2; ++n) {
        s[n][2 * hr] = exp2f(s[n][2 * hr] - mn);
        s[n][2 * hr + 1] = exp2f(s[n][2 * hr + 1] - mn);
        sum += s[n][2 * hr] + s[n][2 * hr + 1];
      }
      lrow[hr] += sum;
    }
    if (rescale) {
#pragma unroll
      for (int n = 0; n < D / 8; ++n) {
        o[n][0] *= corr[0];
        o[n][1] *= corr[0];
        o[n][2] *= corr[1];
        o[n][3] *= corr[1];
      }
    }
    uint32_t pa[4];
    pa[0] = ptx::pack_bf16(s[0][0], s[0][1]);
    pa[1] = ptx::pack_bf16(s[0][2], s[0][3]);
    pa[2] = ptx::pack_bf16(s[1][0], s[1][1]);
    pa[3] = ptx::pack_bf16(s[1][2], s[1][3]);
#pragma unroll
    for (int dp = 0; dp < D / 16; ++dp) {
      uint32_t b0, b1, b2, b3;
      ptx::ldsm_x4_t(vst + swz<D>((lane & 7) + (((lane >> 3) & 1) << 3), dp * 2 + (lane >> 4)), b0, b1, b2, b3);
      ptx::mma_bf16_16816(o[2 * dp], pa, b0, b1);
      ptx::mma_bf16_16816(o[2 * dp + 1], pa, b2, b3);
    }
    __syncwarp();  // everyone done reading this stage before it is refilled
  }
  ptx::cp_async_wait<0>();
#pragma unroll
  for (int hr = 0; hr < 2; ++hr) {
    lrow[hr] += __shfl_xor_sync(0xffffffffu, lrow[hr], 1);
    lrow[hr] += __shfl_xor_sync(0xffffffffu, lrow[hr], 2);
  }
  // ---- merge the 4 warps (SMEM reused)
  __syncthreads();
  float* sm_o = reinterpret_cast<float*>(smem);         // [4][16][D]
  float* sm_ml = sm_o + 4 * 16 * D;                      // [4][16][2]
#pragma unroll
  for (int hr = 0; hr < 2; ++hr) {
    const int r = g + 8 * hr;
    if (r < G) {
#pragma unroll
      for (int n = 0; n < D / 8; ++n) {
        sm_o[(warp * 16 + r) * D + n * 8 + 2 * tq] = o[n][2 * hr];
        sm_o[(warp * 16 + r) * D + n * 8 + 2 * tq + 1] = o[n][2 * hr + 1];
      }
      if (tq == 0) {
        sm_ml[(warp * 16 + r) * 2] = mrow[hr];
        sm_ml[(warp * 16 + r) * 2 + 1] = lrow[hr];
      }
    }
  }
  __syncthreads();
  for (int idx = threadIdx.x; idx < G * D; idx += blockDim.x) {
    const int h = idx / D, d = idx % D;
    float M = -INFINITY;
#pragma unroll
    for (int w = 0; w < 4; ++w) M = fmaxf(M, sm_ml[(w * 16 + h) * 2]);
    float Ls = 0.f, A = 0.f;
#pragma unroll
    for (int w = 0; w < 4; ++w) {
      const float f = exp2f(sm_ml[(w * 16 + h) * 2] - M);
      Ls += sm_ml[(w * 16 + h) * 2 + 1] * f;
      A += sm_o[(w * 16 + h) * D + d] * f;
    }
    if (it.part < 0) {
      a.out[(size_t)t * a.Hq * D + (size_t)(kvh * G + h) * D + d] = __float2bfloat16_rn(A / Ls);
    } else {
      const size_t base = ((size_t)it.part * a.Hkv + kvh) * G + h;
      a.part_o[base * D + d] = A;
      if (d == 0) {
        a.part_ml[base * 2] = M;
        a.part_ml[base * 2 + 1] = Ls;
      }
    }
  }
}

template <int D, int G>
__global__ void __launch_bounds__(128) decode_merge_kernel(const AttnArgs a, const MergeItem* __restrict__ merges) {
  const MergeItem mi = merges[blockIdx.x];
  const int kvh = blockIdx.y;
  const int t = a.cu_q[mi.seq];
  for (int idx = threadIdx.x; idx < G * D; idx += blockDim.x) {
    const int h = idx / D, d = idx % D;
    float M = -INFINITY;
    for (int s = 0; s < mi.nsplit; ++s)
      M = fmaxf(M, a.part_ml[(((size_t)(mi.first + s) * a.Hkv + kvh) * G + h) * 2]);
    float Ls = 0.f, A = 0.f;
    for (int s = 0; s < mi.nsplit; ++s) {
      const size_t base = ((size_t)(mi.first + s) * a.Hkv + kvh) * G + h;
      const float f = exp2f(a.part_ml[base * 2] - M);
      Ls += a.part_ml[base * 2 + 1] * f;
      A += a.part_o[base * D + d] * f;
    }
    a.out[(size_t)t * a.Hq * D + (size_t)(kvh * G + h) * D + d] = __float2bfloat16_rn(A / Ls);
  }
}

template <int D, int G>
int launch_decode_t(const AttnArgs& a, const DecodeItem* items, int n_items, const MergeItem* merges, int n_merges,
                    cudaStream_t s) {
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(decode_attn_kernel<D, G>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         DecodeSmem<D>::BYTES);
    set = true;
  }
  if (n_items > 0) decode_attn_kernel<D, G><<<dim3(n_items, a.Hkv), 128, DecodeSmem<D>::BYTES, s>>>(a, items);
  if (n_merges > 0) decode_merge_kernel<D, G><<<dim3(n_merges, a.Hkv), 128, 0, s>>>(a, merges);
  return GLLM_OK;
}

template <int D>
int launch_decode_d(const AttnArgs& a, const DecodeItem* items, int n_items, const MergeItem* merges, int n_merges,
                    cudaStream_t s) {
  switch (a.Hq / a.Hkv) {
    case 1: return launch_decode_t<D, 1>(a, items, n_items, merges, n_merges, s);
    case 2: return launch_decode_t<D, 2>(a, items, n_items, merges, n_merges, s);
    case 4: return launch_decode_t<D, 4>(a, items, n_items, merges, n_merges, s);
    case 5: return launch_decode_t<D, 5>(a, items, n_items, merges, n_merges, s);
    case 8: return launch_decode_t<D, 8>(a, items, n_items, merges, n_merges, s);
  }
  return set_error(GLLM_EINVAL, "decode attention: unsupported GQA group %d", a.Hq / a.Hkv);
}

}  // namespace

int launch_decode_attention(const AttnArgs& a, const DecodeItem* items, int n_items, const MergeItem* merges,
                            int n_merges, cudaStream_t s) {
  int rc;
  if (a.D == 128)
    rc = launch_decode_d<128>(a, items, n_items, merges, n_merges, s);
  else if (a.D == 64)
    rc = launch_decode_d<64>(a, items, n_items, merges, n_merges, s);
  else
    return set_error(GLLM_EINVAL, "decode attention: head_dim %d unsupported", a.D);
  if (rc) return rc;
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK : set_error(GLLM_ECUDA, "decode attention launch: %s", cudaGetErrorString(e));
}

}  // namespace gllm
