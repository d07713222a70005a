// Decode attention, persistent + TMA (a7, decode rows) -- the default decode path.
//
//   decode row j (position L_j - 1) attends keys [0, L_j - 1]:  o = softmax(q K^T / sqrt(D)) V
//   (decode is memory-bound; GQA: the G = Hq/Hkv query heads of a kv head
//   share every K/V page, so each page is read from HBM once per (row, kv head)).
//
// Work = (decode item, kv head) pairs, items longest-first (host, stage.cu).  Every WARP is an
// independent persistent worker: it claims work with one atomicAdd, and streams the item's
// 16-key pages (K 4 KB + V 4 KB at D = 128, one contiguous [16][D] tile each in the paged
// cache) through a private NST-slot ring in SMEM.  Lane 0 issues the loads as TMA tensor copies
// (SW128 boxes of 16 x 64) plus a 1-D bulk copy of the item's G query rows, completing on the
// slot's mbarrier; the page stream runs ahead ACROSS item boundaries, so the ring never drains
// between items (the v1 kernel, attention.cu, paid a fill + merge per CTA).  The G heads are
// the rows of an m16n8k16 tile: S = Q K^T (2 n-tiles x D/16 k-steps), online softmax with a
// lazy reference max (rescale only when the max grows by > 2^8), O += P V (D/8 n-tiles).
// A finished item writes bf16 rows, or (split rows) an fp32 partial merged by
// decode_merge_kernel.  The last CTA to finish resets the work counter for the next launch.
#include <cuda.h>
#include <cuda_bf16.h>

#include "attention.cuh"
#include "common.h"
#include "ptx.cuh"

namespace gllm {

namespace {

constexpr float LOG2E_D = 1.4426950408889634f;

__device__ __forceinline__ void bulk_load_1d(uint32_t smem_dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   smem_dst),
               "l"(reinterpret_cast<uint64_t>(src)), "r"(bytes), "r"(ptx::smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// (row, 16-byte chunk) of a 16-row page stored as D/64 SW128 atoms of 16 x 128 B (TMA box layout)
__device__ __forceinline__ uint32_t pg(int row, int chunk) {
  return (chunk >> 3) * 2048 + row * 128 + (((chunk & 7) ^ (row & 7)) << 4);
}

template <int D, int G, int NST, int WARPS>
struct DecLayout {
  static constexpr int PAGE = 16 * D * 2;          // one K (or V) page
  static constexpr int SLOT = 2 * PAGE;            // K page + V page
  static constexpr int QB = G * D * 2;             // the G query rows of one (row, kv head)
  static constexpr int RING = NST * SLOT;          // per warp
  static constexpr int QOFF = WARPS * RING;        // Q slots: [WARPS][NST][QB]
  static constexpr int META = QOFF + WARPS * NST * QB;  // int4 [WARPS][NST]
  static constexpr int BAR = META + WARPS * NST * 16;   // uint64 [WARPS][NST]
  static constexpr int BYTES = BAR + WARPS * NST * 8 + 1024;  // + 1024-B alignment slack
};

template <int D, int G, int NST, int WARPS>
__global__ void __launch_bounds__(WARPS * 32)
    decode_attn_tma_kernel(const AttnArgs a, const DecodeItem* __restrict__ items, int n_work, int* __restrict__ ctr,
                           const __grid_constant__ CUtensorMap tmk, const __grid_constant__ CUtensorMap tmv) {
  using Lay = DecLayout<D, G, NST, WARPS>;
  static_assert(G >= 1 && G <= 8, "GQA group must fit the 16-row MMA tile");
  constexpr int ATOMS = D / 64;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, tq = lane & 3;
  uint8_t* ring = smem + warp * Lay::RING;
  const uint32_t ring_u32 = ptx::smem_u32(ring);
  const uint32_t q_u32 = ptx::smem_u32(smem + Lay::QOFF + warp * NST * Lay::QB);
  const uint8_t* qbase = smem + Lay::QOFF + warp * NST * Lay::QB;
  int4* meta = reinterpret_cast<int4*>(smem + Lay::META) + warp * NST;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + Lay::BAR) + warp * NST;
  const int Hkv = a.Hkv;
  const float sl2 = LOG2E_D * rsqrtf((float)D);
  const uint64_t pol = ptx::policy_evict_first();  // each page is read once per layer

  if (lane == 0) {
    for (int s = 0; s < NST; ++s) ptx::mbar_init(&bar[s], 1);
    ptx::fence_barrier_init();
    if (warp == 0) {
      ptx::tma_prefetch(&tmk);
      ptx::tma_prefetch(&tmv);
    }
  }
  __syncwarp();

  // ---- issue side of the page stream (warp-uniform state; lane 0 issues)
  int iw = 0, ip = 0, inp = 0, iq = 0;  // work index, page within the item, pages of the item, Q slot
  int i_seq = 0, i_kvh = 0, i_nb0 = 0;
  auto fetch = [&]() {
    int v = 0;
    if (lane == 0) v = atomicAdd(ctr, 1);
    iw = __shfl_sync(0xffffffffu, v, 0);
    ip = 0;
    if (iw < n_work) {
      const DecodeItem it = items[iw / Hkv];
      i_kvh = iw % Hkv;
      i_seq = it.seq;
      const int L = a.kv_len[it.seq];
      const int k0 = it.split * a.split_len, k1 = min(L, k0 + a.split_len);
      i_nb0 = k0 / 16;
      inp = (k1 + 15) / 16 - i_nb0;
    }
  };
  auto issue = [&](int s) {
    if (iw >= n_work) {
      if (lane == 0) meta[s] = make_int4(-1, 0, 0, 0);
      return;
    }
    const int blk = a.block_table[(size_t)i_seq * a.maxblk + i_nb0 + ip];
    if (lane == 0) {
      const int row = (blk * Hkv + i_kvh) * 16;
      const bool first = ip == 0;
      fence_proxy_async();  // this slot's earlier generic reads (ldmatrix) before the async writes
      ptx::mbar_arrive_expect_tx(&bar[s], Lay::SLOT + (first ? Lay::QB : 0));
      uint8_t* dst = ring + s * Lay::SLOT;
#pragma unroll
      for (int at = 0; at < ATOMS; ++at) {
        ptx::tma_load_2d_hint(dst + at * 2048, &tmk, &bar[s], at * 64, row, pol);
        ptx::tma_load_2d_hint(dst + Lay::PAGE + at * 2048, &tmv, &bar[s], at * 64, row, pol);
      }
      if (first) {
        const int t = a.cu_q[i_seq];
        bulk_load_1d(q_u32 + iq * Lay::QB, a.q + (size_t)t * a.q_stride + (size_t)i_kvh * G * D, Lay::QB, &bar[s]);
      }
      meta[s] = make_int4(iw, ip, (ip == inp - 1 ? 1 : 0) | (first ? 2 : 0), iq);
    }
    if (++ip == inp) {
      iq = (iq + 1) % NST;
      fetch();
    }
  };

  fetch();
#pragma unroll 1
  for (int s = 0; s < NST - 1; ++s) issue(s);

  // ---- consume side
  uint32_t qa[D / 16][4];
  float o[D / 8][4];
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};
  int c_seq = 0, c_kvh = 0, c_k1 = 0, c_nb0 = 0, c_part = -1;
#pragma unroll 1
  for (int i = 0;; ++i) {
    const int s = i % NST;
    issue((i + NST - 1) % NST);  // the slot consumed at iteration i - 1
    __syncwarp();
    const int4 mt = meta[s];
    if (mt.x < 0) break;
    ptx::mbar_wait(&bar[s], (uint32_t)((i / NST) & 1));
    if (mt.z & 2) {  // first page of a work item: its Q rows arrived with this page
      const DecodeItem it = items[mt.x / Hkv];
      c_kvh = mt.x % Hkv;
      c_seq = it.seq;
      const int L = a.kv_len[it.seq];
      const int k0 = it.split * a.split_len;
      c_k1 = min(L, k0 + a.split_len);
      c_nb0 = k0 / 16;
      c_part = it.part;
      const uint8_t* qs = qbase + mt.w * Lay::QB;
#pragma unroll
      for (int ks = 0; ks < D / 16; ++ks) {
        const int c0 = ks * 16 + 2 * tq;
        qa[ks][0] = g < G ? *reinterpret_cast<const uint32_t*>(qs + (g * D + c0) * 2) : 0u;
        qa[ks][1] = 0u;  // rows 8..15 (G <= 8)
        qa[ks][2] = g < G ? *reinterpret_cast<const uint32_t*>(qs + (g * D + c0 + 8) * 2) : 0u;
        qa[ks][3] = 0u;
      }
#pragma unroll
      for (int n = 0; n < D / 8; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
      mrow[0] = mrow[1] = -INFINITY;
      lrow[0] = lrow[1] = 0.f;
    }
    const uint32_t kst = ring_u32 + s * Lay::SLOT;
    const uint32_t vst = kst + Lay::PAGE;
    float sc[2][4] = {{0.f, 0.f, 0.f, 0.f}, {0.f, 0.f, 0.f, 0.f}};
#pragma unroll
    for (int ks = 0; ks < D / 16; ++ks) {
      uint32_t b0, b1, b2, b3;
      ptx::ldsm_x4(kst + pg(((lane >> 4) << 3) + (lane & 7), ks * 2 + ((lane >> 3) & 1)), b0, b1, b2, b3);
      ptx::mma_bf16_16816(sc[0], qa[ks], b0, b1);
      ptx::mma_bf16_16816(sc[1], qa[ks], b2, b3);
    }
    const int kbase = (c_nb0 + mt.y) * 16;
#pragma unroll
    for (int n = 0; n < 2; ++n)
#pragma unroll
      for (int e = 0; e < 4; ++e) sc[n][e] = (kbase + n * 8 + 2 * tq + (e & 1) < c_k1) ? sc[n][e] * sl2 : -INFINITY;
    // rows 8..15 are padding (G <= 8): only the first half-row set carries heads
    float corr = 1.f;
    bool rescale = false;
    {
      float mx = fmaxf(fmaxf(sc[0][0], sc[0][1]), fmaxf(sc[1][0], sc[1][1]));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 1));
      mx = fmaxf(mx, __shfl_xor_sync(0xffffffffu, mx, 2));
      if (mx > mrow[0] + 8.f) {
        corr = exp2f(mrow[0] - mx);
        mrow[0] = mx;
        lrow[0] *= corr;
        rescale = true;
      }
      const float mn = mrow[0];
      sc[0][0] = exp2f(sc[0][0] - mn);
      sc[0][1] = exp2f(sc[0][1] - mn);
      sc[1][0] = exp2f(sc[1][0] - mn);
      sc[1][1] = exp2f(sc[1][1] - mn);
      lrow[0] += sc[0][0] + sc[0][1] + sc[1][0] + sc[1][1];
    }
    if (__any_sync(0xffffffffu, rescale)) {
#pragma unroll
      for (int n = 0; n < D / 8; ++n) {
        o[n][0] *= corr;
        o[n][1] *= corr;
      }
    }
    uint32_t pa[4];
    pa[0] = ptx::pack_bf16(sc[0][0], sc[0][1]);
    pa[1] = 0u;
    pa[2] = ptx::pack_bf16(sc[1][0], sc[1][1]);
    pa[3] = 0u;
#pragma unroll
    for (int dp = 0; dp < D / 16; ++dp) {
      uint32_t b0, b1, b2, b3;
      ptx::ldsm_x4_t(vst + pg((lane & 7) + (((lane >> 3) & 1) << 3), dp * 2 + (lane >> 4)), b0, b1, b2, b3);
      ptx::mma_bf16_16816(o[2 * dp], pa, b0, b1);
      ptx::mma_bf16_16816(o[2 * dp + 1], pa, b2, b3);
    }
    if (mt.z & 1) {  // last page of the item: finish the G rows
      float l = lrow[0];
      l += __shfl_xor_sync(0xffffffffu, l, 1);
      l += __shfl_xor_sync(0xffffffffu, l, 2);
      if (g < G) {
        const int t = a.cu_q[c_seq];
        if (c_part < 0) {
          const float inv = 1.f / l;
          __nv_bfloat16* orow = a.out + (size_t)t * a.Hq * D + (size_t)(c_kvh * G + g) * D;
#pragma unroll
          for (int n = 0; n < D / 8; ++n)
            *reinterpret_cast<uint32_t*>(orow + n * 8 + 2 * tq) = ptx::pack_bf16(o[n][0] * inv, o[n][1] * inv);
        } else {
          const size_t base = ((size_t)c_part * Hkv + c_kvh) * G + g;
#pragma unroll
          for (int n = 0; n < D / 8; ++n)
            *reinterpret_cast<float2*>(a.part_o + base * D + n * 8 + 2 * tq) = make_float2(o[n][0], o[n][1]);
          if (tq == 0) {
            a.part_ml[base * 2] = mrow[0];
            a.part_ml[base * 2 + 1] = l;
          }
        }
      }
    }
    __syncwarp();  // all lanes done reading slot s before it is refilled
  }
  // the last CTA out resets the work counter for the next launch on this stream
  __syncthreads();
  if (threadIdx.x == 0) {
    __threadfence();
    const int done = atomicAdd(ctr + 1, 1);
    if (done == (int)gridDim.x - 1) {
      ctr[0] = 0;
      ctr[1] = 0;
      __threadfence();
    }
  }
}

template <int D, int G>
__global__ void __launch_bounds__(128) decode_merge2_kernel(const AttnArgs a, const MergeItem* __restrict__ merges) {
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

int g_dec_warps = 0;  // GLLM_DECODE_WARPS (A/B): warps per CTA, 4 (default) or 8

template <int D, int G, int NST, int WARPS>
int launch_t(const AttnArgs& a, const CUtensorMap& tmk, const CUtensorMap& tmv, const DecodeItem* items,
             int n_items, const MergeItem* merges, int n_merges, int* ctr, int num_sms, cudaStream_t s) {
  using Lay = DecLayout<D, G, NST, WARPS>;
  static int per_sm = 0;
  if (!per_sm) {
    cudaFuncSetAttribute(decode_attn_tma_kernel<D, G, NST, WARPS>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                         Lay::BYTES);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, decode_attn_tma_kernel<D, G, NST, WARPS>, WARPS * 32,
                                                  Lay::BYTES);
    if (per_sm < 1) per_sm = 1;
  }
  const int n_work = n_items * a.Hkv;
  if (n_work > 0) {
    int grid = per_sm * num_sms;
    const int need = (n_work + WARPS - 1) / WARPS;
    if (grid > need) grid = need;
    decode_attn_tma_kernel<D, G, NST, WARPS><<<grid, WARPS * 32, Lay::BYTES, s>>>(a, items, n_work, ctr, tmk, tmv);
  }
  if (n_merges > 0) decode_merge2_kernel<D, G><<<dim3(n_merges, a.Hkv), 128, 0, s>>>(a, merges);
  return GLLM_OK;
}

template <int D, int G>
int launch_g(const AttnArgs& a, const CUtensorMap& tmk, const CUtensorMap& tmv, const DecodeItem* items, int n_items,
             const MergeItem* merges, int n_merges, int* ctr, int num_sms, cudaStream_t s) {
  if (g_dec_warps == 8) return launch_t<D, G, 3, 8>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
  if (g_dec_warps == 2) return launch_t<D, G, 4, 2>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
  return launch_t<D, G, 3, 4>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
}

template <int D>
int launch_d(const AttnArgs& a, const CUtensorMap& tmk, const CUtensorMap& tmv, const DecodeItem* items, int n_items,
             const MergeItem* merges, int n_merges, int* ctr, int num_sms, cudaStream_t s) {
  switch (a.Hq / a.Hkv) {
    case 1: return launch_g<D, 1>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 2: return launch_g<D, 2>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 4: return launch_g<D, 4>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 5: return launch_g<D, 5>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 8: return launch_g<D, 8>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
  }
  return set_error(GLLM_EINVAL, "decode attention (tma): unsupported GQA group %d", a.Hq / a.Hkv);
}

}  // namespace

bool decode_tma_supported(int D, int G) { return (D == 64 || D == 128) && (G == 1 || G == 2 || G == 4 || G == 5 || G == 8); }

void set_decode_warps(int w) { g_dec_warps = w; }

int launch_decode_attention_tma(const AttnArgs& a, const CUtensorMap& tmk, const CUtensorMap& tmv,
                                const DecodeItem* items, int n_items, const MergeItem* merges, int n_merges, int* ctr,
                                int num_sms, cudaStream_t s) {
  int rc;
  if (a.bs != 16) return set_error(GLLM_EINVAL, "decode attention (tma): block size %d != 16", a.bs);
  if (a.D == 128)
    rc = launch_d<128>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
  else if (a.D == 64)
    rc = launch_d<64>(a, tmk, tmv, items, n_items, merges, n_merges, ctr, num_sms, s);
  else
    return set_error(GLLM_EINVAL, "decode attention (tma): head_dim %d unsupported", a.D);
  if (rc) return rc;
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK : set_error(GLLM_ECUDA, "decode attention launch: %s", cudaGetErrorString(e));
}

}  // namespace gllm
