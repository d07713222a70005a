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
// (SW128 boxes of 16 x 64) completing on the slot's mbarrier (the item's G query rows are read
// from global, L2-hot, when its first page is consumed); the page stream runs ahead ACROSS item
// boundaries, so the ring never drains
// between items (the v1 kernel, attention.cu, paid a fill + merge per CTA).  The G heads are
// the rows of an m16n8k16 tile: S = Q K^T (2 n-tiles x D/16 k-steps), online softmax with a
// lazy reference max (rescale only when the max grows by > 2^8), O += P V (D/8 n-tiles).
// A finished item writes bf16 rows, or (split rows) an fp32 partial; the last split of a row to
// finish merges the partials in place.  The last CTA to finish resets the work counter.
#include <cuda.h>
#include <cuda_bf16.h>

#include "attention.cuh"
#include "common.h"
#include "ptx.cuh"
#include "launch.cuh"

namespace gllm {

namespace {

constexpr float LOG2E_D = 1.4426950408889634f;

__device__ __forceinline__ void fence_proxy_async() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }

// (row, 16-byte chunk) of a 16-row page stored as D/64 SW128 atoms of 16 x 128 B (TMA box layout)
__device__ __forceinline__ uint32_t pg(int row, int chunk) {
  return (chunk >> 3) * 2048 + row * 128 + (((chunk & 7) ^ (row & 7)) << 4);
}

template <int D, int G, int NST, int WARPS>
struct DecLayout {
  static constexpr int PAGE = 16 * D * 2;          // one K (or V) page
  static constexpr int SLOT = 2 * PAGE;            // K page + V page
  static constexpr int RING = NST * SLOT;          // per warp
  static constexpr int META = WARPS * RING;        // int4 [WARPS][NST]
  static constexpr int BAR = META + WARPS * NST * 16;   // uint64 [WARPS][NST]
  static constexpr int BYTES = BAR + WARPS * NST * 8 + 1024;  // + 1024-B alignment slack
};

template <int D, int G, int NST, int WARPS>
__global__ void __launch_bounds__(WARPS * 32)
    decode_attn_tma_kernel(const AttnArgs a, const DecodeItem* __restrict__ items, int n_work, int* __restrict__ ctr) {
  using Lay = DecLayout<D, G, NST, WARPS>;
  static_assert(G >= 1 && G <= 8, "GQA group must fit the 16-row MMA tile");
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int g = lane >> 2, tq = lane & 3;
  uint8_t* ring = smem + warp * Lay::RING;
  const uint32_t ring_u32 = ptx::smem_u32(ring);
  int4* meta = reinterpret_cast<int4*>(smem + Lay::META) + warp * NST;
  uint64_t* bar = reinterpret_cast<uint64_t*>(smem + Lay::BAR) + warp * NST;
  const int Hkv = a.Hkv;
  const float sl2 = LOG2E_D * rsqrtf((float)D);
  const uint64_t pol = ptx::policy_evict_first();  // each page is read once per layer

  pdl_trigger();
  if (lane == 0) {
    for (int s = 0; s < NST; ++s) ptx::mbar_init(&bar[s], 1);
    ptx::fence_barrier_init();
  }
  __syncwarp();
  pdl_wait();  // work counter, Q rows, block table, KV pages: all produced by earlier kernels

  // ---- issue side of the page stream (warp-uniform state; lane 0 issues).  Global reads on
  // this path are issued a step before their value is needed: the next work item is claimed
  // (atomicAdd) two pages before the current one ends -- not earlier, so a warp never sits on a
  // claimed item while others idle (longest-first balance) -- and its header is read one page
  // later; the block table is read 32 entries at a time (lane l holds page base + l).
  int iw = 0, ip = 0, inp = 0;  // work index, page within the item, pages of the item
  int i_seq = 0, i_kvh = 0, i_nb0 = 0;
  int nst = 0;                  // next item: 0 none claimed, 1 claimed (nv in flight), 2 header read
  int nv = 0, n_iw = 0, n_L = 0;
  DecodeItem n_it{0, 0, -1, 1};
  int btw = 0;
  const int32_t* bt_row = a.block_table;
  auto claim = [&]() {
    if (lane == 0) nv = atomicAdd(ctr, 1);
    nst = 1;
  };
  auto resolve = [&]() {
    n_iw = __shfl_sync(0xffffffffu, nv, 0);
    if (n_iw < n_work) {
      n_it = items[n_iw / Hkv];
      n_L = a.kv_len[n_it.seq];
    }
    nst = 2;
  };
  auto fetch = [&]() {
    if (nst == 0) claim();
    if (nst == 1) resolve();
    nst = 0;
    iw = n_iw;
    ip = 0;
    if (iw < n_work) {
      i_kvh = iw % Hkv;
      i_seq = n_it.seq;
      const int k0 = n_it.split * a.split_len, k1 = min(n_L, k0 + a.split_len);
      i_nb0 = k0 / 16;
      inp = (k1 + 15) / 16 - i_nb0;
      bt_row = a.block_table + (size_t)i_seq * a.maxblk + i_nb0;
      btw = lane < inp ? __ldg(bt_row + lane) : 0;
      if (inp <= 2) claim();
    }
  };
  auto issue = [&](int s) {
    if (iw >= n_work) {
      if (lane == 0) meta[s] = make_int4(-1, 0, 0, 0);
      return;
    }
    const int blk = __shfl_sync(0xffffffffu, btw, ip & 31);
    if (lane == 0) {
      const int64_t page = (int64_t)blk * Hkv + i_kvh;  // SMEM-ready page (kvpage.cuh): one copy each
      const bool first = ip == 0;
      fence_proxy_async();  // this slot's earlier generic reads (ldmatrix) before the async writes
      ptx::mbar_arrive_expect_tx(&bar[s], Lay::SLOT);
      uint8_t* dst = ring + s * Lay::SLOT;
      ptx::bulk_load_hint(dst, a.kc + page * 16 * D, Lay::PAGE, &bar[s], pol);
      ptx::bulk_load_hint(dst + Lay::PAGE, a.vc + page * 16 * D, Lay::PAGE, &bar[s], pol);
      meta[s] = make_int4(iw, ip, (ip == inp - 1 ? 1 : 0) | (first ? 2 : 0), 0);
    }
    if (++ip == inp) {
      fetch();
    } else {
      if ((ip & 31) == 0) btw = ip + lane < inp ? __ldg(bt_row + ip + lane) : 0;
      if (nst == 1)
        resolve();
      else if (nst == 0 && ip == inp - 2)
        claim();
    }
  };

  fetch();
#pragma unroll 1
  for (int s = 0; s < NST - 1; ++s) issue(s);

  // ---- consume side
  uint32_t qa[D / 16][4];
  float o[D / 8][4];
  float mrow[2] = {-INFINITY, -INFINITY}, lrow[2] = {0.f, 0.f};
  int c_seq = 0, c_kvh = 0, c_k1 = 0, c_nb0 = 0, c_part = -1, c_split = 0, c_nsplit = 1;
#pragma unroll 1
  for (int i = 0;; ++i) {
    const int s = i % NST;
    issue((i + NST - 1) % NST);  // the slot consumed at iteration i - 1
    __syncwarp();
    const int4 mt = meta[s];
    if (mt.x < 0) break;
    if (mt.z & 2) {  // first page of a work item: its G query rows straight from global (L2)
      const DecodeItem it = items[mt.x / Hkv];
      c_kvh = mt.x % Hkv;
      c_seq = it.seq;
      const int L = a.kv_len[it.seq];
      const int k0 = it.split * a.split_len;
      c_k1 = min(L, k0 + a.split_len);
      c_nb0 = k0 / 16;
      c_part = it.part;
      c_split = it.split;
      c_nsplit = it.nsplit;
      const __nv_bfloat16* qrow = a.q + (size_t)a.cu_q[c_seq] * a.q_stride + (size_t)(c_kvh * G + (g < G ? g : 0)) * D;
#pragma unroll
      for (int ks = 0; ks < D / 16; ++ks) {
        const int c0 = ks * 16 + 2 * tq;
        qa[ks][0] = g < G ? __ldg(reinterpret_cast<const unsigned int*>(qrow + c0)) : 0u;
        qa[ks][1] = 0u;  // rows 8..15 (G <= 8)
        qa[ks][2] = g < G ? __ldg(reinterpret_cast<const unsigned int*>(qrow + c0 + 8)) : 0u;
        qa[ks][3] = 0u;
      }
#pragma unroll
      for (int n = 0; n < D / 8; ++n) o[n][0] = o[n][1] = o[n][2] = o[n][3] = 0.f;
      mrow[0] = mrow[1] = -INFINITY;
      lrow[0] = lrow[1] = 0.f;
    }
    ptx::mbar_wait(&bar[s], (uint32_t)((i / NST) & 1));
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
      if (c_part >= 0) {
        // split row: the last split to arrive merges all partials of (row, kv head) in place
        // (threadfence + arrival counter, as split-K fix-up) -- no separate merge launch
        const int first = c_part - c_split;
        __threadfence();
        __syncwarp();
        int prev = 0;
        if (lane == 0) prev = atomicAdd(a.part_ctr + (size_t)first * Hkv + c_kvh, 1);
        prev = __shfl_sync(0xffffffffu, prev, 0);
        if (prev == c_nsplit - 1) {
          __threadfence();
          if (lane == 0) a.part_ctr[(size_t)first * Hkv + c_kvh] = 0;  // ready for the next launch
          // Merge of the row's nsplit partials, latency-tolerant: (1) lane l reduces the (max, sum)
          // statistics of splits l, l + 32, ... (independent loads), combined across the warp in a
          // fixed order; (2) lane l owns output elements l + 32k and accumulates the splits' O
          // rows four splits per step, so four independent loads per element are in flight
          // (a dependent L2 round trip per split made long rows' merges dominate small batches).
          constexpr int PER = G * D / 32;
          const int t = a.cu_q[c_seq];
          const size_t pbase = (size_t)first * Hkv + c_kvh;  // split sp's (G, D) block: (pbase + sp*Hkv)*G
          float M[G], Ls[G];
#pragma unroll
          for (int h = 0; h < G; ++h) M[h] = -INFINITY;
          for (int sp = lane; sp < c_nsplit; sp += 32) {
#pragma unroll
            for (int h = 0; h < G; ++h) M[h] = fmaxf(M[h], __ldcg(a.part_ml + ((pbase + (size_t)sp * Hkv) * G + h) * 2));
          }
#pragma unroll
          for (int h = 0; h < G; ++h) {
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) M[h] = fmaxf(M[h], __shfl_xor_sync(0xffffffffu, M[h], o));
            Ls[h] = 0.f;
          }
          for (int sp = lane; sp < c_nsplit; sp += 32) {
#pragma unroll
            for (int h = 0; h < G; ++h) {
              const float2 ml = __ldcg(reinterpret_cast<const float2*>(a.part_ml + ((pbase + (size_t)sp * Hkv) * G + h) * 2));
              Ls[h] += ml.y * exp2f(ml.x - M[h]);
            }
          }
#pragma unroll
          for (int h = 0; h < G; ++h)
#pragma unroll
            for (int o = 16; o > 0; o >>= 1) Ls[h] += __shfl_xor_sync(0xffffffffu, Ls[h], o);
          float acc[PER];
#pragma unroll
          for (int k = 0; k < PER; ++k) acc[k] = 0.f;
          constexpr int QU = PER >= 32 ? 2 : 4;  // splits per step (register budget at G = 8)
          for (int sp0 = 0; sp0 < c_nsplit; sp0 += QU) {
            float v[QU][PER], f[QU][G];
#pragma unroll
            for (int q = 0; q < QU; ++q) {
              const int sp = min(sp0 + q, c_nsplit - 1);
              const size_t b0 = (pbase + (size_t)sp * Hkv) * G;
#pragma unroll
              for (int h = 0; h < G; ++h) {
                const float mm = __ldcg(a.part_ml + (b0 + h) * 2);
                f[q][h] = sp0 + q < c_nsplit ? exp2f(mm - M[h]) : 0.f;
              }
#pragma unroll
              for (int k = 0; k < PER; ++k) v[q][k] = __ldcg(a.part_o + b0 * D + lane + 32 * k);
            }
#pragma unroll
            for (int q = 0; q < QU; ++q)
#pragma unroll
              for (int k = 0; k < PER; ++k) acc[k] += v[q][k] * f[q][(lane + 32 * k) / D];
          }
#pragma unroll
          for (int k = 0; k < PER; ++k) {
            const int idx = lane + 32 * k;
            a.out[(size_t)t * a.Hq * D + (size_t)c_kvh * G * D + idx] = __float2bfloat16_rn(acc[k] / Ls[idx / D]);
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

template <int D, int G, int NST, int WARPS>
int launch_t(const AttnArgs& a, const DecodeItem* items,
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
    launch_pdl(decode_attn_tma_kernel<D, G, NST, WARPS>, dim3(grid), dim3(WARPS * 32), Lay::BYTES, s, 1, a, items,
               n_work, ctr);
  }
  (void)merges;
  (void)n_merges;  // split rows are merged inside the kernel by their last split
  return GLLM_OK;
}

template <int D, int G>
int launch_g(const AttnArgs& a, const DecodeItem* items, int n_items,
             const MergeItem* merges, int n_merges, int* ctr, int num_sms, cudaStream_t s) {
  // 3-slot page ring x 4 warps, 2 CTAs per SM (profiles/r02/decode_split_ab.txt: 6 slots x 4 warps at
  // 1 CTA per SM is 15-25% slower -- the per-page mma.sync work of fewer warps limits it)
  return launch_t<D, G, 3, 4>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
}

template <int D>
int launch_d(const AttnArgs& a, const DecodeItem* items, int n_items,
             const MergeItem* merges, int n_merges, int* ctr, int num_sms, cudaStream_t s) {
  switch (a.Hq / a.Hkv) {
    case 1: return launch_g<D, 1>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 2: return launch_g<D, 2>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 4: return launch_g<D, 4>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 5: return launch_g<D, 5>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
    case 8: return launch_g<D, 8>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
  }
  return set_error(GLLM_EINVAL, "decode attention (tma): unsupported GQA group %d", a.Hq / a.Hkv);
}

}  // namespace

int decode_workers(int num_sms) {  // warp workers of the persistent decode kernel (host split policy)
  return 8 * num_sms;  // 2 CTAs of 4 warps per SM
}

bool decode_tma_supported(int D, int G) { return (D == 64 || D == 128) && (G == 1 || G == 2 || G == 4 || G == 5 || G == 8); }

int launch_decode_attention_tma(const AttnArgs& a, const DecodeItem* items, int n_items, const MergeItem* merges, int n_merges, int* ctr,
                                int num_sms, cudaStream_t s) {
  int rc;
  if (a.bs != 16) return set_error(GLLM_EINVAL, "decode attention (tma): block size %d != 16", a.bs);
  if (a.D == 128)
    rc = launch_d<128>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
  else if (a.D == 64)
    rc = launch_d<64>(a, items, n_items, merges, n_merges, ctr, num_sms, s);
  else
    return set_error(GLLM_EINVAL, "decode attention (tma): head_dim %d unsupported", a.D);
  if (rc) return rc;
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK : set_error(GLLM_ECUDA, "decode attention launch: %s", cudaGetErrorString(e));
}

}  // namespace gllm
