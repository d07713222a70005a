// Prefill (chunked, causal, paged) attention on 5th-gen tensor cores -- part of a7.
// (The header below describes v1, the default; v2 (GLLM_PREFILL_V2=1) pipelines it, see prefill_attn_tc_kernel.)
//
// CTA = 128 flattened (token, group-head) query rows of one chunk x one kv head (the G query
// heads sharing a kv head reuse every K/V tile); 4 warps, thread t owns row t = TMEM lane t.
// Per 64-key tile j of the paged cache (4 pages, cp.async double-buffered, SW128 layout):
//   S_j = Q K_j^T     tcgen05.mma M=128 N=64 K=D   (Q, K K-major in SMEM)   -> TMEM cols [0, 64)
//   softmax           tcgen05.ld of the row, causal mask, online max / exp2 / sum in registers;
//                     O is rescaled in TMEM (ld/st) only when the running max grows by > 2^8
//   O += P_j V_j      tcgen05.mma M=128 N=D K=64  (P bf16 written to TMEM with tcgen05.st and
//                     read from there as the A operand; V MN-major in SMEM) -> TMEM
// SMEM = Q + 2 x (K, V) = 96 KB at D = 128, TMEM = 256 columns: two CTAs per SM, whose
// softmax and MMA phases interleave.
// one thread issues the MMAs and commits them to mbarriers; the next tile's K/V loads overlap
// the current tile.  Final: O / l -> bf16 rows of the attention output.
#include <cuda_bf16.h>

#include <cstdlib>

#include "attention.cuh"
#include "common.h"
#include "ptx.cuh"

namespace gllm {

namespace {

constexpr float LOG2E_T = 1.4426950408889634f;
constexpr int TC_ROWS = 128;
constexpr int TC_KT = 64;  // keys per tile
constexpr float RESCALE_LOG2 = 8.0f;

template <int D>
struct TcSmem {
  static constexpr int ATOMS = D / 64;              // 64-element (128-byte) swizzle atoms along D
  static constexpr int Q_ATOM = TC_ROWS * 128;      // bytes of one Q atom column
  static constexpr int KV_ATOM = TC_KT * 128;       // bytes of one K (or V) atom column
  static constexpr int Q = 0;
  static constexpr int K0 = Q + ATOMS * Q_ATOM;
  static constexpr int V0 = K0 + ATOMS * KV_ATOM;
  static constexpr int K1 = V0 + ATOMS * KV_ATOM;
  static constexpr int V1 = K1 + ATOMS * KV_ATOM;
  static constexpr int BAR = V1 + ATOMS * KV_ATOM;  // (P lives in TMEM)
  static constexpr int BYTES = BAR + 64 + 1024;    // + alignment slack
};

// byte offset of (row, 16-byte chunk along the row) in an atom-tiled SW128 tile with `rows` rows
__device__ __forceinline__ uint32_t sw128(int rows, int row, int chunk) {
  return (chunk >> 3) * (rows * 128) + row * 128 + (((chunk & 7) ^ (row & 7)) << 4);
}

// K-major operand descriptor (SW128, 8-row groups 1024 B apart)
__device__ __forceinline__ uint64_t desc_k(uint32_t addr) { return ptx::umma_desc_sw128(addr); }
// MN-major operand descriptor (SW128): LBO = stride between 64-element MN atoms, SBO = stride
// between 8-row K groups (1024 B)
__device__ __forceinline__ uint64_t desc_mn(uint32_t addr, uint32_t lbo_bytes) {
  uint64_t d = 0;
  d |= (uint64_t)((addr & 0x3FFFFu) >> 4);
  d |= (uint64_t)((lbo_bytes >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
__host__ __device__ constexpr uint32_t idesc_bf16(int M, int N, bool b_mn_major) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((b_mn_major ? 1u : 0u) << 16) | ((uint32_t)(N >> 3) << 17) |
         ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tmem_st_32x32b_x32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
      "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
      "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}
__device__ __forceinline__ float fast_exp2(float x) {  // ex2.approx: 2^-inf = +0
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
__device__ __forceinline__ void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
// D[tmem] (+)= A[tmem] . B[smem]: the A operand (here P, bf16 pairs per 32-bit column, row = lane)
// is read from TMEM
__device__ __forceinline__ void umma_bf16_ta(uint32_t tmem_d, uint32_t tmem_a, uint64_t bdesc, uint32_t idesc,
                                             uint32_t accumulate) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "r"(tmem_a), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}

// v1 (default): S_j, softmax_j and PV_j in series per CTA; two CTAs per SM overlap each other.
template <int D>
__global__ void __launch_bounds__(128, 2)
    prefill_attn_tc_v1_kernel(const AttnArgs a, const PrefillItem* __restrict__ items) {
  using L = TcSmem<D>;
  constexpr int NCH = D / 8;  // 16-byte chunks per K/V/Q row
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = ptx::smem_u32(smem);
  uint64_t* bar_s = reinterpret_cast<uint64_t*>(smem + L::BAR);
  uint64_t* bar_pv = bar_s + 1;
  uint32_t* tmem_ptr = reinterpret_cast<uint32_t*>(bar_s + 2);

  const PrefillItem it = items[blockIdx.x];
  const int kvh = blockIdx.y;
  const int G = a.Hq / a.Hkv;
  const int tid = threadIdx.x, warp = tid >> 5;
  const int t0 = a.cu_q[it.seq];
  const int c = a.cu_q[it.seq + 1] - t0;
  const int s0 = a.kv_len[it.seq] - c;
  const int nrows = c * G;
  const int max_pos = s0 + min(it.row0 + TC_ROWS - 1, nrows - 1) / G;
  const int n_kt = (max_pos + TC_KT) / TC_KT;
  const int nblk_seq = (a.kv_len[it.seq] + 15) / 16;
  const int32_t* bt = a.block_table + (size_t)it.seq * a.maxblk;
  const float sl2 = LOG2E_T * rsqrtf((float)D);

  if (tid == 0) {
    ptx::mbar_init(bar_s, 1);
    ptx::mbar_init(bar_pv, 1);
    ptx::fence_barrier_init();
  }
  if (warp == 0) ptx::tmem_alloc(tmem_ptr, 256);  // S: [0, 64), P (bf16x2): [64, 96), O: [128, 128 + D)
  if (warp == 0) ptx::tmem_relinquish();

  // ---- Q rows -> SMEM (rows beyond the chunk repeat the last row; never stored)
  for (int idx = tid; idx < TC_ROWS * NCH; idx += 128) {
    const int r = idx / NCH, ch = idx % NCH;
    const int rr = min(it.row0 + r, nrows - 1);
    const int tok = rr / G, h = kvh * G + rr % G;
    ptx::cp_async16(sbase + L::Q + sw128(TC_ROWS, r, ch),
                    a.q + (size_t)(t0 + tok) * a.q_stride + (size_t)h * D + ch * 8, true);
  }
  auto load_kv = [&](int kt, int buf) {
    const uint32_t kb = sbase + (buf ? L::K1 : L::K0), vb = sbase + (buf ? L::V1 : L::V0);
    for (int idx = tid; idx < TC_KT * NCH; idx += 128) {
      const int r = idx / NCH, ch = idx % NCH;
      const int key = kt * TC_KT + r;
      const int blk = key >> 4;
      const bool ok = blk < nblk_seq;
      const size_t page = ok ? (size_t)bt[blk] : 0;
      const size_t off = ((page * a.Hkv + kvh) * 16 + (key & 15)) * D + ch * 8;
      ptx::cp_async16(kb + sw128(TC_KT, r, ch), a.kc + off, ok);
      ptx::cp_async16(vb + sw128(TC_KT, r, ch), a.vc + off, ok);
    }
  };
  load_kv(0, 0);
  ptx::cp_async_commit();

  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_ptr;
  const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
  const uint32_t t_s = tmem + lane_off, t_p = tmem + lane_off + 64, t_o = tmem + lane_off + 128;

  const int rr = it.row0 + tid;
  const int rrc = min(rr, nrows - 1);
  const int pos = s0 + rrc / G;  // this row's causal limit (keys 0..pos)
  float m_ref = -INFINITY, l = 0.f;
  constexpr uint32_t idesc_s = idesc_bf16(TC_ROWS, TC_KT, false);
  constexpr uint32_t idesc_o = idesc_bf16(TC_ROWS, D, true);

  for (int j = 0; j < n_kt; ++j) {
    const int buf = j & 1;
    ptx::cp_async_wait<0>();
    fence_proxy_async_smem();  // cp.async (generic proxy) writes -> visible to the tensor core
    __syncthreads();
    if (tid == 0) {
      ptx::tc_fence_after();
      const uint32_t kb = sbase + (buf ? L::K1 : L::K0);
#pragma unroll
      for (int ks = 0; ks < D / 16; ++ks)
        ptx::umma_bf16(t_s - lane_off, desc_k(sbase + L::Q + (ks / 4) * L::Q_ATOM + (ks % 4) * 32),
                       desc_k(kb + (ks / 4) * L::KV_ATOM + (ks % 4) * 32), idesc_s, ks > 0);
      ptx::umma_commit(bar_s);
    }
    if (j > 0) ptx::mbar_wait(bar_pv, (j - 1) & 1);  // PV_{j-1} done: P, V_{j-1} and O are free
    if (j + 1 < n_kt) load_kv(j + 1, buf ^ 1);
    ptx::cp_async_commit();
    ptx::mbar_wait(bar_s, j & 1);
    ptx::tc_fence_after();
    uint32_t sr[2][32];
    ptx::tmem_ld_32x32b_x32(t_s, sr[0]);
    ptx::tmem_ld_32x32b_x32(t_s + 32, sr[1]);
    ptx::tmem_ld_wait();
    // raw scores; the causal mask is applied only on tiles that cross this row's diagonal, and
    // the 1/sqrt(D)*log2(e) scale is folded into the max and into the exp2 argument (one FFMA)
    float s[64];
#pragma unroll
    for (int i = 0; i < 64; ++i) s[i] = __uint_as_float(sr[i >> 5][i & 31]);
    if (j * TC_KT + TC_KT - 1 > pos) {
#pragma unroll
      for (int i = 0; i < 64; ++i)
        if (j * TC_KT + i > pos) s[i] = -INFINITY;
    }
    float mx4[4] = {s[0], s[1], s[2], s[3]};
#pragma unroll
    for (int i = 4; i < 64; ++i) mx4[i & 3] = fmaxf(mx4[i & 3], s[i]);
    const float mx = fmaxf(fmaxf(mx4[0], mx4[1]), fmaxf(mx4[2], mx4[3])) * sl2;
    // lazy rescale: exact because l and O share the reference max.  tcgen05.ld/st are warp-
    // collective (.sync.aligned), so the O pass runs for the whole warp when any lane needs it
    // (lanes that do not rescale multiply by 1).
    const bool mine = mx > m_ref + RESCALE_LOG2;
    const float corr = mine ? exp2f(m_ref - mx) : 1.f;
    if (mine) {
      l *= corr;
      m_ref = mx;
    }
    if (j > 0 && __any_sync(0xffffffffu, mine)) {
#pragma unroll
      for (int cb = 0; cb < D / 32; ++cb) {
        uint32_t orr[32];
        ptx::tmem_ld_32x32b_x32(t_o + cb * 32, orr);
        ptx::tmem_ld_wait();
#pragma unroll
        for (int i = 0; i < 32; ++i) orr[i] = __float_as_uint(__uint_as_float(orr[i]) * corr);
        tmem_st_32x32b_x32(t_o + cb * 32, orr);
      }
      tmem_st_wait();
    }
    // P row (bf16 pairs) -> TMEM cols [64, 96): the A operand of the PV MMA
    {
      uint32_t pw[32];
      float la = 0.f, lb = 0.f;
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const float p0 = fast_exp2(fmaf(s[2 * i], sl2, -m_ref)), p1 = fast_exp2(fmaf(s[2 * i + 1], sl2, -m_ref));
        la += p0;
        lb += p1;
        pw[i] = ptx::pack_bf16(p0, p1);
      }
      l += la + lb;
      tmem_st_32x32b_x32(t_p, pw);
      tmem_st_wait();
    }
    ptx::tc_fence_before();
    __syncthreads();
    if (tid == 0) {
      ptx::tc_fence_after();
      const uint32_t vb = sbase + (buf ? L::V1 : L::V0);
#pragma unroll
      for (int kk = 0; kk < TC_KT / 16; ++kk)  // K = 16 keys = 8 TMEM columns of packed P per step
        umma_bf16_ta(t_o - lane_off, t_p - lane_off + kk * 8, desc_mn(vb + kk * 2048, L::KV_ATOM), idesc_o,
                     (j > 0 || kk > 0) ? 1u : 0u);
      ptx::umma_commit(bar_pv);
    }
  }
  ptx::mbar_wait(bar_pv, (n_kt - 1) & 1);
  ptx::tc_fence_after();
  const bool valid = rr < nrows;
  const float inv = 1.f / l;
  __nv_bfloat16* dst = a.out + (size_t)(t0 + rrc / G) * a.Hq * D + (size_t)(kvh * G + rrc % G) * D;
#pragma unroll
  for (int cb = 0; cb < D / 32; ++cb) {
    uint32_t orr[32];
    ptx::tmem_ld_32x32b_x32(t_o + cb * 32, orr);
    ptx::tmem_ld_wait();
    if (valid) {
      uint4* d4 = reinterpret_cast<uint4*>(dst + cb * 32);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint4 w;
        w.x = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 0]) * inv, __uint_as_float(orr[q * 8 + 1]) * inv);
        w.y = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 2]) * inv, __uint_as_float(orr[q * 8 + 3]) * inv);
        w.z = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 4]) * inv, __uint_as_float(orr[q * 8 + 5]) * inv);
        w.w = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 6]) * inv, __uint_as_float(orr[q * 8 + 7]) * inv);
        d4[q] = w;
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 256);
  }
}

// v2: software-pipelined.  TMEM: two S buffers [0, 64) and [64, 128) (P_j overwrites S_j in place
// once the row is in registers), O at [128, 128 + D).  Per key tile j the issuing thread queues
// S_{j+1} = Q K_{j+1}^T BEFORE the softmax of S_j starts, so the tensor core computes the next
// scores while the 128 threads run the softmax; tcgen05.mma executes in issue order, which makes
// the overwrite of P_{j-1} by S_{j+1} safe behind PV_{j-1}.  K_{j+2} is fetched as soon as S_j
// is done and V_{j+1} once PV_{j-1} is done, each as its own cp.async group (two K and two V
// buffers; SMEM as v1).
template <int D>
__global__ void __launch_bounds__(128, 2)
    prefill_attn_tc_kernel(const AttnArgs a, const PrefillItem* __restrict__ items) {
  using L = TcSmem<D>;
  constexpr int NCH = D / 8;  // 16-byte chunks per K/V/Q row
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = ptx::smem_u32(smem);
  uint64_t* bar_s = reinterpret_cast<uint64_t*>(smem + L::BAR);  // [2]: S buffer b complete
  uint64_t* bar_pv = bar_s + 2;
  uint32_t* tmem_ptr = reinterpret_cast<uint32_t*>(bar_s + 3);

  const PrefillItem it = items[blockIdx.x];
  const int kvh = blockIdx.y;
  const int G = a.Hq / a.Hkv;
  const int tid = threadIdx.x, warp = tid >> 5;
  const int t0 = a.cu_q[it.seq];
  const int c = a.cu_q[it.seq + 1] - t0;
  const int s0 = a.kv_len[it.seq] - c;
  const int nrows = c * G;
  const int max_pos = s0 + min(it.row0 + TC_ROWS - 1, nrows - 1) / G;
  const int n_kt = (max_pos + TC_KT) / TC_KT;
  const int nblk_seq = (a.kv_len[it.seq] + 15) / 16;
  const int32_t* bt = a.block_table + (size_t)it.seq * a.maxblk;
  const float sl2 = LOG2E_T * rsqrtf((float)D);

  if (tid == 0) {
    ptx::mbar_init(&bar_s[0], 1);
    ptx::mbar_init(&bar_s[1], 1);
    ptx::mbar_init(bar_pv, 1);
    ptx::fence_barrier_init();
  }
  if (warp == 0) ptx::tmem_alloc(tmem_ptr, 256);
  if (warp == 0) ptx::tmem_relinquish();

  for (int idx = tid; idx < TC_ROWS * NCH; idx += 128) {
    const int r = idx / NCH, ch = idx % NCH;
    const int rr = min(it.row0 + r, nrows - 1);
    const int tok = rr / G, h = kvh * G + rr % G;
    ptx::cp_async16(sbase + L::Q + sw128(TC_ROWS, r, ch),
                    a.q + (size_t)(t0 + tok) * a.q_stride + (size_t)h * D + ch * 8, true);
  }
  // one 64-key tile of K (or V) of the paged cache into buffer `buf`
  auto load_tile = [&](const __nv_bfloat16* cache, int kt, uint32_t dst) {
    for (int idx = tid; idx < TC_KT * NCH; idx += 128) {
      const int r = idx / NCH, ch = idx % NCH;
      const int key = kt * TC_KT + r;
      const int blk = key >> 4;
      const bool ok = blk < nblk_seq;
      const size_t page = ok ? (size_t)bt[blk] : 0;
      ptx::cp_async16(dst + sw128(TC_KT, r, ch), cache + ((page * a.Hkv + kvh) * 16 + (key & 15)) * D + ch * 8, ok);
    }
  };
  auto kbuf = [&](int b) { return sbase + (b ? L::K1 : L::K0); };
  auto vbuf = [&](int b) { return sbase + (b ? L::V1 : L::V0); };
  // cp.async groups, in commit order: {Q, K_0, K_1}, {V_0}, then per tile j: {K_{j+2}}, {V_{j+1}}
  load_tile(a.kc, 0, kbuf(0));
  if (n_kt > 1) load_tile(a.kc, 1, kbuf(1));
  ptx::cp_async_commit();
  load_tile(a.vc, 0, vbuf(0));
  ptx::cp_async_commit();

  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_ptr;
  const uint32_t lane_off = (uint32_t)(warp * 32) << 16;
  const uint32_t t_o = tmem + lane_off + 128;
  constexpr uint32_t idesc_s = idesc_bf16(TC_ROWS, TC_KT, false);
  constexpr uint32_t idesc_o = idesc_bf16(TC_ROWS, D, true);
  auto issue_s = [&](int j) {  // thread 0: S_j -> S buffer j & 1
    ptx::tc_fence_after();
    const uint32_t kb = kbuf(j & 1);
#pragma unroll
    for (int ks = 0; ks < D / 16; ++ks)
      ptx::umma_bf16(tmem + (j & 1) * TC_KT, desc_k(sbase + L::Q + (ks / 4) * L::Q_ATOM + (ks % 4) * 32),
                     desc_k(kb + (ks / 4) * L::KV_ATOM + (ks % 4) * 32), idesc_s, ks > 0);
    ptx::umma_commit(&bar_s[j & 1]);
  };
  ptx::cp_async_wait<1>();  // Q, K_0, K_1
  fence_proxy_async_smem();
  __syncthreads();
  if (tid == 0) issue_s(0);

  const int rr = it.row0 + tid;
  const int rrc = min(rr, nrows - 1);
  const int pos = s0 + rrc / G;  // this row's causal limit (keys 0..pos)
  float m_ref = -INFINITY, l = 0.f;

  for (int j = 0; j < n_kt; ++j) {
    const int b = j & 1;
    // A: queue S_{j+1} behind PV_{j-1} (K_{j+1} is the older of the two newest groups)
    if (j + 1 < n_kt) {
      ptx::cp_async_wait<1>();
      fence_proxy_async_smem();
      __syncthreads();
      if (tid == 0) issue_s(j + 1);
    }
    // B: S_j -> registers; its K buffer is free for K_{j+2}
    ptx::mbar_wait(&bar_s[b], (j >> 1) & 1);
    ptx::tc_fence_after();
    uint32_t sr[2][32];
    const uint32_t t_s = tmem + lane_off + b * TC_KT;
    ptx::tmem_ld_32x32b_x32(t_s, sr[0]);
    ptx::tmem_ld_32x32b_x32(t_s + 32, sr[1]);
    ptx::tmem_ld_wait();
    if (j + 2 < n_kt) load_tile(a.kc, j + 2, kbuf(b));
    ptx::cp_async_commit();
    // C: online softmax (lazy rescale, see v1), P_j over S_j
    float s[64];
    float mx = -INFINITY;
#pragma unroll
    for (int i = 0; i < 64; ++i) {
      const int key = j * TC_KT + i;
      s[i] = key <= pos ? __uint_as_float(sr[i >> 5][i & 31]) * sl2 : -INFINITY;
      mx = fmaxf(mx, s[i]);
    }
    const bool mine = mx > m_ref + RESCALE_LOG2;
    const float corr = mine ? exp2f(m_ref - mx) : 1.f;
    if (mine) {
      l *= corr;
      m_ref = mx;
    }
    if (j > 0 && __any_sync(0xffffffffu, mine)) {
      ptx::mbar_wait(bar_pv, (j - 1) & 1);  // O final for tiles < j
      ptx::tc_fence_after();
#pragma unroll
      for (int cb = 0; cb < D / 32; ++cb) {
        uint32_t orr[32];
        ptx::tmem_ld_32x32b_x32(t_o + cb * 32, orr);
        ptx::tmem_ld_wait();
#pragma unroll
        for (int i = 0; i < 32; ++i) orr[i] = __float_as_uint(__uint_as_float(orr[i]) * corr);
        tmem_st_32x32b_x32(t_o + cb * 32, orr);
      }
    }
    {
      uint32_t pw[32];
#pragma unroll
      for (int i = 0; i < 32; ++i) {
        const float p0 = exp2f(s[2 * i] - m_ref), p1 = exp2f(s[2 * i + 1] - m_ref);
        l += p0 + p1;
        pw[i] = ptx::pack_bf16(p0, p1);
      }
      tmem_st_32x32b_x32(t_s, pw);
      tmem_st_wait();
    }
    // D: PV_{j-1} done -> its V buffer takes V_{j+1}
    if (j > 0) ptx::mbar_wait(bar_pv, (j - 1) & 1);
    if (j + 1 < n_kt) load_tile(a.vc, j + 1, vbuf(b ^ 1));
    ptx::cp_async_commit();
    // E: O += P_j V_j (V_j is the oldest of the three newest groups)
    ptx::cp_async_wait<2>();
    fence_proxy_async_smem();
    ptx::tc_fence_before();
    __syncthreads();
    if (tid == 0) {
      ptx::tc_fence_after();
      const uint32_t vb = vbuf(b);
#pragma unroll
      for (int kk = 0; kk < TC_KT / 16; ++kk)
        umma_bf16_ta(tmem + 128, tmem + b * TC_KT + kk * 8, desc_mn(vb + kk * 2048, L::KV_ATOM), idesc_o,
                     (j > 0 || kk > 0) ? 1u : 0u);
      ptx::umma_commit(bar_pv);
    }
  }
  ptx::mbar_wait(bar_pv, (n_kt - 1) & 1);
  ptx::tc_fence_after();
  const bool valid = rr < nrows;
  const float inv = 1.f / l;
  __nv_bfloat16* dst = a.out + (size_t)(t0 + rrc / G) * a.Hq * D + (size_t)(kvh * G + rrc % G) * D;
#pragma unroll
  for (int cb = 0; cb < D / 32; ++cb) {
    uint32_t orr[32];
    ptx::tmem_ld_32x32b_x32(t_o + cb * 32, orr);
    ptx::tmem_ld_wait();
    if (valid) {
      uint4* d4 = reinterpret_cast<uint4*>(dst + cb * 32);
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        uint4 w;
        w.x = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 0]) * inv, __uint_as_float(orr[q * 8 + 1]) * inv);
        w.y = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 2]) * inv, __uint_as_float(orr[q * 8 + 3]) * inv);
        w.z = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 4]) * inv, __uint_as_float(orr[q * 8 + 5]) * inv);
        w.w = ptx::pack_bf16(__uint_as_float(orr[q * 8 + 6]) * inv, __uint_as_float(orr[q * 8 + 7]) * inv);
        d4[q] = w;
      }
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 256);
  }
}

// v1 is the default: measured on B200 (tools/ab.sh, profiles/r01/ab_prefill.txt) the pipelined v2
// is 10-20% slower -- two co-resident CTAs per SM already interleave softmax and MMA phases.
const bool g_prefill_v1 = [] {
  const char* e = std::getenv("GLLM_PREFILL_V2");
  return !(e && e[0] == '1');
}();

// Dynamic SMEM actually reserved per prefill CTA.  Padding it past half an SM (GLLM_PREFILL_PAD_KB)
// caps prefill at one CTA per SM, leaving the other slot to a persistent decode CTA that runs
// concurrently (A/B knob; see stage.cu attention step).
int prefill_smem_bytes(int need) {
  static const int pad = [] {
    const char* e = std::getenv("GLLM_PREFILL_PAD_KB");
    return e ? std::atoi(e) * 1024 : 0;
  }();
  return need > pad ? need : pad;
}

template <int D>
int launch_tc(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s) {
  const int bytes = prefill_smem_bytes(TcSmem<D>::BYTES);
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(prefill_attn_tc_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    cudaFuncSetAttribute(prefill_attn_tc_v1_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    set = true;
  }
  if (g_prefill_v1)
    prefill_attn_tc_v1_kernel<D><<<dim3(n_items, a.Hkv), 128, bytes, s>>>(a, items);
  else
    prefill_attn_tc_kernel<D><<<dim3(n_items, a.Hkv), 128, bytes, s>>>(a, items);
  return GLLM_OK;
}

}  // namespace

int launch_prefill_attention_tc(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s) {
  if (n_items <= 0) return GLLM_OK;
  if (a.D == 128)
    launch_tc<128>(a, items, n_items, s);
  else if (a.D == 64)
    launch_tc<64>(a, items, n_items, s);
  else
    return set_error(GLLM_EINVAL, "prefill attention (tcgen05): head_dim %d unsupported", a.D);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK : set_error(GLLM_ECUDA, "prefill attention (tcgen05) launch: %s",
                                                cudaGetErrorString(e));
}

}  // namespace gllm
