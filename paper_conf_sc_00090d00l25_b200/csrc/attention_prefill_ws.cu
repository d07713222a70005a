// Prefill (chunked, causal, paged) attention, warp-specialised on tcgen05 -- part of a7.
//
// PAPER.md L77 (prefill is compute-bound), L212 (attention over the paged KV cache), L354 (cost
// quadratic in context).  Computes, for every row of a prefill chunk at offset s0,
//   o = softmax(q K[0..s0+j]^T / sqrt(D)) V[0..s0+j]      (GQA: query head h reads kv head h / G)
//
// CTA = two Q tiles (A, B) of 128 flattened (token, group-head) rows of one chunk x one kv head;
// both tiles share every K/V tile, and their softmax phases alternate with the other tile's MMAs
// (ping-pong), so the tensor core and the SFU/FMA pipes run concurrently.  12 warps:
//   warps 8, 10 K / V producers: 128-key K and V tiles = 8 pages (16 x 64 SW128 boxes of the
//               [kv_blocks*Hkv*16, D] page map) per tile, NS-stage rings with separate K and V
//               release (K slots free after the S MMAs, V slots after the PV MMAs), block table
//               read a tile ahead (warp 11 owns the TMEM allocation, 512 columns)
//   warp 9      MMA issuer (one thread):  S_X = Q_X K_j^T  (M=128 N=128 K=D, both K-major)
//                                          O_X += P_X V_j    (M=128 N=D K=128, P from TMEM, V MN-major)
//               issue order per key tile j: PV_A(j), S_A(j+1), PV_B(j), [release stage], S_B(j+1),
//               so S_A(j+1) computes while tile B's softmax runs and vice versa
//   warps 0-3   softmax of tile A, warps 4-7 tile B: thread = row = TMEM lane; max pass over
//               the 128 scores (tcgen05.ld), lazy O rescale (only when the max grows by > 2^8,
//               exact because l and O share the reference max), exp2 pass writing bf16 P over
//               S in TMEM (tcgen05.st) -- P is the A operand of the PV MMA
// TMEM: S_A [0,128) S_B [128,256) O_A [256,256+D) O_B [384,384+D); P_X = first 64 cols of S_X.
// SMEM: Q 2 x 128 x D, NS x (K + V) 128 x D tiles (D=128: 64 KB + 2 x 64 KB).
#include <cuda_bf16.h>

#include <cstdlib>

#include "attention.cuh"
#include "common.h"
#include "ptx.cuh"
#include "launch.cuh"

namespace gllm {

#ifdef GLLM_VARIANT_TRACE
#define TR_WAIT(acc, expr)              \
  {                                     \
    const long long c0__ = clock64();   \
    expr;                               \
    acc += clock64() - c0__;            \
  }
#else
#define TR_WAIT(acc, expr) expr;
#endif

#ifdef GLLM_VARIANT_TRACE
// measurement build only (build.py --variant=trace): per-CTA timeline of the prefill kernel
__device__ unsigned long long* g_pf_trace = nullptr;
constexpr int PF_TR = 20;  // words per CTA record
__device__ __forceinline__ unsigned long long gtime() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
#endif

namespace {

constexpr float LOG2E_W = 1.4426950408889634f;
constexpr int WS_ROWS = 128;  // rows per Q tile (= TMEM lanes)
constexpr int WS_KT = 128;    // keys per tile
constexpr int WS_NSK = 3;     // K ring stages (the S MMAs' operand: the critical path)
constexpr int WS_NSV = 2;     // V ring stages (V is needed only after the tile's softmax)
constexpr int WS_THREADS = 384;
constexpr float WS_RESCALE_LOG2 = 8.0f;
// warp roles: 0-3 softmax of Q tile A, 4-7 softmax of tile B (TMEM lane quarter = warp % 4), 8 K
// producer, 9 MMA issuer, 10 V producer, 11 TMEM allocator.  The producers and the MMA issuer take
// the highest warp ids: the SMSP arbiter issues the highest eligible warp id first, so a busy
// softmax on the same SMSP does not delay the next MMA group or copy (they used to be warps 0-2).
constexpr int PW_K = 8, PW_MMA = 9, PW_V = 10, PW_ALLOC = 11;

template <int D>
struct WsSmem {
  static constexpr int ATOMS = D / 64;            // 64-element (128-byte) swizzle atoms along D
  static constexpr int Q_ATOM = WS_ROWS * 128;    // one atom column of a Q tile
  static constexpr int KV_ATOM = WS_KT * 128;     // one atom column of a K (or V) tile
  static constexpr int Q_TILE = ATOMS * Q_ATOM;
  static constexpr int KV_TILE = ATOMS * KV_ATOM;
  static constexpr int Q = 0;
  static constexpr int K = Q + 2 * Q_TILE;
  static constexpr int V = K + WS_NSK * KV_TILE;
  static constexpr int BAR = V + WS_NSV * KV_TILE;
  // barriers: q_full, kfull[NSK], kempty[NSK], vfull[NSV], vempty[NSV], sfull[2], pfull[2], ofull[2]; tmem slot
  static constexpr int NBAR = 1 + 2 * WS_NSK + 2 * WS_NSV + 6;
  static constexpr int BYTES = BAR + NBAR * 8 + 16 + 1024;  // + 1024-B alignment slack
};

__device__ __forceinline__ uint32_t sw128(int rows, int row, int chunk) {
  return (chunk >> 3) * (rows * 128) + row * 128 + (((chunk & 7) ^ (row & 7)) << 4);
}
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
__device__ __forceinline__ void tmem_st_x16(uint32_t taddr, const uint32_t (&r)[16]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x16.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16};" ::"r"(
          taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15])
      : "memory");
}
__device__ __forceinline__ void tmem_st_x32(uint32_t taddr, const uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.st.sync.aligned.32x32b.x32.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15,%16,"
      "%17,%18,%19,%20,%21,%22,%23,%24,%25,%26,%27,%28,%29,%30,%31,%32};" ::"r"(taddr),
      "r"(r[0]), "r"(r[1]), "r"(r[2]), "r"(r[3]), "r"(r[4]), "r"(r[5]), "r"(r[6]), "r"(r[7]), "r"(r[8]), "r"(r[9]),
      "r"(r[10]), "r"(r[11]), "r"(r[12]), "r"(r[13]), "r"(r[14]), "r"(r[15]), "r"(r[16]), "r"(r[17]), "r"(r[18]),
      "r"(r[19]), "r"(r[20]), "r"(r[21]), "r"(r[22]), "r"(r[23]), "r"(r[24]), "r"(r[25]), "r"(r[26]), "r"(r[27]),
      "r"(r[28]), "r"(r[29]), "r"(r[30]), "r"(r[31])
      : "memory");
}
__device__ __forceinline__ void tmem_st_wait() { asm volatile("tcgen05.wait::st.sync.aligned;" ::: "memory"); }
__device__ __forceinline__ float ex2(float x) {  // ex2.approx: 2^-inf = +0
  float y;
  asm("ex2.approx.ftz.f32 %0, %1;" : "=f"(y) : "f"(x));
  return y;
}
// packed fp32 pairs (sm_100 FFMA2 / FADD2)
__device__ __forceinline__ uint64_t f2pack(float a, float b) {
  uint64_t r;
  asm("mov.b64 %0, {%1, %2};" : "=l"(r) : "f"(a), "f"(b));
  return r;
}
__device__ __forceinline__ void f2unpack(uint64_t v, float& a, float& b) {
  asm("mov.b64 {%0, %1}, %2;" : "=f"(a), "=f"(b) : "l"(v));
}
__device__ __forceinline__ uint64_t ffma2(uint64_t a, uint64_t b, uint64_t c) {
  uint64_t d;
  asm("fma.rn.f32x2 %0, %1, %2, %3;" : "=l"(d) : "l"(a), "l"(b), "l"(c));
  return d;
}
__device__ __forceinline__ uint64_t fadd2(uint64_t a, uint64_t b) {
  uint64_t d;
  asm("add.rn.f32x2 %0, %1, %2;" : "=l"(d) : "l"(a), "l"(b));
  return d;
}

// three-input max (sm_100 FMNMX3): the row-max pass issues half the ALU-pipe instructions
__device__ __forceinline__ float fmax3(float a, float b, float c) {
  float r;
  asm("max.f32 %0, %1, %2, %3;" : "=f"(r) : "f"(a), "f"(b), "f"(c));
  return r;
}

// 2^x on the FMA pipe for a pair (x0, x1) packed as f32x2: round-to-nearest split x = j + f
// (f in [-1/2, 1/2]) with the 1.5 * 2^23 shifter, 2^f by a degree-3 polynomial fitted to the
// relative error on [-1/2, 1/2] (max 1.0e-4, below the bf16 rounding of P), 2^j added to the
// exponent bits; x clamped at -126 so the result stays normal (~1e-38: zero next to the row's
// 2^0 terms).
__device__ __forceinline__ void ex2_poly2(uint64_t x2, float& y0, float& y1) {
  float a, b;
  f2unpack(x2, a, b);
  a = fmaxf(a, -126.f);
  b = fmaxf(b, -126.f);
  const uint64_t r = fadd2(f2pack(a, b), f2pack(12582912.f, 12582912.f));  // low mantissa bits = round(x)
  const uint64_t j = fadd2(r, f2pack(-12582912.f, -12582912.f));
  const uint64_t f = fadd2(f2pack(a, b), j ^ 0x8000000080000000ull);  // x - round(x)
  uint64_t p = ffma2(f, f2pack(0.05500893f, 0.05500893f), f2pack(0.24221096f, 0.24221096f));
  p = ffma2(p, f, f2pack(0.69328293f, 0.69328293f));
  p = ffma2(p, f, f2pack(1.f, 1.f));
  float p0, p1, r0, r1;
  f2unpack(p, p0, p1);
  f2unpack(r, r0, r1);
  y0 = __int_as_float(__float_as_int(p0) + (__float_as_int(r0) << 23));
  y1 = __int_as_float(__float_as_int(p1) + (__float_as_int(r1) << 23));
}
#if defined(GLLM_VARIANT_EMU1)
constexpr uint32_t WS_EMU_PAIRS = 0x8000u;  // A/B builds: which of the 16 pairs of a 32-score chunk
#elif defined(GLLM_VARIANT_EMU2)
constexpr uint32_t WS_EMU_PAIRS = 0x8080u;
#elif defined(GLLM_VARIANT_EMU4)
constexpr uint32_t WS_EMU_PAIRS = 0x8888u;
#else
constexpr uint32_t WS_EMU_PAIRS = 0u;
#endif

// Orders later uses of tcgen05.ld destination registers after the tcgen05.wait::ld that
// precedes this call (the compiler sees no dependency between the wait and those registers).
__device__ __forceinline__ void reg_fence(uint32_t (&r)[32]) {
#pragma unroll
  for (int i = 0; i < 32; ++i) asm volatile("" : "+r"(r[i])::"memory");
}

// one lane of the (converged) warp: true in the elected lane
__device__ __forceinline__ bool elect_one() {
  uint32_t pred = 0;
  asm volatile(
      "{\n.reg .pred P1;\nelect.sync _|P1, 0xffffffff;\nselp.b32 %0, 1, 0, P1;\n}\n"
      : "+r"(pred));
  return pred != 0;
}

// D[tmem] (+)= A[tmem] . B[smem]
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

template <int D>
__global__ void __launch_bounds__(WS_THREADS, 1)
    prefill_attn_ws_kernel(const AttnArgs a, const PrefillItem* __restrict__ items) {
  using L = WsSmem<D>;
  constexpr int ATOMS = L::ATOMS;
  constexpr int NCH = D / 8;  // 16-byte chunks per Q row
  constexpr int PAGES = WS_KT / 16;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  const uint32_t sbase = ptx::smem_u32(smem);
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + L::BAR);
  uint64_t* q_full = bars;
  uint64_t* kfull = bars + 1;
  uint64_t* kempty = kfull + WS_NSK;  // K slot free: the last S MMA reading it completed
  uint64_t* vfull = kempty + WS_NSK;
  uint64_t* vempty = vfull + WS_NSV;  // V slot free: the last PV MMA reading it completed
  uint64_t* sfull = vempty + WS_NSV;
  uint64_t* pfull = sfull + 2;
  uint64_t* ofull = pfull + 2;
  uint32_t* tmem_slot = reinterpret_cast<uint32_t*>(bars + L::NBAR);

  pdl_trigger();
#ifdef GLLM_VARIANT_TRACE
  unsigned long long tr_wq = 0, tr_wk = 0, tr_wv = 0, tr_wp = 0;
#endif
  pdl_wait();
#ifdef GLLM_VARIANT_TRACE
  const unsigned long long tr_t0 = gtime();  // after the PDL wait: the kernel's own span
#endif
  // grid (Hkv, items): CTAs are dispatched x-fastest, so every kv head of the longest item goes
  // first and the whole grid runs longest-first (the host sorts items by key tiles)
  const PrefillItem it = items[blockIdx.y];
  const int kvh = blockIdx.x;
  const int G = a.Hq / a.Hkv;
  const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
  const int t0 = a.cu_q[it.seq];
  const int c = a.cu_q[it.seq + 1] - t0;
  const int s0 = a.kv_len[it.seq] - c;
  const int nrows = c * G;
  const bool hasB = it.row0 + WS_ROWS < nrows;
  // key tiles each Q tile needs (causal): tile X covers keys 0 .. s0 + (its last row) / G
  const int nA = (s0 + min(it.row0 + WS_ROWS - 1, nrows - 1) / G) / WS_KT + 1;
  const int nB = hasB ? (s0 + min(it.row0 + 2 * WS_ROWS - 1, nrows - 1) / G) / WS_KT + 1 : 0;
  const int n_kt = hasB ? nB : nA;
  const int nblk_seq = (a.kv_len[it.seq] + 15) / 16;
  const int32_t* bt = a.block_table + (size_t)it.seq * a.maxblk;

  if (tid == 0) {
    ptx::mbar_init(q_full, 8);  // one arrive per softmax warp
    for (int s = 0; s < WS_NSK; ++s) {
      ptx::mbar_init(&kfull[s], 1);
      ptx::mbar_init(&kempty[s], 1);
    }
    for (int s = 0; s < WS_NSV; ++s) {
      ptx::mbar_init(&vfull[s], 1);
      ptx::mbar_init(&vempty[s], 1);
    }
    for (int x = 0; x < 2; ++x) {
      ptx::mbar_init(&sfull[x], 1);
      ptx::mbar_init(&pfull[x], 4);  // one arrive per softmax warp
      ptx::mbar_init(&ofull[x], 1);
    }
    ptx::fence_barrier_init();
  }
  if (warp == PW_ALLOC) {
    ptx::tmem_alloc(tmem_slot, 512);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  // register budget by role (per warpgroup, inside each role's branch so the allocator sees each
  // region's budget): producers / MMA issuer / idle warp 56, the softmax warpgroups 224 (they hold a
  // full 128-score row: one TMEM pass per key tile)

  if (warp >= 8) asm volatile("setmaxnreg.dec.sync.aligned.u32 56;" ::: "memory");
  if (warp == PW_K || warp == PW_V) {
    // ---------------- K / V producers: warp 8 streams the K tiles, warp 10 the V tiles.  A page of
    // the cache is already in the SW128 layout (kvpage.cuh), so each 2 KB page atom is copied with
    // 16-byte cp.async (lane l: chunks l, l+32, l+64, l+96; a warp instruction moves 512 B) to its
    // rows of the tile: 16 x 2 KB TMA boxes per tile cost ~2000 cycles of TMA issue per SM, as much
    // as the tile's four MMAs.  A tile's copies are one commit group; the tile is published (fence
    // to the async proxy, then one arrive) once the group completes, while the next tile's copies
    // are in flight.  K ring 3 deep, V ring 2 (V is needed only after the tile's softmax).
    const bool is_k = warp == PW_K;
    const __nv_bfloat16* cache = is_k ? a.kc : a.vc;
    const int ns = is_k ? WS_NSK : WS_NSV;
    uint64_t* full = is_k ? kfull : vfull;
    uint64_t* empty = is_k ? kempty : vempty;
    const uint32_t base = sbase + (is_k ? L::K : L::V);
    auto read_bt = [&](int j) {  // block ids of tile j's pages (past the sequence: its page 0)
      const int kb = j * PAGES + lane;
      return (lane < PAGES && j < n_kt) ? __ldg(bt + (kb < nblk_seq ? kb : 0)) : 0;
    };
    auto publish = [&](int j) {  // tile j's copies (the older commit group) landed
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&full[j % ns]);
    };
    int bnext = read_bt(0);
#pragma unroll 1
    for (int j = 0; j < n_kt; ++j) {
      int bp[PAGES];
#pragma unroll
      for (int p = 0; p < PAGES; ++p) bp[p] = __shfl_sync(0xffffffffu, bnext, p);
      bnext = read_bt(j + 1);
      const int sl = j % ns;
      if (j >= ns) ptx::mbar_wait(&empty[sl], (uint32_t)(((j / ns) - 1) & 1));
      const uint32_t dst = base + sl * L::KV_TILE;
#pragma unroll
      for (int p = 0; p < PAGES; ++p) {
        const __nv_bfloat16* src = cache + ((int64_t)bp[p] * a.Hkv + kvh) * 16 * D;
#pragma unroll
        for (int at = 0; at < ATOMS; ++at)
#pragma unroll
          for (int q = 0; q < 4; ++q)
            ptx::cp_async16(dst + at * L::KV_ATOM + p * 2048 + (lane + 32 * q) * 16, src + at * 1024 + (lane + 32 * q) * 8,
                            true);
      }
      ptx::cp_async_commit();
      if (j >= 1) {
        ptx::cp_async_wait<1>();
        publish(j - 1);
      }
    }
    if (n_kt > 0) {
      ptx::cp_async_wait<0>();
      publish(n_kt - 1);
    }
  } else if (warp == PW_MMA) {
    // ---------------- MMA issuer.  The whole warp runs the schedule (barrier waits, descriptor
    // arithmetic: warp-uniform values the compiler keeps in uniform registers) and one elected lane
    // issues each tcgen05 op.  Descriptors are built once per operand tile; a K step adds its
    // constant byte offset >> 4 to the start-address field (an N = 128 MMA is 64 cycles of tensor
    // work, so per-instruction descriptor building and re-election used to make the issue the
    // bottleneck).
    {
      constexpr uint32_t idesc_s = idesc_bf16(WS_ROWS, WS_KT, false);
      constexpr uint32_t idesc_o = idesc_bf16(WS_ROWS, D, true);
      const uint64_t dq[2] = {ptx::umma_desc_sw128(sbase + L::Q), ptx::umma_desc_sw128(sbase + L::Q + L::Q_TILE)};
      auto issue_s = [&](int x, int j) {
        const uint64_t dk = ptx::umma_desc_sw128(sbase + L::K + (j % WS_NSK) * L::KV_TILE);
        if (elect_one()) {
#pragma unroll
          for (int ks = 0; ks < D / 16; ++ks) {
            const uint64_t oq = (uint64_t)(((ks / 4) * L::Q_ATOM + (ks % 4) * 32) >> 4);
            const uint64_t ok = (uint64_t)(((ks / 4) * L::KV_ATOM + (ks % 4) * 32) >> 4);
            ptx::umma_bf16(tmem + x * 128, dq[x] + oq, dk + ok, idesc_s, ks > 0);
          }
          ptx::umma_commit(&sfull[x]);
        }
        __syncwarp();
      };
      auto issue_pv = [&](int x, int j) {
        const uint64_t dv = desc_mn(sbase + L::V + (j % WS_NSV) * L::KV_TILE, L::KV_ATOM);
        if (elect_one()) {
#pragma unroll
          for (int kk = 0; kk < WS_KT / 16; ++kk)  // 16 keys = 8 TMEM columns of packed P per step
            umma_bf16_ta(tmem + 256 + x * 128, tmem + x * 128 + kk * 8, dv + (uint64_t)((kk * 2048) >> 4), idesc_o,
                         (j > 0 || kk > 0) ? 1u : 0u);
        }
        __syncwarp();
      };
      auto commit = [&](uint64_t* bar) {
        if (elect_one()) ptx::umma_commit(bar);
        __syncwarp();
      };
      auto wait_k = [&](int j) {
        TR_WAIT(tr_wk, ptx::mbar_wait(&kfull[j % WS_NSK], (uint32_t)((j / WS_NSK) & 1)));
        ptx::tc_fence_after();
      };
      TR_WAIT(tr_wq, ptx::mbar_wait(q_full, 0));
      ptx::tc_fence_after();
      wait_k(0);
      issue_s(0, 0);
      if (hasB) issue_s(1, 0);
      commit(&kempty[0]);  // K(0) is read by S_A(0), S_B(0) only
#pragma unroll 1
      for (int j = 0; j < n_kt; ++j) {
        const int s = j % WS_NSV;
        TR_WAIT(tr_wv, ptx::mbar_wait(&vfull[s], (uint32_t)((j / WS_NSV) & 1)));
        bool k_next = false;
        if (j < nA) {
          TR_WAIT(tr_wp, ptx::mbar_wait(&pfull[0], (uint32_t)(j & 1)));
          ptx::tc_fence_after();
          issue_pv(0, j);
          if (j + 1 < nA) {
            wait_k(j + 1);
            k_next = true;
            issue_s(0, j + 1);
          } else {
            commit(&ofull[0]);
          }
        }
        if (hasB) {
          TR_WAIT(tr_wp, ptx::mbar_wait(&pfull[1], (uint32_t)(j & 1)));
          ptx::tc_fence_after();
          issue_pv(1, j);
        }
        commit(&vempty[s]);  // V(j) free once the PVs issued so far complete
        if (hasB) {
          if (j + 1 < nB) {
            if (!k_next) wait_k(j + 1);
            issue_s(1, j + 1);
          } else {
            commit(&ofull[1]);
          }
        }
        if (j + 1 < n_kt) commit(&kempty[(j + 1) % WS_NSK]);  // every S of tile j+1 issued
      }
#ifdef GLLM_VARIANT_TRACE
      if (lane == 0 && g_pf_trace) {
        unsigned long long* rec = g_pf_trace + (size_t)(blockIdx.y * gridDim.x + blockIdx.x) * PF_TR;
        unsigned smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        rec[0] = tr_t0;
        rec[1] = gtime();
        rec[3] = smid;
        rec[4] = tr_wq;
        rec[5] = tr_wk;
        rec[6] = tr_wv;
        rec[7] = tr_wp;
        rec[8] = n_kt;
        rec[9] = nA + nB;
      }
#endif
    }
  } else if (warp < 8) {
    // ---------------- softmax warpgroups (tile X = 0: warps 0-3, X = 1: warps 4-7)
    asm volatile("setmaxnreg.inc.sync.aligned.u32 224;" ::: "memory");
    const int x = warp >> 2;
    const int r = (warp & 3) * 32 + lane;  // row of the Q tile = TMEM lane
    const int rr = it.row0 + x * WS_ROWS + r;
    const int rrc = min(rr, nrows - 1);
    // Q row -> SMEM (rows past the chunk repeat the last row; their output is never stored)
    {
      const int tok = rrc / G, h = kvh * G + rrc % G;
      const __nv_bfloat16* src = a.q + (size_t)(t0 + tok) * a.q_stride + (size_t)h * D;
      const uint32_t qb = sbase + L::Q + x * L::Q_TILE;
#pragma unroll
      for (int ch = 0; ch < NCH; ++ch) ptx::cp_async16(qb + sw128(WS_ROWS, r, ch), src + ch * 8, true);
      ptx::cp_async_commit();
      ptx::cp_async_wait<0>();
      fence_proxy_async_smem();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(q_full);
    }
    const int nx = x == 0 ? nA : nB;
    const int pos = s0 + rrc / G;  // this row's causal limit (keys 0..pos)
    const float sl2 = LOG2E_W * rsqrtf((float)D);
    const uint32_t lane_off = (uint32_t)((warp & 3) * 32) << 16;
    const uint32_t t_s = tmem + lane_off + x * 128;
    const uint32_t t_o = tmem + lane_off + 256 + x * 128;
    float m_ref = -INFINITY, l = 0.f;
#ifdef GLLM_VARIANT_TRACE
    long long ph_w = 0, ph_ld = 0, ph_max = 0, ph_exp = 0, c_a = 0, c_b;
#define PH(acc)    \
  c_b = clock64(); \
  acc += c_b - c_a; \
  c_a = c_b;
#else
#define PH(acc)
#endif
#pragma unroll 1
    for (int j = 0; j < nx; ++j) {
#ifdef GLLM_VARIANT_TRACE
      c_a = clock64();
#endif
      ptx::mbar_wait(&sfull[x], (uint32_t)(j & 1));
      ptx::tc_fence_after();
      PH(ph_w)
      const int kbase = j * WS_KT;
      // causal masking only where some row of this warp ends inside the tile (warp-uniform, so
      // the unmasked path carries no per-element compares)
      const bool diag_w = __any_sync(0xffffffffu, kbase + WS_KT - 1 > pos);
      // one TMEM pass: the whole 128-score row into registers (four loads in flight, one wait)
      uint32_t sr[WS_KT / 32][32];
#pragma unroll
      for (int cq = 0; cq < WS_KT / 32; ++cq) ptx::tmem_ld_32x32b_x32(t_s + cq * 32, sr[cq]);
      ptx::tmem_ld_wait();
#pragma unroll
      for (int cq = 0; cq < WS_KT / 32; ++cq) reg_fence(sr[cq]);
      PH(ph_ld)
      float mx;
      {
        float m4[4] = {-INFINITY, -INFINITY, -INFINITY, -INFINITY};
#pragma unroll
        for (int cq = 0; cq < WS_KT / 32; ++cq) {
          if (diag_w) {
#pragma unroll
            for (int i = 0; i < 32; i += 2)
              m4[(i >> 1) & 3] = fmax3(m4[(i >> 1) & 3], kbase + cq * 32 + i > pos ? -INFINITY : __uint_as_float(sr[cq][i]),
                                       kbase + cq * 32 + i + 1 > pos ? -INFINITY : __uint_as_float(sr[cq][i + 1]));
          } else {
#pragma unroll
            for (int i = 0; i < 32; i += 2)
              m4[(i >> 1) & 3] = fmax3(m4[(i >> 1) & 3], __uint_as_float(sr[cq][i]), __uint_as_float(sr[cq][i + 1]));
          }
        }
        mx = fmaxf(fmaxf(m4[0], m4[1]), fmaxf(m4[2], m4[3])) * sl2;
      }
      const bool mine = mx > m_ref + WS_RESCALE_LOG2;
      const float corr = mine ? ex2(m_ref - mx) : 1.f;
      if (mine) {
        l *= corr;
        m_ref = mx;
      }
      // O_X holds PV_X(0..j-1), complete: S_X(j) was committed after PV_X(j-1)
      if (j > 0 && __any_sync(0xffffffffu, mine)) {
#pragma unroll 1
        for (int cb = 0; cb < D / 32; ++cb) {
          uint32_t orr[32];
          ptx::tmem_ld_32x32b_x32(t_o + cb * 32, orr);
          ptx::tmem_ld_wait();
#pragma unroll
          for (int i = 0; i < 32; ++i) orr[i] = __float_as_uint(__uint_as_float(orr[i]) * corr);
          tmem_st_x32(t_o + cb * 32, orr);
        }
      }
      PH(ph_max)
      // P = exp2(s * scale - m) as bf16 pairs written over the S columns (chunk cq's P lands in
      // columns [16cq, 16cq + 16), whose scores are already in registers); the scale and the row
      // sum run as packed f32x2 FFMA2 / FADD2 (half the FMA-pipe issues)
      float la = 0.f, lb = 0.f;
      {
        const uint64_t sc2 = f2pack(sl2, sl2), nm2 = f2pack(-m_ref, -m_ref);
        uint64_t l2 = f2pack(0.f, 0.f);
#pragma unroll
        for (int cq = 0; cq < WS_KT / 32; ++cq) {
          uint32_t pw[16];
#pragma unroll
          for (int i = 0; i < 16; ++i) {
            float x0, x1;
            const uint64_t xx = ffma2(f2pack(__uint_as_float(sr[cq][2 * i]), __uint_as_float(sr[cq][2 * i + 1])), sc2, nm2);
            float p0, p1;
            if ((WS_EMU_PAIRS >> i) & 1) {
              ex2_poly2(xx, p0, p1);
            } else {
              f2unpack(xx, x0, x1);
              p0 = ex2(x0);
              p1 = ex2(x1);
            }
            if (diag_w) {
              if (kbase + cq * 32 + 2 * i > pos) p0 = 0.f;
              if (kbase + cq * 32 + 2 * i + 1 > pos) p1 = 0.f;
            }
            l2 = fadd2(l2, f2pack(p0, p1));
            pw[i] = ptx::pack_bf16(p0, p1);
          }
          tmem_st_x16(t_s + cq * 16, pw);
        }
        f2unpack(l2, la, lb);
      }
      l += la + lb;
      tmem_st_wait();
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&pfull[x]);
      PH(ph_exp)
    }
#ifdef GLLM_VARIANT_TRACE
    if ((warp & 3) == 0 && lane == 0 && g_pf_trace) {  // warps 0 (tile A) and 4 (tile B)
      unsigned long long* rec = g_pf_trace + (size_t)(blockIdx.y * gridDim.x + blockIdx.x) * PF_TR + 10 + 5 * x;
      rec[0] = ph_w;
      rec[1] = ph_ld;
      rec[2] = ph_max;
      rec[3] = ph_exp;
      rec[4] = nx;
    }
#endif
#undef PH
    if (nx > 0) {
      ptx::mbar_wait(&ofull[x], 0);
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
    }
  }
  ptx::tc_fence_before();
  __syncthreads();
  if (warp == PW_ALLOC) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem, 512);
  }
#ifdef GLLM_VARIANT_TRACE
  if (threadIdx.x == 0 && g_pf_trace) g_pf_trace[(size_t)(blockIdx.y * gridDim.x + blockIdx.x) * PF_TR + 2] = gtime();
#endif
}

template <int D>
int launch_ws(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s) {
  constexpr int bytes = WsSmem<D>::BYTES;
  static bool set = false;
  if (!set) {
    cudaFuncSetAttribute(prefill_attn_ws_kernel<D>, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes);
    set = true;
  }
  launch_pdl(prefill_attn_ws_kernel<D>, dim3(a.Hkv, n_items), dim3(WS_THREADS), bytes, s, 1, a, items);
  return GLLM_OK;
}

}  // namespace

int prefill_ws_rows_per_item() { return 2 * WS_ROWS; }

int launch_prefill_attention_ws(const AttnArgs& a, const PrefillItem* items, int n_items, cudaStream_t s) {
  if (n_items <= 0) return GLLM_OK;
  if (a.bs != 16) return set_error(GLLM_EINVAL, "prefill attention (ws): block size %d unsupported", a.bs);
  if (a.D == 128)
    launch_ws<128>(a, items, n_items, s);
  else if (a.D == 64)
    launch_ws<64>(a, items, n_items, s);
  else
    return set_error(GLLM_EINVAL, "prefill attention (ws): head_dim %d unsupported", a.D);
  cudaError_t e = cudaGetLastError();
  return e == cudaSuccess ? GLLM_OK
                          : set_error(GLLM_ECUDA, "prefill attention (ws) launch: %s", cudaGetErrorString(e));
}

}  // namespace gllm

#ifdef GLLM_VARIANT_TRACE
// measurement build only: arm (n_ctas > 0) or disarm (0) the prefill trace; records of PF_TR words
// per CTA [t_start, t_mma_end, t_end (globaltimer ns), smid, wait cycles q / k / v / p, key tiles,
// tiles of both Q tiles]
extern "C" GLLM_API int gllm_prefill_trace_arm(void* dev_buf) {
  unsigned long long* p = static_cast<unsigned long long*>(dev_buf);
  cudaMemcpyToSymbol(gllm::g_pf_trace, &p, sizeof(p));
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
#endif
