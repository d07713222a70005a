// Persistent warp-specialised tcgen05 GEMM for sm_100a (a5, a8, a9, a10, a11 of DESIGN.md §2).
//
//   Y[M,N] = X[M,K] . W[N,K]^T      X = activations (bf16, K-major), W = weights (bf16, K-major)
//
// Two variants of one kernel template:
//   CG = 2 (default for >= ~1 wave of work): a CTA pair (cluster of 2 on one TPC) computes a
//          256 x 256 tile with tcgen05.mma.cta_group::2 (M=256, N=256, K=16); each CTA loads its
//          128 rows of A and 128 of the 256 rows of B (halving SMEM/L2 operand traffic per
//          FLOP), 6-stage TMA ring of 32 KB stages (5 for the residual add, whose whole tiles
//          stage the residual through SMEM by TMA: res_epilogue_tile), the leader CTA issues the
//          MMAs and commits to both CTAs' barriers (multicast); each CTA drains its own 128 x 256
//          TMEM accumulator.
//   CG = 1: one CTA per 128 x 256 tile (tcgen05.mma.cta_group::1, M=128), 4-stage ring of 48 KB
//          stages; used for small T, where it also supports stream-K (equal k-block ranges per
//          CTA, partial tiles combined with fp32 vector reductions or through a workspace).
// Both: single-thread MMA issue, double-buffered fp32 TMEM accumulator (2 x 256 columns), 4
// epilogue warps (tcgen05.ld) with the fused epilogues: bias, fp32 residual add, SiLU*up,
// RoPE + paged KV append, row argmax for the greedy LM head.  Stage weights (B) are stored tiled
// (gemm.cuh weight_tiled_index: 16 KB contiguous 128 x 64 blocks), so each B box is one DRAM run.
//   warps 0-3: epilogue (warp i reads TMEM lanes 32i..32i+31)
//   warp 4: TMA producer   warp 5: MMA issuer   warp 6: TMEM allocator   warp 7: residual loader
// The single-thread producer and MMA roles sit in the higher warp ids: the SMSP arbiter issues
// the highest eligible warp id first, so a heavy epilogue of the previous tile (on the same SMSPs)
// does not delay the MMA issue of the next tile.
#include <cudaTypedefs.h>

#include <algorithm>
#include <cstdio>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "common.h"
#include "gemm.cuh"
#include "kvpage.cuh"
#include "launch.cuh"
#include "ptx.cuh"

namespace gllm {

int g_force_cg = 0;

namespace {

constexpr int TMEM_COLS = 2 * GEMM_BN;
constexpr int W_PROD = 4, W_MMA = 5, W_ALLOC = 6, W_RES = 7;  // warp roles of gemm_tc_kernel (0-3: epilogue)

// The CTA-pair residual-add kernel (RES) stages the residual through shared memory: RES_BUFS x
// chunks of [128 rows][32 fp32] (16 KB, 128-byte swizzle) loaded by TMA ahead of the accumulator,
// updated in place and stored back by TMA with bf16(x) from XB_BUFS [128][32] bf16 buffers (8 KB,
// 64-byte swizzle).  Its operand ring is one stage shorter to make room.
template <int CG, int EPI>
struct Cfg {
  static constexpr bool RES = CG == 2 && EPI == EPI_ADD_F32;
  static constexpr int B_ROWS = GEMM_BN / CG;  // rows of the B tile loaded by each CTA
  static constexpr int A_BYTES = GEMM_BM * GEMM_BK * 2;
  static constexpr int B_BYTES = B_ROWS * GEMM_BK * 2;
  static constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
#ifdef GLLM_VARIANT_LOWSMEM  // measurement build: leave room for a co-resident attention CTA
  static constexpr int STAGES = CG == 2 ? 4 : 3;
#else
  static constexpr int STAGES = RES ? 5 : (CG == 2 ? 6 : GEMM_STAGES);
#endif
  static constexpr int RES_BUFS = RES ? 3 : 0, RES_BYTES = GEMM_BM * 32 * 4;
  static constexpr int XB_BUFS = RES ? 2 : 0, XB_BYTES = GEMM_BM * 32 * 2;
  static constexpr int RES_OFF = STAGES * STAGE_BYTES;                 // after the operand ring
  static constexpr int BAR_OFF = RES_OFF + RES_BUFS * RES_BYTES + XB_BUFS * XB_BYTES;
  static constexpr int STG_FLOATS = 32 * 36;  // per epilogue warp: 32 x 32 transpose tile (row stride 36)
  static constexpr int STG_BYTES = RES ? 0 : 4 * STG_FLOATS * 4;
  static constexpr int SMEM_BYTES = BAR_OFF + 1024 + 256 + STG_BYTES;
  static constexpr int TILE_M = GEMM_BM * CG;  // rows of one (cluster) tile
};

// x * sigmoid(x) with the approximate reciprocal (MUFU.RCP, ~1 ulp): the IEEE division it replaces
// (reciprocal + Newton step + a range check with a slow path per element) made the SiLU epilogue of
// a 128 x 256 tile take ~9 us, exposed after each CTA's last gate_up tile
__device__ __forceinline__ float silu_f(float x) { return x * __frcp_rn(1.0f + __expf(-x)); }

__device__ __forceinline__ uint32_t cluster_rank() {
  uint32_t r;
  asm volatile("mov.u32 %0, %%cluster_ctarank;" : "=r"(r));
  return r;
}
__device__ __forceinline__ void cluster_sync_all() {
  asm volatile("barrier.cluster.arrive.release.aligned;\nbarrier.cluster.wait.acquire.aligned;" ::: "memory");
}
// TMA 2-D load of this CTA's half of a 2-CTA tile; completion bytes land on the LEADER's barrier
// (peer bit of the shared::cluster address cleared).
__device__ __forceinline__ void tma_load_2d_cg2(void* smem_dst, const CUtensorMap* map, uint64_t* bar, int32_t c0,
                                                int32_t c1) {
  const uint32_t mbar = ptx::smem_u32(bar) & 0xFEFFFFFFu;
  asm volatile(
      "cp.async.bulk.tensor.2d.cta_group::2.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, "
      "%4}], [%2];" ::"r"(ptx::smem_u32(smem_dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(mbar), "r"(c0), "r"(c1)
      : "memory");
}
__device__ __forceinline__ void umma_bf16_cg2(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                              uint32_t accumulate) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "setp.ne.b32 p, %4, 0;\n"
      "tcgen05.mma.cta_group::2.kind::f16 [%0], %1, %2, %3, p;\n"
      "}\n" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate)
      : "memory");
}
// commit of the leader's MMAs, arriving on the barrier at the same offset in both CTAs
__device__ __forceinline__ void umma_commit_cg2(uint64_t* bar) {
  asm volatile(
      "tcgen05.commit.cta_group::2.mbarrier::arrive::one.shared::cluster.multicast::cluster.b64 [%0], %1;" ::"r"(
          ptx::smem_u32(bar)),
      "h"((uint16_t)3)
      : "memory");
}
// distributed shared memory: the address of `addr` in cluster CTA `rank`, and a 16-byte load there
__device__ __forceinline__ uint32_t mapa_u32(uint32_t addr, uint32_t rank) {
  uint32_t r;
  asm volatile("mapa.shared::cluster.u32 %0, %1, %2;" : "=r"(r) : "r"(addr), "r"(rank));
  return r;
}
__device__ __forceinline__ float4 ld_dsmem_v4(uint32_t addr) {
  float4 v;
  asm volatile("ld.shared::cluster.v4.f32 {%0, %1, %2, %3}, [%4];"
               : "=f"(v.x), "=f"(v.y), "=f"(v.z), "=f"(v.w)
               : "r"(addr)
               : "memory");
  return v;
}
#ifdef GLLM_VARIANT_TRACE
// measurement build only (build.py --variant=trace): per-CTA phase stamps of the GEMM (globaltimer ns)
__device__ unsigned long long* g_gm_trace = nullptr;
constexpr int GM_TR = 48;  // words per CTA: 0 entry, 1 setup done, 2 last MMA issued, 3 accumulator ready
                           // (epilogue warp 4), 4 partial in SMEM / first tile drained, 5 cluster sync,
                           // 6 reduce + epilogue done, 7 exit, 8 smid, 9 first operand stage landed
                           // (MMA issuer), 10 + 2j / 11 + 2j: tile j's accumulator ready / drained
                           // (epilogue warp 4, j < 16)
__device__ __forceinline__ void gm_stamp(int i) {
  if (g_gm_trace) {
    unsigned long long t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    g_gm_trace[(size_t)blockIdx.x * GM_TR + i] = t;
  }
}
#define GM_STAMP(i) gm_stamp(i)
#define GM_STAMP_TILE(j, w) \
  if ((j) < 16) gm_stamp(10 + 2 * (j) + (w))
#else
#define GM_STAMP_TILE(j, w) \
  do {                      \
  } while (0)
#define GM_STAMP(i) \
  do {              \
  } while (0)
#endif
// cluster split-K: each CTA's fp32 partial tile in its own SMEM as 8 planes, one per 32-column chunk:
// plane c = [128 rows][32 floats] (16 KB contiguous), the 16-byte granules of row r XOR-swizzled by
// r & 7 (conflict-free when thread = row).  Every CTA uses the same layout, so the reduction over the
// cluster is an element-wise sum of whole planes: a warp reads 512 contiguous bytes of a peer's plane
// per instruction (DSMEM wants coalesced accesses; per-row 16-byte reads ran at ~3 B/cycle).
constexpr int CL_PLANE = 128 * 32 * 4;
constexpr int SKC_MAX_S = 8;  // cluster split-K: at most 8 CTAs per tile (portable cluster size)
__device__ __forceinline__ uint32_t cl_off(int row, int c, int q) {  // byte offset of granule q of (row, chunk c)
  return (uint32_t)(c * CL_PLANE + row * 128 + ((q ^ (row & 7)) << 4));
}
struct ClSrc {
  uint32_t part;  // local SMEM address of the reduced planes (0: not cluster split-K)
  int S, r;       // cluster size, this CTA's rank
};
// The 32-column chunks of a tile whose epilogue cluster rank r runs: unit u = a chunk, or for the
// RoPE epilogue a rotate-half pair (c, c + D/64) of one head, or for SiLU-mul a gate / up pair;
// units are dealt round robin.
template <int EPI>
__device__ __forceinline__ bool cl_owns(const GemmArgs& p, int c, int S, int r) {
  int unit = c;
  if constexpr (EPI == EPI_QKV_ROPE) {
    const int per_head = p.head_dim / 32;
    unit = (c / per_head) * (per_head / 2) + (c % per_head) % (per_head / 2);
  } else if constexpr (EPI == EPI_SILU_MUL) {
    unit = c % (GEMM_BN / 64);
  }
  return unit % S == r;
}

// arrive on the leader CTA's copy of a barrier (from either CTA of the pair)
__device__ __forceinline__ void mbar_arrive_leader(uint64_t* bar) {
  asm volatile(
      "{\n"
      ".reg .b32 ra;\n"
      "mapa.shared::cluster.u32 ra, %0, 0;\n"
      "mbarrier.arrive.release.cluster.shared::cluster.b64 _, [ra];\n"
      "}\n" ::"r"(ptx::smem_u32(bar))
      : "memory");
}
template <int CG>
__device__ __forceinline__ void tmem_alloc_cg(uint32_t* dst, uint32_t ncols) {
  if constexpr (CG == 1) {
    ptx::tmem_alloc(dst, ncols);
    ptx::tmem_relinquish();
  } else {
    asm volatile("tcgen05.alloc.cta_group::2.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(ptx::smem_u32(dst)),
                 "r"(ncols)
                 : "memory");
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::2.sync.aligned;" ::: "memory");
  }
}
template <int CG>
__device__ __forceinline__ void tmem_dealloc_cg(uint32_t taddr, uint32_t ncols) {
  if constexpr (CG == 1)
    ptx::tmem_dealloc(taddr, ncols);
  else
    asm volatile("tcgen05.dealloc.cta_group::2.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols) : "memory");
}

// Job iterator shared by the three warp roles (each role walks the same sequence).  `unit` is
// the CTA (CG=1) or the cluster (CG=2) index, `nunits` their count.
// mode 0: whole tiles round robin.  mode 1: stream-K over all (tile, k-block) units.  mode 2
// (hybrid): whole tiles for the first dp_tiles = full waves, then stream-K over the tail tiles'
// k-blocks, so a last wave that would be mostly empty is spread over every unit.
struct Jobs {
  int mode, ntiles, nk, per, total, unit, nunits, dp_tiles;
  int it, u, u1;
  __device__ void init(const GemmArgs& p, int unit_, int nunits_, int num_m) {
    mode = p.streamk;
    ntiles = num_m * p.num_n_tiles;
    nk = p.K / GEMM_BK;
    per = p.units_per_cta;
    dp_tiles = mode == 2 ? p.dp_tiles : 0;
    total = (ntiles - dp_tiles) * nk;
    unit = unit_;
    nunits = nunits_;
    it = 0;
    u = unit * per;
    u1 = min(total, u + per);
  }
  __device__ bool next(int& tile, int& kb0, int& kb1) {
    if (mode == 3) {  // cluster split-K: one (tile, k range) per CTA; unit = the CTA index
      if (it++ > 0) return false;
      const int S = per, r = unit % S;
      tile = unit / S;
      kb0 = r * nk / S;
      kb1 = (r + 1) * nk / S;
      return true;
    }
    if (mode == 0 || (mode == 2 && unit + it * nunits < dp_tiles)) {
      tile = unit + it * nunits;
      ++it;
      kb0 = 0;
      kb1 = nk;
      return tile < (mode == 0 ? ntiles : dp_tiles);
    }
    if (u >= u1) return false;
    tile = u / nk;
    kb0 = u - tile * nk;
    kb1 = min(nk, kb0 + (u1 - u));
    u += kb1 - kb0;
    tile += dp_tiles;
    return true;
  }
};

__device__ __forceinline__ void store_bf16x32(__nv_bfloat16* dst, const float* v) {
  uint4* d = reinterpret_cast<uint4*>(dst);
#pragma unroll
  for (int q = 0; q < 4; ++q) {
    uint4 w;
    w.x = ptx::pack_bf16(v[q * 8 + 0], v[q * 8 + 1]);
    w.y = ptx::pack_bf16(v[q * 8 + 2], v[q * 8 + 3]);
    w.z = ptx::pack_bf16(v[q * 8 + 4], v[q * 8 + 5]);
    w.w = ptx::pack_bf16(v[q * 8 + 6], v[q * 8 + 7]);
    d[q] = w;
  }
}

// 32 consecutive fp32 reductions as 8 vector reductions (red.global.add.v4.f32, sm_90+)
__device__ __forceinline__ void atomic_add_f32x32(float* dst, const uint32_t (&r)[32]) {
#pragma unroll
  for (int q = 0; q < 8; ++q)
    asm volatile("red.global.add.v4.f32 [%0], {%1, %2, %3, %4};" ::"l"(dst + 4 * q), "r"(r[q * 4 + 0]),
                 "r"(r[q * 4 + 1]), "r"(r[q * 4 + 2]), "r"(r[q * 4 + 3])
                 : "memory");
}

// RoPE (rotate-half) of a 32-element chunk pair (x1 = dims i0.., x2 = dims i0+D/2..) with the
// row's (cos, sin) table, then stores to q (row of `out`), or to the paged K / V cache.
__device__ __forceinline__ void qkv_rope_store(const GemmArgs& p, int row, int col1, int i0, float* x1, float* x2,
                                               int64_t blk, int64_t off) {
  const int D = p.head_dim, half = D / 2;
  if (col1 < p.q_dim + p.kv_dim) {
    const float4* cs = reinterpret_cast<const float4*>(p.rope_cs + (size_t)row * half + i0);
#pragma unroll
    for (int j = 0; j < 16; ++j) {
      const float4 v = __ldg(cs + j);  // (cos, sin) of elements 2j, 2j+1
      const float a1 = x1[2 * j], a2 = x2[2 * j], b1 = x1[2 * j + 1], b2 = x2[2 * j + 1];
      x1[2 * j] = a1 * v.x - a2 * v.y;
      x2[2 * j] = a2 * v.x + a1 * v.y;
      x1[2 * j + 1] = b1 * v.z - b2 * v.w;
      x2[2 * j + 1] = b2 * v.z + b1 * v.w;
    }
  }
  if (col1 < p.q_dim) {
    __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(p.out) + (size_t)row * p.ldo;
    store_bf16x32(out + col1, x1);
    store_bf16x32(out + col1 + half, x2);
  } else {  // paged K / V append in the SMEM-ready page layout (kvpage.cuh): four 16-byte chunks each
    const bool is_k = col1 < p.q_dim + p.kv_dim;
    const int cc = col1 - p.q_dim - (is_k ? 0 : p.kv_dim);
    const int64_t page = blk * p.n_kv_heads + cc / D;
    __nv_bfloat16* cache = is_k ? p.kc : p.vc;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      uint4 w1, w2;
      w1.x = ptx::pack_bf16(x1[8 * q + 0], x1[8 * q + 1]);
      w1.y = ptx::pack_bf16(x1[8 * q + 2], x1[8 * q + 3]);
      w1.z = ptx::pack_bf16(x1[8 * q + 4], x1[8 * q + 5]);
      w1.w = ptx::pack_bf16(x1[8 * q + 6], x1[8 * q + 7]);
      w2.x = ptx::pack_bf16(x2[8 * q + 0], x2[8 * q + 1]);
      w2.y = ptx::pack_bf16(x2[8 * q + 2], x2[8 * q + 3]);
      w2.z = ptx::pack_bf16(x2[8 * q + 4], x2[8 * q + 5]);
      w2.w = ptx::pack_bf16(x2[8 * q + 6], x2[8 * q + 7]);
      *reinterpret_cast<uint4*>(cache + kv_page_elem(page, (int)off, i0 + 8 * q, D)) = w1;
      *reinterpret_cast<uint4*>(cache + kv_page_elem(page, (int)off, i0 + half + 8 * q, D)) = w2;
    }
  }
}

// fused RMSNorm scale of an output row (1 when the A operand is already normalised)
__device__ __forceinline__ float row_scale(const GemmArgs& p, int row) {
  return (p.row_ss != nullptr && row < p.M) ? rsqrtf(__ldg(p.row_ss + row) * p.inv_h + p.eps) : 1.0f;
}

// One warp's 32 rows of one 256-column accumulator tile: wait for the MMAs (tfull), drain TMEM,
// apply the fused epilogue.  `partial`: stream-K segment, combine atomically (the residual add
// straight into x; non-additive epilogues into the fp32 workspace ws, finished by
// gemm_finish_kernel).  `cl`: cluster split-K, the tile's sums come from the cluster's SMEM.
template <int EPI>
__device__ __forceinline__ void epilogue_tile(const GemmArgs& p, uint32_t tbase, int row, int n_blk, bool partial,
                                              uint64_t* tfull_bar, uint32_t parity, float* stg,
                                              ClSrc cl = ClSrc{0u, 1, 0}) {
  const bool row_ok = row < p.M;
  const bool from_cl = cl.part != 0u;  // cluster split-K: sums of the cluster's partial tiles (DSMEM)
  // column chunks (32 wide) this CTA finishes: all, or (cluster split-K) its share of the tile's
  // epilogue units -- a chunk, or a rotate-half / gate-up chunk pair
  auto own = [&](int c) { return !from_cl || cl_owns<EPI>(p, c, cl.S, cl.r); };
  const int trow = threadIdx.x & 127;
  const float rs = (EPI == EPI_ADD_F32 || EPI == EPI_ARGMAX) ? 1.0f : row_scale(p, row);
  uint32_t r[32];
  auto wait_acc = [&]() {
    ptx::mbar_wait(tfull_bar, parity);
    ptx::tc_fence_after();
  };
  // While the MMAs of this tile run, pull the epilogue's other inputs into L2: the residual row
  // segment (read-modify-write) or the row's RoPE table; one 128-B line per prefetch.
  if (row_ok && !partial) {
    if constexpr (EPI == EPI_ADD_F32) {
      const float* xr = reinterpret_cast<const float*>(p.out) + (size_t)row * p.ldo + n_blk * GEMM_BN;
      const int ncol = min(GEMM_BN, p.N - n_blk * GEMM_BN);
      for (int c = 0; c < ncol; c += 32) asm volatile("prefetch.global.L2 [%0];" ::"l"(xr + c));
    } else if constexpr (EPI == EPI_QKV_ROPE) {
      const float* cs = reinterpret_cast<const float*>(p.rope_cs + (size_t)row * (p.head_dim / 2));
      for (int c = 0; c < p.head_dim; c += 32) asm volatile("prefetch.global.L2 [%0];" ::"l"(cs + c));
    }
  }
  if (!from_cl && p.ws != nullptr && partial) {  // stream-K segment of a non-additive epilogue
    wait_acc();
#pragma unroll 1
    for (int c = 0; c < GEMM_BN / 32; ++c) {
      ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
      ptx::tmem_ld_wait();
      const int col0 = n_blk * GEMM_BN + c * 32;
      if (row_ok && col0 < p.N) atomic_add_f32x32(p.ws + (size_t)row * p.N + col0, r);
    }
    return;  // gemm_finish_kernel applies the epilogue
  }
  if (p.zero_rows != nullptr && n_blk == 0 && row_ok && !partial && cl.r == 0) p.zero_rows[row] = 0.f;
  // accumulator columns [col, col + 32) of this tile's row: from TMEM or (cluster split-K) summed
  // over the cluster's partial tiles
  auto ld = [&](int col, uint32_t(&v)[32]) {
    if (from_cl) {  // the chunk's cluster sum, already reduced into this CTA's plane
#pragma unroll
      for (int q = 0; q < 8; ++q) {
        float4 x;
        asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                     : "=f"(x.x), "=f"(x.y), "=f"(x.z), "=f"(x.w)
                     : "r"(cl.part + cl_off(trow, col / 32, q)));
        v[4 * q] = __float_as_uint(x.x);
        v[4 * q + 1] = __float_as_uint(x.y);
        v[4 * q + 2] = __float_as_uint(x.z);
        v[4 * q + 3] = __float_as_uint(x.w);
      }
      return;
    }
    ptx::tmem_ld_32x32b_x32(tbase + col, v);
  };
  auto ld_wait = [&]() {
    if (!from_cl) ptx::tmem_ld_wait();
  };
  auto wait_src = [&]() {
    if (!from_cl) wait_acc();
  };
  if constexpr (EPI == EPI_STORE_BF16) {
    wait_src();
    __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(p.out);
#pragma unroll 1
    for (int c = 0; c < GEMM_BN / 32; ++c) {
      if (!own(c)) continue;
      ld(c * 32, r);
      ld_wait();
      const int col0 = n_blk * GEMM_BN + c * 32;
      if (row_ok && col0 < p.N) {
        float v[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) v[j] = __uint_as_float(r[j]) * rs + (p.bias ? __ldg(p.bias + col0 + j) : 0.f);
        store_bf16x32(out + (size_t)row * p.ldo + col0, v);
      }
    }
  } else if constexpr (EPI == EPI_ADD_F32) {
    if (partial) {  // stream-K segment: fp32 vector reductions, one row per thread
      float* rowp = reinterpret_cast<float*>(p.out) + (size_t)row * p.ldo + n_blk * GEMM_BN;
      wait_acc();
#pragma unroll 1
      for (int c = 0; c < GEMM_BN / 32; ++c) {
        ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
        ptx::tmem_ld_wait();
        if (row_ok && n_blk * GEMM_BN + c * 32 < p.N) atomic_add_f32x32(rowp + c * 32, r);
      }
    } else {
      // Whole tile: each 32 x 32 chunk of the accumulator (thread = row after tcgen05.ld) is
      // re-laid through SMEM so that 8 lanes cover one row's 32 columns (float4 each): every
      // warp access of the residual read-modify-write and of the bf16 copy for the next norm
      // is 4 whole 128-B (64-B) row segments instead of 32 scattered rows, which keeps the
      // L1/SMEM pipe free for the concurrent mainloop's operand reads.
      const int lane = threadIdx.x & 31, row0 = row - lane;
      const int rsub = lane >> 3, c4 = (lane & 7) * 4;  // this lane: rows rsub + 4k, columns c4..c4+3
      float ss[8];
#pragma unroll
      for (int k = 0; k < 8; ++k) ss[k] = 0.f;
      // the residual rows of chunk c + 1 are loaded while chunk c is combined (two register
      // buffers); chunk 0's are loaded before the accumulator is ready, under the mainloop
      auto load_x = [&](int c, float4(&xv)[8]) {
        const int col = n_blk * GEMM_BN + c * 32 + c4;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const int rr = rsub + 4 * k;
          xv[k] = (col < p.N && row0 + rr < p.M)
                      ? *reinterpret_cast<const float4*>(reinterpret_cast<const float*>(p.out) +
                                                         (size_t)(row0 + rr) * p.ldo + col)
                      : make_float4(0.f, 0.f, 0.f, 0.f);
        }
      };
      auto combine = [&](int c, const float4(&xv)[8]) {
        ld(c * 32, r);
        ld_wait();
#pragma unroll
        for (int q = 0; q < 8; ++q)  // row `lane` of the chunk (stride 36 floats: conflict-free v4)
          *reinterpret_cast<float4*>(stg + lane * 36 + 4 * q) =
              make_float4(__uint_as_float(r[4 * q]), __uint_as_float(r[4 * q + 1]), __uint_as_float(r[4 * q + 2]),
                          __uint_as_float(r[4 * q + 3]));
        __syncwarp();
        const int col = n_blk * GEMM_BN + c * 32 + c4;
        const bool col_ok = col < p.N;
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          const int rr = rsub + 4 * k;
          if (col_ok && row0 + rr < p.M) {
            const float4 a4 = *reinterpret_cast<const float4*>(stg + rr * 36 + c4);
            float4 x = xv[k];
            x.x += a4.x;
            x.y += a4.y;
            x.z += a4.z;
            x.w += a4.w;
            *reinterpret_cast<float4*>(reinterpret_cast<float*>(p.out) + (size_t)(row0 + rr) * p.ldo + col) = x;
            if (p.out_peer) *reinterpret_cast<float4*>(p.out_peer + (size_t)(row0 + rr) * p.ldo + col) = x;
            if (p.xb_out) {
              uint2 b;
              b.x = ptx::pack_bf16(x.x, x.y);
              b.y = ptx::pack_bf16(x.z, x.w);
              *reinterpret_cast<uint2*>(p.xb_out + (size_t)(row0 + rr) * p.ldo + col) = b;
              ss[k] = fmaf(x.x, x.x, fmaf(x.y, x.y, fmaf(x.z, x.z, fmaf(x.w, x.w, ss[k]))));
            }
          }
        }
        __syncwarp();
      };
      float4 xa[8], xb[8];
      if (from_cl) {  // this CTA's chunks of the tile, summed over the cluster
        int c = 0;
        while (c < GEMM_BN / 32 && !own(c)) ++c;
        if (c < GEMM_BN / 32) load_x(c, xa);
#pragma unroll 1
        while (c < GEMM_BN / 32) {
          int cn = c + 1;
          while (cn < GEMM_BN / 32 && !own(cn)) ++cn;
          if (cn < GEMM_BN / 32) load_x(cn, xb);
          combine(c, xa);
#pragma unroll
          for (int k = 0; k < 8; ++k) xa[k] = xb[k];
          c = cn;
        }
      } else {
        load_x(0, xa);
        wait_acc();
#pragma unroll 1
        for (int c = 0; c < GEMM_BN / 32; c += 2) {
          load_x(c + 1, xb);
          combine(c, xa);
          if (c + 2 < GEMM_BN / 32) load_x(c + 2, xa);
          combine(c + 1, xb);
        }
      }
      if (p.ss_out) {  // row rsub + 4k: its 32 columns of this tile are spread over 8 lanes
#pragma unroll
        for (int k = 0; k < 8; ++k) {
          float v = ss[k];
          v += __shfl_xor_sync(0xffffffffu, v, 1);
          v += __shfl_xor_sync(0xffffffffu, v, 2);
          v += __shfl_xor_sync(0xffffffffu, v, 4);
          const int rw = row0 + rsub + 4 * k;
          if ((lane & 7) == 0 && rw < p.M && n_blk * GEMM_BN < p.N) atomicAdd(p.ss_out + rw, v);
        }
      }
    }
  } else if constexpr (EPI == EPI_SILU_MUL) {
    wait_src();
    __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(p.out);
    uint32_t u[32];
#pragma unroll 1
    for (int c = 0; c < GEMM_BN / 64; ++c) {
      if (!own(c)) continue;
      ld(c * 32, r);                // gate columns
      ld(GEMM_BN / 2 + c * 32, u);  // up columns
      ld_wait();
      const int col0 = n_blk * (GEMM_BN / 2) + c * 32;
      if (row_ok && col0 < p.N / 2) {
        float h[32];
#pragma unroll
        for (int j = 0; j < 32; ++j) h[j] = silu_f(__uint_as_float(r[j]) * rs) * (__uint_as_float(u[j]) * rs);
        store_bf16x32(out + (size_t)row * p.ldo + col0, h);
      }
    }
  } else if constexpr (EPI == EPI_QKV_ROPE) {
    // The 256 columns of a tile are whole heads (D | 256); rotate-half partners (i, i + D/2)
    // are 32-column chunks c and c + D/64 of the same head.
    const int per_head = p.head_dim / 32;
    const int slot = row_ok ? __ldg(p.slots + row) : 0;
    const int64_t blk = slot / p.block_size, off = slot % p.block_size;
    uint32_t u[32];
    wait_src();
#pragma unroll 1
    for (int c = 0; c < GEMM_BN / 32; ++c) {
      const int hpos = c % per_head;
      if (hpos >= per_head / 2 || !own(c)) continue;
      ld(c * 32, r);
      ld((c + per_head / 2) * 32, u);
      ld_wait();
      const int col1 = n_blk * GEMM_BN + c * 32;
      if (!row_ok || col1 >= p.N) continue;
      float x1[32], x2[32];
#pragma unroll
      for (int j = 0; j < 32; ++j) {
        x1[j] = __uint_as_float(r[j]) * rs + (p.bias ? __ldg(p.bias + col1 + j) : 0.f);
        x2[j] = __uint_as_float(u[j]) * rs + (p.bias ? __ldg(p.bias + col1 + p.head_dim / 2 + j) : 0.f);
      }
      qkv_rope_store(p, row, col1, hpos * 32, x1, x2, blk, off);
    }
  } else {  // EPI_ARGMAX
    wait_acc();
    float best = -INFINITY;
    int best_i = 0x7fffffff;
#pragma unroll 1
    for (int c = 0; c < GEMM_BN / 32; ++c) {
      ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
      ptx::tmem_ld_wait();
      const int col0 = n_blk * GEMM_BN + c * 32;
#pragma unroll
      for (int j = 0; j < 32; ++j) {
        const float v = __uint_as_float(r[j]);
        if (col0 + j < p.N && v > best) {  // strict: lowest column wins ties (R18)
          best = v;
          best_i = col0 + j;
        }
      }
    }
    if (row_ok) {
      p.part_val[(size_t)row * p.num_n_tiles + n_blk] = best;
      p.part_idx[(size_t)row * p.num_n_tiles + n_blk] = best_i;
    }
  }
}

// Residual add of one whole tile through shared memory (CTA-pair kernel, EPI_ADD_F32): this
// CTA's 128 rows x the tile's 32-column chunks.  Thread = row (TMEM lane).  Per chunk: the
// accumulator columns from TMEM, the residual chunk from its TMA-loaded buffer (loaded ahead by
// the residual loader warp while the MMAs ran), x += acc written back in place, bf16(x) into an XB
// buffer; one elected thread TMA-stores both chunks and hands the residual buffer back to the
// loader once the store has read it.  The row's sum of squares accumulates in a register.
template <int EPI, int CG>
__device__ __forceinline__ void res_epilogue_tile(const GemmArgs& p, const CUtensorMap* tmx, const CUtensorMap* tmxb,
                                                  uint32_t tbase, int row_base, int n_blk, uint64_t* tfull_bar,
                                                  uint32_t parity, uint32_t res_s, uint32_t xb_s, uint64_t* res_full,
                                                  uint64_t* res_empty, int& rc, int& xc) {
  using C = Cfg<CG, EPI>;
  const int t = threadIdx.x;  // row of the CTA's 128 (epilogue warps 0-3)
  const int row = row_base + t;
  const bool issuer = t == 0;
  const int nch = min(GEMM_BN, p.N - n_blk * GEMM_BN) / 32;
  float ss = 0.f;
  uint32_t r[32];
  ptx::mbar_wait(tfull_bar, parity);
  ptx::tc_fence_after();
  int prev_buf = -1;
#pragma unroll 1
  for (int c = 0; c < nch; ++c) {
    const int buf = rc % C::RES_BUFS;
    ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
    ptx::mbar_wait(&res_full[buf], (uint32_t)((rc / C::RES_BUFS) & 1));
    ptx::tmem_ld_wait();
    const uint32_t xs = res_s + buf * C::RES_BYTES + t * 128;
    float x[32];
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t a = xs + ((q ^ (t & 7)) << 4);
      asm volatile("ld.shared.v4.f32 {%0, %1, %2, %3}, [%4];"
                   : "=f"(x[4 * q]), "=f"(x[4 * q + 1]), "=f"(x[4 * q + 2]), "=f"(x[4 * q + 3])
                   : "r"(a));
    }
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      x[j] += __uint_as_float(r[j]);
      ss = fmaf(x[j], x[j], ss);
    }
#pragma unroll
    for (int q = 0; q < 8; ++q) {
      const uint32_t a = xs + ((q ^ (t & 7)) << 4);
      asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(a), "f"(x[4 * q]), "f"(x[4 * q + 1]),
                   "f"(x[4 * q + 2]), "f"(x[4 * q + 3])
                   : "memory");
    }
    const int col0 = n_blk * GEMM_BN + c * 32;
    if (p.out_peer != nullptr && row < p.M) {  // fused stage hand-off: the new rows to the peer slot too
      float4* d = reinterpret_cast<float4*>(p.out_peer + (size_t)row * p.ldo + col0);
#pragma unroll
      for (int q = 0; q < 8; ++q) d[q] = make_float4(x[4 * q], x[4 * q + 1], x[4 * q + 2], x[4 * q + 3]);
    }
    const uint32_t xbs = xb_s + (xc % C::XB_BUFS) * C::XB_BYTES;
    if (p.xb_out != nullptr) {
      ptx::named_bar_sync(1, 128);  // the store that last read this XB buffer has finished reading it
#pragma unroll
      for (int u = 0; u < 4; ++u) {
        const uint32_t a = xbs + t * 64 + ((u ^ ((t >> 1) & 3)) << 4);
        asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(a), "r"(ptx::pack_bf16(x[8 * u], x[8 * u + 1])),
                     "r"(ptx::pack_bf16(x[8 * u + 2], x[8 * u + 3])), "r"(ptx::pack_bf16(x[8 * u + 4], x[8 * u + 5])),
                     "r"(ptx::pack_bf16(x[8 * u + 6], x[8 * u + 7]))
                     : "memory");
      }
    }
    ptx::fence_proxy_async_smem();
    ptx::named_bar_sync(1, 128);
    if (issuer) {
      ptx::tma_store_2d(tmx, res_s + buf * C::RES_BYTES, col0, row_base);
      if (p.xb_out != nullptr) ptx::tma_store_2d(tmxb, xbs, col0, row_base);
      ptx::bulk_commit();
      ptx::bulk_wait_read<1>();  // the previous chunk's stores have read their buffers
      if (prev_buf >= 0) ptx::mbar_arrive(&res_empty[prev_buf]);
    }
    prev_buf = buf;
    ++rc;
    ++xc;
  }
  if (issuer && prev_buf >= 0) {
    ptx::bulk_wait_read<0>();
    ptx::mbar_arrive(&res_empty[prev_buf]);
  }
  if (p.ss_out != nullptr && row < p.M && nch > 0) atomicAdd(p.ss_out + row, ss);
}

template <int EPI, int CG>
__global__ void __launch_bounds__(256, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b,
                   const __grid_constant__ CUtensorMap tma_x, const __grid_constant__ CUtensorMap tma_xb,
                   const GemmArgs p) {
  using C = Cfg<CG, EPI>;
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + C::STAGES * C::A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(smem + C::BAR_OFF);
  uint64_t* empty = full + C::STAGES;
  uint64_t* tfull = empty + C::STAGES;
  uint64_t* tempty = tfull + 2;
  uint64_t* res_full = tempty + 2;  // RES: residual chunk buffers loaded / free
  uint64_t* res_empty = res_full + C::RES_BUFS;
  uint32_t* tmem_ptr = reinterpret_cast<uint32_t*>(res_empty + C::RES_BUFS);
  float* stg = reinterpret_cast<float*>(smem + C::BAR_OFF + 256);  // epilogue transpose tiles
  const uint32_t res_s = ptx::smem_u32(smem + C::RES_OFF);
  const uint32_t xb_s = res_s + C::RES_BUFS * C::RES_BYTES;

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  const bool skc = p.streamk == 3;  // cluster split-K (CG = 1 kernel launched in clusters of split_s)
  const uint32_t rank = CG == 2 ? cluster_rank() : 0;
  const bool leader = rank == 0;
  pdl_trigger();
  if (threadIdx.x == 0) GM_STAMP(0);
  if (warp == W_PROD && lane == 0) {
    ptx::tma_prefetch(&tma_a);
    ptx::tma_prefetch(&tma_b);
  }
  if constexpr (C::RES) {
    if (warp == W_RES && lane == 0) {
      ptx::tma_prefetch(&tma_x);
      if (p.xb_out) ptx::tma_prefetch(&tma_xb);
    }
  }
  if (warp == W_MMA && lane == 0) {
    for (int s = 0; s < C::STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      ptx::mbar_init(&tfull[s], 1);
      ptx::mbar_init(&tempty[s], 4 * CG);  // every epilogue warp of the pair releases the leader's buffer
    }
    for (int s = 0; s < C::RES_BUFS; ++s) {
      ptx::mbar_init(&res_full[s], 1);
      ptx::mbar_init(&res_empty[s], 1);
    }
    ptx::fence_barrier_init();
  }
  if (warp == W_ALLOC) tmem_alloc_cg<CG>(tmem_ptr, TMEM_COLS);
  ptx::tc_fence_before();
  if (CG == 2 || skc)
    cluster_sync_all();
  else
    __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_ptr;
  if (threadIdx.x == 0) GM_STAMP(1);
  // A operand, residual, workspace, slots: produced by earlier kernels.  The producer thread waits
  // after issuing the dependency-free weight tiles of its first ring fill (below).
  if (warp != W_PROD || lane != 0) pdl_wait();

  const int num_m = (p.M + C::TILE_M - 1) / C::TILE_M;
  Jobs jobs;
  jobs.init(p, skc ? (int)blockIdx.x : (int)blockIdx.x / CG, gridDim.x / CG, num_m);
  int tile, kb0, kb1;

  if (warp == W_PROD) {
    if (lane == 0) {
      // ---------------- TMA producer (both CTAs of a pair load their halves)
      // B box coordinates: the row-major [N, K] map (k, row), or the tiled weight's [blocks*128, 64]
      // view, where the 128-row slab of `row` at k-block kb is block slab * nk + kb
      const int nkb = p.K / GEMM_BK;
      auto bx = [&](int kb) -> int32_t { return p.b_tiled ? 0 : kb * GEMM_BK; };
      auto by = [&](int row, int kb) -> int32_t { return p.b_tiled ? ((row >> 7) * nkb + kb) * 128 : row; };
      int stage = 0;
      uint32_t phase = 0;
      int pre = 0;  // stages whose B tile (and expect_tx) went out before the wait
      if (p.b_static) {
        Jobs pj = jobs;
        if (pj.next(tile, kb0, kb1)) {
          const int b_row = (tile / num_m) * GEMM_BN + rank * C::B_ROWS;
          pre = min(C::STAGES, kb1 - kb0);
          for (int i = 0; i < pre; ++i) {  // fresh ring: every empty barrier passes
            const int kb = kb0 + i;
            if constexpr (CG == 1) {
              ptx::mbar_arrive_expect_tx(&full[i], C::STAGE_BYTES);
              ptx::tma_load_2d(sB + i * C::B_BYTES, &tma_b, &full[i], bx(kb), by(b_row, kb));
              ptx::tma_load_2d(sB + i * C::B_BYTES + GEMM_B_BOX * 128, &tma_b, &full[i], bx(kb),
                               by(b_row + GEMM_B_BOX, kb));
            } else {
              if (leader) ptx::mbar_arrive_expect_tx(&full[i], 2 * C::STAGE_BYTES);
              tma_load_2d_cg2(sB + i * C::B_BYTES, &tma_b, &full[i], bx(kb), by(b_row, kb));
            }
          }
        }
      }
      pdl_wait();
      while (jobs.next(tile, kb0, kb1)) {
        const int m_blk = tile % num_m, n_blk = tile / num_m;
        const int a_row = m_blk * C::TILE_M + rank * GEMM_BM;
        const int b_row = n_blk * GEMM_BN + rank * C::B_ROWS;
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&empty[stage], phase ^ 1);
          if (pre > 0) {  // B and the expect_tx of this stage were issued before the wait
            if constexpr (CG == 1)
              ptx::tma_load_2d(sA + stage * C::A_BYTES, &tma_a, &full[stage], kb * GEMM_BK, a_row);
            else
              tma_load_2d_cg2(sA + stage * C::A_BYTES, &tma_a, &full[stage], kb * GEMM_BK, a_row);
            --pre;
          } else if constexpr (CG == 1) {
            ptx::mbar_arrive_expect_tx(&full[stage], C::STAGE_BYTES);
            ptx::tma_load_2d(sA + stage * C::A_BYTES, &tma_a, &full[stage], kb * GEMM_BK, a_row);
            ptx::tma_load_2d(sB + stage * C::B_BYTES, &tma_b, &full[stage], bx(kb), by(b_row, kb));
            ptx::tma_load_2d(sB + stage * C::B_BYTES + GEMM_B_BOX * 128, &tma_b, &full[stage], bx(kb),
                             by(b_row + GEMM_B_BOX, kb));
          } else {
            if (leader) ptx::mbar_arrive_expect_tx(&full[stage], 2 * C::STAGE_BYTES);
            tma_load_2d_cg2(sA + stage * C::A_BYTES, &tma_a, &full[stage], kb * GEMM_BK, a_row);
            tma_load_2d_cg2(sB + stage * C::B_BYTES, &tma_b, &full[stage], bx(kb), by(b_row, kb));
          }
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == W_MMA) {
    if (lane == 0 && leader) {
      // ---------------- MMA issuer (single thread of the leader CTA)
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(C::TILE_M, GEMM_BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      while (jobs.next(tile, kb0, kb1)) {
        ptx::mbar_wait(&tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * GEMM_BN;
        for (int kb = kb0; kb < kb1; ++kb) {
          ptx::mbar_wait(&full[stage], phase);
          ptx::tc_fence_after();
#ifdef GLLM_VARIANT_TRACE
          if (kb == kb0 && acc == 0 && acc_phase == 0) GM_STAMP(9);
#endif
          const uint32_t a_addr = ptx::smem_u32(sA + stage * C::A_BYTES);
          const uint32_t b_addr = ptx::smem_u32(sB + stage * C::B_BYTES);
#pragma unroll
          for (int k = 0; k < GEMM_BK / 16; ++k) {
            const uint64_t ad = ptx::umma_desc_sw128(a_addr + k * 32), bd = ptx::umma_desc_sw128(b_addr + k * 32);
            const uint32_t accum = (kb > kb0 || k > 0) ? 1u : 0u;
            if constexpr (CG == 1)
              ptx::umma_bf16(d_tmem, ad, bd, idesc, accum);
            else
              umma_bf16_cg2(d_tmem, ad, bd, idesc, accum);
          }
          if constexpr (CG == 1)
            ptx::umma_commit(&empty[stage]);  // frees the SMEM slot once these MMAs retire
          else
            umma_commit_cg2(&empty[stage]);   // ... in both CTAs
          if (++stage == C::STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        if constexpr (CG == 1)
          ptx::umma_commit(&tfull[acc]);  // accumulator ready for the epilogue
        else
          umma_commit_cg2(&tfull[acc]);
        acc ^= 1;
        if (acc == 0) acc_phase ^= 1;
      }
      GM_STAMP(2);
    }
  } else if (C::RES && warp == W_RES) {
    // ---------------- residual loader (RES): x chunks of this CTA's whole tiles, RES_BUFS ahead
    if (lane == 0) {
      int rc = 0;
      while (jobs.next(tile, kb0, kb1)) {
        if (kb0 != 0 || kb1 != jobs.nk) continue;  // partial tiles reduce into x with vector atomics
        const int m_blk = tile % num_m, n_blk = tile / num_m;
        const int row_base = m_blk * C::TILE_M + rank * GEMM_BM;
        const int nch = min(GEMM_BN, p.N - n_blk * GEMM_BN) / 32;
        for (int c = 0; c < nch; ++c, ++rc) {
          const int buf = rc % C::RES_BUFS;
          if (rc >= C::RES_BUFS) ptx::mbar_wait(&res_empty[buf], (uint32_t)(((rc / C::RES_BUFS) - 1) & 1));
          ptx::mbar_arrive_expect_tx(&res_full[buf], C::RES_BYTES);
          ptx::tma_load_2d(smem + C::RES_OFF + buf * C::RES_BYTES, &tma_x, &res_full[buf], n_blk * GEMM_BN + c * 32,
                           row_base);
        }
      }
    }
  } else if (warp < 4 && skc) {
    // ---------------- cluster split-K: this CTA's partial tile -> its SMEM (the operand ring is
    // idle: every stage was consumed by the MMAs the tfull commit covers)
    if (jobs.next(tile, kb0, kb1)) {
      ptx::mbar_wait(&tfull[0], 0);
      ptx::tc_fence_after();
      if (threadIdx.x == 0) GM_STAMP(3);
      const int rl = warp * 32 + lane;
      const uint32_t tb = tmem_base + ((uint32_t)(warp * 32) << 16);
      const uint32_t part = ptx::smem_u32(sA);
      uint32_t r[32];
#pragma unroll 1
      for (int c = 0; c < GEMM_BN / 32; ++c) {
        ptx::tmem_ld_32x32b_x32(tb + c * 32, r);
        ptx::tmem_ld_wait();
#pragma unroll
        for (int q = 0; q < 8; ++q)
          asm volatile("st.shared.v4.b32 [%0], {%1, %2, %3, %4};" ::"r"(part + cl_off(rl, c, q)), "r"(r[4 * q]),
                       "r"(r[4 * q + 1]), "r"(r[4 * q + 2]), "r"(r[4 * q + 3])
                       : "memory");
      }
      if (threadIdx.x == 0) GM_STAMP(4);
    }
  } else if (warp < 4) {
    // ---------------- epilogue warps (each CTA drains its own 128 rows)
    const int ew = warp;
    int acc = 0;
    uint32_t acc_phase = 0;
    int ntile = 0;
    int res_rc = 0, res_xc = 0;  // RES: residual / bf16 chunk buffers consumed so far
    while (jobs.next(tile, kb0, kb1)) {
      const int m_blk = tile % num_m, n_blk = tile / num_m;
      const int row = m_blk * C::TILE_M + rank * GEMM_BM + ew * 32 + lane;
#ifdef GLLM_VARIANT_TRACE
      if (threadIdx.x == 0) {
        ptx::mbar_wait(&tfull[acc], acc_phase);
        GM_STAMP_TILE(ntile, 0);
      }
      __syncwarp();
#endif
      const uint32_t tbase = tmem_base + ((uint32_t)(ew * 32) << 16) + acc * GEMM_BN;
      const bool partial = kb0 != 0 || kb1 != jobs.nk;
      if constexpr (C::RES) {
        if (!partial)
          res_epilogue_tile<EPI, CG>(p, &tma_x, &tma_xb, tbase, m_blk * C::TILE_M + rank * GEMM_BM, n_blk, &tfull[acc],
                                     acc_phase, res_s, xb_s, res_full, res_empty, res_rc, res_xc);
        else
          epilogue_tile<EPI>(p, tbase, row, n_blk, true, &tfull[acc], acc_phase, stg + ew * C::STG_FLOATS);
      } else {
        epilogue_tile<EPI>(p, tbase, row, n_blk, partial, &tfull[acc], acc_phase, stg + ew * C::STG_FLOATS);
      }
      if (threadIdx.x == 0) {
        GM_STAMP(4);
        GM_STAMP_TILE(ntile, 1);
      }
      ++ntile;
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) {
        if constexpr (CG == 1)
          ptx::mbar_arrive(&tempty[acc]);
        else
          mbar_arrive_leader(&tempty[acc]);
      }
      acc ^= 1;
      if (acc == 0) acc_phase ^= 1;
    }
    if constexpr (C::RES) {
      if (threadIdx.x == 0) ptx::bulk_wait<0>();  // the residual / bf16 stores are performed
    }
  }
  if (skc) {
    // every partial of the cluster is in SMEM: each CTA reduces its share of the tile's column
    // chunks over DSMEM (rank order) and runs the epilogue; the second cluster barrier keeps every
    // CTA's SMEM alive until the last remote read
    cluster_sync_all();
    if (threadIdx.x == 0) GM_STAMP(5);
    {
      // sum this CTA's planes over the cluster (rank order 0..S-1: deterministic), coalesced, all 8
      // warps: thread t adds granules t, t + 256, t + 512, t + 768 of each owned plane, every
      // source's load in flight before the first add (DSMEM round trips are ~200+ cycles), and
      // writes the sum back into its own plane for the row-per-thread epilogue
      const uint32_t part = ptx::smem_u32(sA);
      const int S = p.split_s, my = (int)cluster_rank();
      Jobs ej;
      ej.init(p, blockIdx.x, gridDim.x, num_m);
      if (ej.next(tile, kb0, kb1)) {
#pragma unroll 1
        for (int c = 0; c < GEMM_BN / 32; ++c) {
          if (!cl_owns<EPI>(p, c, S, my)) continue;
          const uint32_t a0 = part + c * CL_PLANE + threadIdx.x * 16;
          float4 x[4][SKC_MAX_S];
#pragma unroll
          for (int src = 0; src < SKC_MAX_S; ++src)
            if (src < S)
#pragma unroll
              for (int g = 0; g < 4; ++g) x[g][src] = ld_dsmem_v4(mapa_u32(a0 + g * 4096, (uint32_t)src));
#pragma unroll
          for (int g = 0; g < 4; ++g) {
            float4 acc = x[g][0];
#pragma unroll
            for (int src = 1; src < SKC_MAX_S; ++src)
              if (src < S) {
                acc.x += x[g][src].x;
                acc.y += x[g][src].y;
                acc.z += x[g][src].z;
                acc.w += x[g][src].w;
              }
            asm volatile("st.shared.v4.f32 [%0], {%1, %2, %3, %4};" ::"r"(a0 + g * 4096), "f"(acc.x), "f"(acc.y),
                         "f"(acc.z), "f"(acc.w)
                         : "memory");
          }
        }
      }
      __syncthreads();  // planes complete
    }
    if (warp < 4) {
      Jobs ej;
      ej.init(p, blockIdx.x, gridDim.x, num_m);
      if (ej.next(tile, kb0, kb1)) {
        const int ew = warp;
        const int m_blk = tile % num_m, n_blk = tile / num_m;
        const int row = m_blk * C::TILE_M + ew * 32 + lane;
        epilogue_tile<EPI>(p, tmem_base + ((uint32_t)(ew * 32) << 16), row, n_blk, false, &tfull[0], 0,
                           stg + ew * C::STG_FLOATS, ClSrc{ptx::smem_u32(sA), p.split_s, (int)cluster_rank()});
      }
      if (threadIdx.x == 0) GM_STAMP(6);
    }
    ptx::tc_fence_before();
    cluster_sync_all();
  } else {
    ptx::tc_fence_before();
    if constexpr (CG == 2)
      cluster_sync_all();
    else
      __syncthreads();
  }
  if (warp == W_ALLOC) {
    ptx::tc_fence_after();
    tmem_dealloc_cg<CG>(tmem_base, TMEM_COLS);
  }
#ifdef GLLM_VARIANT_TRACE
  if (threadIdx.x == 0 && g_gm_trace) {
    GM_STAMP(7);
    uint32_t smid;
    asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
    g_gm_trace[(size_t)blockIdx.x * GM_TR + 8] = smid;
  }
#endif
}

// Workspace mode: apply the non-additive epilogue to the fp32 sums in ws [M, N].
// One thread per (row, 32-column chunk) of the OUTPUT space of the epilogue.
// Plain (coherent) loads, not __ldg: the finish pass clears the same words after reading them, and
// a read-only load may legally be reordered after those stores.
__device__ __forceinline__ void ld_f32x32(const float* src, float (&v)[32]) {  // 8 x 16-B loads
  const float4* s4 = reinterpret_cast<const float4*>(src);
#pragma unroll
  for (int q = 0; q < 8; ++q) {
    const float4 x = s4[q];
    v[4 * q] = x.x;
    v[4 * q + 1] = x.y;
    v[4 * q + 2] = x.z;
    v[4 * q + 3] = x.w;
  }
}

// the finish pass leaves the workspace zero for the next stream-K launch (no memset launch, so the
// PDL chain runs unbroken from the producing kernel into the GEMM)
__device__ __forceinline__ void zero_f32x32(const float* p) {
  float4* d = reinterpret_cast<float4*>(const_cast<float*>(p));
#pragma unroll
  for (int q = 0; q < 8; ++q) d[q] = make_float4(0.f, 0.f, 0.f, 0.f);
}

template <int EPI>
__global__ void __launch_bounds__(256) gemm_finish_kernel(const GemmArgs p) {
  pdl_trigger();
  pdl_wait();
  const int chunks_per_row = (EPI == EPI_SILU_MUL) ? p.N / 64 : p.N / 32;
  const int idx = blockIdx.x * blockDim.x + threadIdx.x;
  if (idx >= p.M * chunks_per_row) return;
  const int row = idx / chunks_per_row, c = idx % chunks_per_row;
  const float* w = p.ws + (size_t)row * p.N;
  const float rs = row_scale(p, row);
  if (p.zero_rows != nullptr && c == 0) p.zero_rows[row] = 0.f;
  if constexpr (EPI == EPI_STORE_BF16) {
    float v[32];
    ld_f32x32(w + c * 32, v);
    zero_f32x32(w + c * 32);
#pragma unroll
    for (int j = 0; j < 32; ++j) v[j] = v[j] * rs + (p.bias ? p.bias[c * 32 + j] : 0.f);
    store_bf16x32(reinterpret_cast<__nv_bfloat16*>(p.out) + (size_t)row * p.ldo + c * 32, v);
  } else if constexpr (EPI == EPI_SILU_MUL) {
    const int n_blk = c / 4, cc = c % 4;  // output chunk -> (tile, chunk within the 128 gate columns)
    const float* g = w + n_blk * GEMM_BN + cc * 32;
    const float* u = g + GEMM_BN / 2;
    float h[32], uv[32];
    ld_f32x32(g, h);
    ld_f32x32(u, uv);
    zero_f32x32(g);
    zero_f32x32(u);
#pragma unroll
    for (int j = 0; j < 32; ++j) h[j] = silu_f(h[j] * rs) * (uv[j] * rs);
    store_bf16x32(reinterpret_cast<__nv_bfloat16*>(p.out) + (size_t)row * p.ldo + c * 32, h);
  } else if constexpr (EPI == EPI_QKV_ROPE) {
    const int per_head = p.head_dim / 32, hpos = c % per_head;
    if (hpos >= per_head / 2) return;
    const int col1 = c * 32, half = p.head_dim / 2;
    float x1[32], x2[32];
    ld_f32x32(w + col1, x1);
    ld_f32x32(w + col1 + half, x2);
    zero_f32x32(w + col1);
    zero_f32x32(w + col1 + half);
#pragma unroll
    for (int j = 0; j < 32; ++j) {
      x1[j] = x1[j] * rs + (p.bias ? p.bias[col1 + j] : 0.f);
      x2[j] = x2[j] * rs + (p.bias ? p.bias[col1 + half + j] : 0.f);
    }
    const int slot = p.slots[row];
    qkv_rope_store(p, row, col1, hpos * 32, x1, x2, slot / p.block_size, slot % p.block_size);
  }
}

PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;
std::once_flag g_encode_once;

// Scheduling decision (host).  Returns 1 for stream-K (CG=1 only).
int choose_streamk(int M, int N, int ntiles, int nk, int epi, int num_sms) {
  if (epi == EPI_ARGMAX || nk < 8) return 0;
  const int waves = (ntiles + num_sms - 1) / num_sms;
  const double eff = (double)ntiles / ((double)waves * num_sms);
  // Measured on B200: with >= one wave of tiles the reductions of partial tiles cost more than
  // the last-wave imbalance they remove, so stream-K is used only below one wave (small T).
  if (ntiles >= num_sms) return 0;
  if (epi == EPI_ADD_F32) return 1;  // partial tiles: fp32 vector reductions into the residual
  // non-additive epilogues go through the fp32 workspace (memset + reductions + finish pass)
  return (eff < 0.5 && (size_t)M * N <= GEMM_WS_ELEMS) ? 1 : 0;
}

// CTA-pair tiles need at least one wave of 256 x 256 tiles.  Measured on B200 (profiles/r01/
// ab_gemm_cg.txt): with the coalesced residual epilogue the pair kernel wins for every epilogue at
// the C1 shapes (T ~ 2090: O 0.62 -> 0.67, down 0.83 -> 0.93, gate_up 0.96 -> 1.0 of sustained
// cuBLAS bf16; QKV was already on it).
int choose_cg(int M, int N, int epi, int num_sms) {
  if (g_force_cg) return g_force_cg;
  const int nn = (N + GEMM_BN - 1) / GEMM_BN;
  const int tiles2 = ((M + 255) / 256) * nn;
  // LM head with 129-256 sampled rows (C2's ~250): one CTA-pair M tile covers every row, so each
  // CTA streams half of each weight tile once (two 1-CTA M tiles each stream all of it): C2 lm_head
  // 3.82 -> 3.51 ms over 10 steps, 0.75 -> 0.82 (profiles/r02/gemm_sched/lm_head_cg2.txt); at C1's
  // ~800 rows the two layouts measured the same
  if (epi == EPI_ARGMAX) return (M > GEMM_BM && M <= 2 * GEMM_BM) ? 2 : 1;
  if (M < 256) return 1;
  // below one wave of pair tiles the residual add takes stream-K over the pairs (hybrid_dp_tiles):
  // the 1-CTA tile streams 48 KB of operands per 64-deep k-block, more than TMA's ~60-90 B/cycle per
  // SM feeds at the MMA rate (tools/micro/tma_box.cu); the pair streams 32 KB per CTA
  if (tiles2 * 2 < num_sms && epi != EPI_ADD_F32) return 1;
  // wave quantisation of whole tiles: the pair kernel is the faster per tile, but a 128-row tile
  // grid can fill its waves much better (C2's QKV at T ~ 625: 140 tiles on 148 SMs in one wave
  // vs 84 pair tiles on 74 pairs in two; measured 49 vs 68 us)
  if (epi != EPI_ADD_F32) {
    const int tiles1 = ((M + 127) / 128) * nn, u1 = num_sms, u2 = num_sms / 2;
    const double e1 = (double)tiles1 / (double)(((tiles1 + u1 - 1) / u1) * u1);
    const double e2 = (double)tiles2 / (double)(((tiles2 + u2 - 1) / u2) * u2);
    if (e1 > e2 + 0.15) return 1;
  }
  if (epi == EPI_STORE_BF16 || epi == EPI_QKV_ROPE) return 2;
  return 2;
}

// CTA-pair hybrid (Jobs mode 2) for the residual-add epilogue: when the last wave of 256 x 256
// tiles would be less than ~80% full (e.g. C3's O / down GEMMs at T ~ 900: 80 tiles on 74 pairs),
// the tail tiles' k-blocks are spread over every pair and combined with fp32 vector reductions.
// Returns the whole-tile count (0 = no hybrid).  (Non-additive epilogues through the fp32 workspace
// measured slower than whole tiles, profiles/r01/gemm_sched.txt.)
// Returns the whole-tile count (-1 = no hybrid).  Below one wave of pair tiles that leaves more than
// 25% of the pairs idle, 0: every tile's k-blocks are spread over all pairs (stream-K over the
// CTA-pair kernel).
int hybrid_dp_tiles(int M, int N, int K, int epi, int cg, int num_sms) {
  if (cg != 2 || epi != EPI_ADD_F32 || K / GEMM_BK < 8) return -1;
  const int units = num_sms / 2;
  const int ntiles = ((M + 255) / 256) * ((N + GEMM_BN - 1) / GEMM_BN);
  // one wave at >= 75% of the pairs: whole tiles (C2's O / down at T ~ 625: 60 tiles on 74 pairs,
  // 43.0 -> 41.0 and 94.2 -> 83.9 us vs stream-K, and the fused bf16(x) / norm statistics stay on:
  // profiles/r02/gemm_sched/gemm_c2_c3_c1_default_det_cg1.jsonl); below that every tile's k-blocks go over all pairs
  if (ntiles < units) return ntiles * 100 < units * 75 ? 0 : -1;
  const int tail = ntiles % units;
  if (tail == 0 || tail * 10 >= units * 8) return -1;
  return ntiles - tail;
}

// Cluster split-K (Jobs mode 3) for small-T, few-tile GEMMs with a non-additive epilogue (C4's QKV at
// T ~ 128): one M tile, tiles x S <= SMs with S = the k-split per tile (2..8, at most the epilogue's
// units per tile: 8 chunks, or 4 chunk pairs for RoPE / SiLU).  It replaces stream-K's fp32 workspace
// + finish pass (C4 QKV 60 -> 50 us, profiles/r02/gemm_small_t.txt).  The residual-add epilogue keeps
// stream-K (vector reductions straight into the residual): its cluster variant measured ~15 us of
// extra fixed cost per launch (O 38 -> 51 us).  Returns S (0 = not used).
int skc_split(int M, int N, int K, int epi, int num_sms) {
  if (M > GEMM_BM || epi == EPI_ARGMAX || epi == EPI_ADD_F32) return 0;
  const int ntiles = (N + GEMM_BN - 1) / GEMM_BN, nk = K / GEMM_BK;
  const int cap = (epi == EPI_SILU_MUL || epi == EPI_QKV_ROPE) ? 4 : 8;
  int S = std::min(std::min(cap, num_sms / std::max(ntiles, 1)), nk / 4);
  return S >= 2 ? S : 0;
}

}  // namespace

bool gemm_uses_streamk(int M, int N, int K, int epi, int num_sms, bool deterministic) {
  if (M <= 0 || deterministic) return false;
  if (!g_force_cg && skc_split(M, N, K, epi, num_sms)) return false;  // whole tiles, reduced in-cluster
  const int cg = choose_cg(M, N, epi, num_sms);
  if (cg == 2) return hybrid_dp_tiles(M, N, K, epi, cg, num_sms) >= 0;
  const int ntiles = ((M + GEMM_BM - 1) / GEMM_BM) * ((N + GEMM_BN - 1) / GEMM_BN);
  return choose_streamk(M, N, ntiles, K / GEMM_BK, epi, num_sms) != 0;
}

size_t gemm_workspace_elems(int M, int N, int K, int epi, int num_sms) {
  const int ntiles = ((M + GEMM_BM - 1) / GEMM_BM) * ((N + GEMM_BN - 1) / GEMM_BN);
  if (epi == EPI_ADD_F32 || choose_cg(M, N, epi, num_sms) == 2 || (!g_force_cg && skc_split(M, N, K, epi, num_sms)) ||
      !choose_streamk(M, N, ntiles, K / GEMM_BK, epi, num_sms))
    return 0;
  return (size_t)M * N;
}

int make_tmap_bf16(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  std::call_once(g_encode_once, [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  });
  if (map == nullptr) return GLLM_OK;  // entry-point resolution only (encode_2d)
  if (!g_encode) return set_error(GLLM_ECUDA, "cuTensorMapEncodeTiled unavailable");
  if ((reinterpret_cast<uintptr_t>(base) & 15) || (cols * 2) % 16)
    return set_error(GLLM_EINVAL, "tensor map: base/stride not 16-byte aligned");
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * 2};
  cuuint32_t box[2] = {64, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
                        CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
                        CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error(GLLM_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return GLLM_OK;
}

static int encode_2d(CUtensorMap* map, CUtensorMapDataType dt, int esize, const void* base, uint64_t rows,
                     uint64_t cols, uint32_t box_cols, uint32_t box_rows, CUtensorMapSwizzle sw) {
  make_tmap_bf16(nullptr, nullptr, 0, 0, 0);  // resolves the driver entry point once
  if (!g_encode) return set_error(GLLM_ECUDA, "cuTensorMapEncodeTiled unavailable");
  if ((reinterpret_cast<uintptr_t>(base) & 15) || (cols * esize) % 16)
    return set_error(GLLM_EINVAL, "tensor map: base/stride not 16-byte aligned");
  cuuint64_t dims[2] = {cols, rows};
  cuuint64_t strides[1] = {cols * esize};
  cuuint32_t box[2] = {box_cols, box_rows};
  cuuint32_t estr[2] = {1, 1};
  CUresult r = g_encode(map, dt, 2, const_cast<void*>(base), dims, strides, box, estr, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        sw, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) return set_error(GLLM_ECUDA, "cuTensorMapEncodeTiled failed (%d)", (int)r);
  return GLLM_OK;
}

int make_tmap_weight_tiled(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols) {
  if (cols % 64) return set_error(GLLM_EINVAL, "tiled weight: cols %% 64 != 0");
  return make_tmap_bf16(map, base, ((rows + 127) / 128) * (cols / 64) * 128, 64, GEMM_B_BOX);
}

int make_tmap_res_f32(CUtensorMap* map, const float* base, uint64_t rows, uint64_t cols) {
  return encode_2d(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 4, base, rows, cols, 32, GEMM_BM, CU_TENSOR_MAP_SWIZZLE_128B);
}
int make_tmap_res_bf16(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols) {
  return encode_2d(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, base, rows, cols, 32, GEMM_BM, CU_TENSOR_MAP_SWIZZLE_64B);
}

int num_sms_of_current_device() {
  int dev = 0, n = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n > 0 ? n : 148;
}

template <int EPI, int CG>
static int launch_t(const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& tx, const CUtensorMap& txb,
                    const GemmArgs& args, cudaStream_t stream, int num_sms) {
  using C = Cfg<CG, EPI>;
  static bool attr_set = false;  // per-process; the attribute is per-function
  if (!attr_set) {
    cudaError_t e =
        cudaFuncSetAttribute(gemm_tc_kernel<EPI, CG>, cudaFuncAttributeMaxDynamicSharedMemorySize, C::SMEM_BYTES);
    if (e != cudaSuccess) return set_error(GLLM_ECUDA, "gemm smem attribute: %s", cudaGetErrorString(e));
    attr_set = true;
  }
  const int num_m = (args.M + C::TILE_M - 1) / C::TILE_M;
  const int ntiles = num_m * args.num_n_tiles;
  int grid;
  if (args.streamk == 3) {
    grid = ntiles * args.split_s;
  } else if (args.streamk == 1) {
    const int total = ntiles * (args.K / GEMM_BK);
    grid = (total + args.units_per_cta - 1) / args.units_per_cta;
  } else if (args.streamk == 2) {
    grid = (num_sms / CG) * CG;
  } else {
    // whole tiles, persistent: as few units as keep the wave count (C4's gate_up at T = 128: 224
    // tiles -> 112 CTAs x 2 instead of 148 CTAs of which 76 take a second tile alone at the per-SM
    // TMA rate); a wave-quantised makespan is the same either way when the tiles are tensor-bound
    const int units = num_sms / CG, waves = (ntiles + units - 1) / units;
    grid = ((ntiles + waves - 1) / waves) * CG;
  }
  if (grid <= 0) return GLLM_OK;
  {
    const int cluster = args.streamk == 3 ? args.split_s : CG;
    cudaError_t e =
        launch_pdl(gemm_tc_kernel<EPI, CG>, dim3(grid), dim3(256), C::SMEM_BYTES, stream, cluster, a, b, tx, txb, args);
    if (e != cudaSuccess) return set_error(GLLM_ECUDA, "gemm (%d-CTA) launch: %s", CG, cudaGetErrorString(e));
  }
  if (args.ws) {
    const int chunks = args.M * ((EPI == EPI_SILU_MUL) ? args.N / 64 : args.N / 32);
    launch_pdl(gemm_finish_kernel<EPI>, dim3((chunks + 255) / 256), dim3(256), 0, stream, 1, args);
  }
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_error(GLLM_ECUDA, "gemm launch: %s", cudaGetErrorString(e));
  return GLLM_OK;
}

template <int EPI>
static int launch_e(const CUtensorMap& a, const CUtensorMap& b, const CUtensorMap& tx, const CUtensorMap& txb,
                    const GemmArgs& args, cudaStream_t stream, int num_sms, int cg) {
  return cg == 2 ? launch_t<EPI, 2>(a, b, tx, txb, args, stream, num_sms)
                 : launch_t<EPI, 1>(a, b, tx, txb, args, stream, num_sms);
}

int launch_gemm(const CUtensorMap& a, const CUtensorMap& b, GemmEpi epi, const GemmArgs& args0, cudaStream_t stream,
                int num_sms, const CUtensorMap* tm_x, const CUtensorMap* tm_xb) {
  if (args0.K % GEMM_BK != 0 || args0.M < 0 || args0.N <= 0 || args0.N % 32)
    return set_error(GLLM_EINVAL, "gemm: K %% 64 != 0 or bad M/N (M=%d N=%d K=%d)", args0.M, args0.N, args0.K);
  if (args0.M == 0) return GLLM_OK;
  GemmArgs args = args0;
  const int cg = choose_cg(args.M, args.N, epi, num_sms);
  args.num_m_tiles = (args.M + GEMM_BM - 1) / GEMM_BM;
  args.num_n_tiles = (args.N + GEMM_BN - 1) / GEMM_BN;
  const int ntiles = args.num_m_tiles * args.num_n_tiles, nk = args.K / GEMM_BK;
  args.streamk = (cg == 1 && !args.deterministic) ? choose_streamk(args.M, args.N, ntiles, nk, epi, num_sms) : 0;
  args.units_per_cta = args.streamk ? (ntiles * nk + num_sms - 1) / num_sms : 0;
  args.dp_tiles = 0;
  args.split_s = 0;
  if (cg == 1 && !g_force_cg) {
    const int S = skc_split(args.M, args.N, args.K, epi, num_sms);
    if (S > 0) {  // cluster split-K replaces stream-K: no workspace, no atomics, no finish pass
      args.streamk = 3;
      args.split_s = S;
      args.units_per_cta = S;
    }
  }
  bool hybrid = false;
  if (cg == 2 && !args.deterministic && !args.xb_out && !args.ss_out && !args.out_peer) {  // partial tiles: no fused outputs
    const int dp = hybrid_dp_tiles(args.M, args.N, args.K, epi, cg, num_sms);
    if (dp >= 0) {
      const int ntiles2 = ((args.M + 255) / 256) * args.num_n_tiles, units = num_sms / 2;
      args.streamk = 2;
      args.dp_tiles = dp;
      args.units_per_cta = ((ntiles2 - dp) * nk + units - 1) / units;
      hybrid = true;
    }
  }
  if (args.streamk && args.streamk != 3 && epi != EPI_ADD_F32) {
    if (!args0.ws) return set_error(GLLM_EINVAL, "gemm: stream-K workspace required");
  } else {
    args.ws = nullptr;
  }
  static const CUtensorMap none{};  // the epilogue maps of the other kernels (never dereferenced)
  args.res_tma = 0;
  if (epi == EPI_ADD_F32 && cg == 2) {  // the CTA-pair residual kernel stages x through TMA
    if (tm_x == nullptr || (args.xb_out != nullptr && tm_xb == nullptr))
      return set_error(GLLM_EINVAL, "gemm: residual add needs the x (and bf16 x) tensor maps");
    args.res_tma = 1;
  }
  const CUtensorMap& tx = tm_x ? *tm_x : none;
  const CUtensorMap& txb = tm_xb ? *tm_xb : none;
  switch (epi) {
    case EPI_STORE_BF16: return launch_e<EPI_STORE_BF16>(a, b, tx, txb, args, stream, num_sms, cg);
    case EPI_ADD_F32: return launch_e<EPI_ADD_F32>(a, b, tx, txb, args, stream, num_sms, cg);
    case EPI_SILU_MUL: return launch_e<EPI_SILU_MUL>(a, b, tx, txb, args, stream, num_sms, cg);
    case EPI_ARGMAX: return launch_e<EPI_ARGMAX>(a, b, tx, txb, args, stream, num_sms, cg);
    case EPI_QKV_ROPE: return launch_e<EPI_QKV_ROPE>(a, b, tx, txb, args, stream, num_sms, cg);
  }
  return set_error(GLLM_EINVAL, "gemm: unknown epilogue");
}

}  // namespace gllm

#ifdef GLLM_VARIANT_TRACE
// measurement build only: arm (a device buffer of GM_TR words per CTA) or disarm (nullptr) the GEMM trace
extern "C" GLLM_API int gllm_gemm_trace_arm(void* dev_buf) {
  unsigned long long* p = static_cast<unsigned long long*>(dev_buf);
  cudaMemcpyToSymbol(gllm::g_gm_trace, &p, sizeof(p));
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
#endif
