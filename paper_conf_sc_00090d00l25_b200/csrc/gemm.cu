// Persistent warp-specialised tcgen05 GEMM for sm_100a (a5, a8, a9, a10, a11 of DESIGN.md §2).
//
//   Y[M,N] = X[M,K] . W[N,K]^T      X = activations (bf16, K-major), W = weights (bf16, K-major)
//
// Tile 128 x 256 x 64, 4-stage TMA -> SMEM ring (128-byte swizzle), one
// elected thread issues tcgen05.mma (M=128, N=256, K=16) into a double-
// buffered fp32 TMEM accumulator (2 x 256 columns), 4 epilogue warps drain
// TMEM with tcgen05.ld and apply the fused epilogue (bias, fp32 residual add,
// SiLU*up, or a row-wise argmax for the greedy LM head).  Warp roles:
//   warp 0: TMA producer      warp 1: MMA issuer      warp 2: TMEM allocator
//   warps 4-7: epilogue (warp 4+i reads TMEM lanes 32i..32i+31)
#include <cudaTypedefs.h>

#include <cstdio>
#include <mutex>

#include "common.h"
#include "gemm.cuh"
#include "ptx.cuh"

namespace gllm {

namespace {

constexpr int A_BYTES = GEMM_BM * GEMM_BK * 2;
constexpr int B_BYTES = GEMM_BN * GEMM_BK * 2;
constexpr int STAGE_BYTES = A_BYTES + B_BYTES;
constexpr int SMEM_BYTES = GEMM_STAGES * STAGE_BYTES + 1024 + 256;
constexpr int TMEM_COLS = 2 * GEMM_BN;

__device__ __forceinline__ float silu_f(float x) { return x / (1.0f + __expf(-x)); }

template <int EPI>
__global__ void __launch_bounds__(256, 1)
    gemm_tc_kernel(const __grid_constant__ CUtensorMap tma_a, const __grid_constant__ CUtensorMap tma_b,
                   const GemmArgs p) {
  extern __shared__ uint8_t smem_raw[];
  uint8_t* smem = reinterpret_cast<uint8_t*>((reinterpret_cast<uintptr_t>(smem_raw) + 1023) & ~uintptr_t(1023));
  uint8_t* sA = smem;
  uint8_t* sB = smem + GEMM_STAGES * A_BYTES;
  uint64_t* full = reinterpret_cast<uint64_t*>(sB + GEMM_STAGES * B_BYTES);
  uint64_t* empty = full + GEMM_STAGES;
  uint64_t* tfull = empty + GEMM_STAGES;
  uint64_t* tempty = tfull + 2;
  uint32_t* tmem_ptr = reinterpret_cast<uint32_t*>(tempty + 2);

  const int warp = threadIdx.x >> 5;
  const int lane = threadIdx.x & 31;
  if (warp == 0 && lane == 0) {
    ptx::tma_prefetch(&tma_a);
    ptx::tma_prefetch(&tma_b);
  }
  if (warp == 1 && lane == 0) {
    for (int s = 0; s < GEMM_STAGES; ++s) {
      ptx::mbar_init(&full[s], 1);
      ptx::mbar_init(&empty[s], 1);
    }
    for (int s = 0; s < 2; ++s) {
      ptx::mbar_init(&tfull[s], 1);
      ptx::mbar_init(&tempty[s], 4);
    }
    ptx::fence_barrier_init();
  }
  if (warp == 2) {
    ptx::tmem_alloc(tmem_ptr, TMEM_COLS);
    ptx::tmem_relinquish();
  }
  ptx::tc_fence_before();
  __syncthreads();
  ptx::tc_fence_after();
  const uint32_t tmem_base = *tmem_ptr;

  const int num_m = p.num_m_tiles;
  const int ntiles = num_m * p.num_n_tiles;
  const int nk = p.K / GEMM_BK;

  if (warp == 0) {
    if (lane == 0) {
      // ---------------- TMA producer
      int stage = 0;
      uint32_t phase = 0;
      for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int m_blk = tile % num_m, n_blk = tile / num_m;
        for (int kb = 0; kb < nk; ++kb) {
          ptx::mbar_wait(&empty[stage], phase ^ 1);
          ptx::mbar_arrive_expect_tx(&full[stage], STAGE_BYTES);
          ptx::tma_load_2d(sA + stage * A_BYTES, &tma_a, &full[stage], kb * GEMM_BK, m_blk * GEMM_BM);
          ptx::tma_load_2d(sB + stage * B_BYTES, &tma_b, &full[stage], kb * GEMM_BK, n_blk * GEMM_BN);
          if (++stage == GEMM_STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
      }
    }
  } else if (warp == 1) {
    if (lane == 0) {
      // ---------------- MMA issuer (single thread)
      constexpr uint32_t idesc = ptx::umma_idesc_bf16(GEMM_BM, GEMM_BN);
      int stage = 0;
      uint32_t phase = 0;
      int acc = 0;
      uint32_t acc_phase = 0;
      for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        ptx::mbar_wait(&tempty[acc], acc_phase ^ 1);
        ptx::tc_fence_after();
        const uint32_t d_tmem = tmem_base + acc * GEMM_BN;
        for (int kb = 0; kb < nk; ++kb) {
          ptx::mbar_wait(&full[stage], phase);
          ptx::tc_fence_after();
          const uint32_t a_addr = ptx::smem_u32(sA + stage * A_BYTES);
          const uint32_t b_addr = ptx::smem_u32(sB + stage * B_BYTES);
#pragma unroll
          for (int k = 0; k < GEMM_BK / 16; ++k) {
            ptx::umma_bf16(d_tmem, ptx::umma_desc_sw128(a_addr + k * 32), ptx::umma_desc_sw128(b_addr + k * 32),
                           idesc, (kb | k) != 0);
          }
          ptx::umma_commit(&empty[stage]);  // frees the SMEM slot once these MMAs retire
          if (++stage == GEMM_STAGES) {
            stage = 0;
            phase ^= 1;
          }
        }
        ptx::umma_commit(&tfull[acc]);  // accumulator ready for the epilogue
        acc ^= 1;
        if (acc == 0) acc_phase ^= 1;
      }
    }
  } else if (warp >= 4) {
    // ---------------- epilogue warps
    const int ew = warp - 4;
    int acc = 0;
    uint32_t acc_phase = 0;
    for (int tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
      const int m_blk = tile % num_m, n_blk = tile / num_m;
      ptx::mbar_wait(&tfull[acc], acc_phase);
      ptx::tc_fence_after();
      const int row = m_blk * GEMM_BM + ew * 32 + lane;
      const bool row_ok = row < p.M;
      const uint32_t tbase = tmem_base + ((uint32_t)(ew * 32) << 16) + acc * GEMM_BN;
      uint32_t r[32];
      if constexpr (EPI == EPI_STORE_BF16) {
        __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(p.out);
#pragma unroll 1
        for (int c = 0; c < GEMM_BN / 32; ++c) {
          ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
          ptx::tmem_ld_wait();
          const int col0 = n_blk * GEMM_BN + c * 32;
          if (row_ok && col0 < p.N) {
            float v[32];
#pragma unroll
            for (int j = 0; j < 32; ++j) v[j] = __uint_as_float(r[j]);
            if (p.bias) {
#pragma unroll
              for (int j = 0; j < 32; ++j) v[j] += __ldg(p.bias + col0 + j);
            }
            uint4* dst = reinterpret_cast<uint4*>(out + (size_t)row * p.ldo + col0);
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              uint4 w;
              w.x = ptx::pack_bf16(v[q * 8 + 0], v[q * 8 + 1]);
              w.y = ptx::pack_bf16(v[q * 8 + 2], v[q * 8 + 3]);
              w.z = ptx::pack_bf16(v[q * 8 + 4], v[q * 8 + 5]);
              w.w = ptx::pack_bf16(v[q * 8 + 6], v[q * 8 + 7]);
              dst[q] = w;
            }
          }
        }
      } else if constexpr (EPI == EPI_ADD_F32) {
        float* out = reinterpret_cast<float*>(p.out);
#pragma unroll 1
        for (int c = 0; c < GEMM_BN / 32; ++c) {
          ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
          ptx::tmem_ld_wait();
          const int col0 = n_blk * GEMM_BN + c * 32;
          if (row_ok && col0 < p.N) {
            float4* dst = reinterpret_cast<float4*>(out + (size_t)row * p.ldo + col0);
#pragma unroll
            for (int q = 0; q < 8; ++q) {
              float4 x = dst[q];
              x.x += __uint_as_float(r[q * 4 + 0]);
              x.y += __uint_as_float(r[q * 4 + 1]);
              x.z += __uint_as_float(r[q * 4 + 2]);
              x.w += __uint_as_float(r[q * 4 + 3]);
              dst[q] = x;
            }
          }
        }
      } else if constexpr (EPI == EPI_SILU_MUL) {
        __nv_bfloat16* out = reinterpret_cast<__nv_bfloat16*>(p.out);
        uint32_t u[32];
#pragma unroll 1
        for (int c = 0; c < GEMM_BN / 64; ++c) {
          ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);                  // gate columns
          ptx::tmem_ld_32x32b_x32(tbase + GEMM_BN / 2 + c * 32, u);    // up columns
          ptx::tmem_ld_wait();
          const int col0 = n_blk * (GEMM_BN / 2) + c * 32;
          if (row_ok && col0 < p.N / 2) {
            uint4* dst = reinterpret_cast<uint4*>(out + (size_t)row * p.ldo + col0);
#pragma unroll
            for (int q = 0; q < 4; ++q) {
              float h[8];
#pragma unroll
              for (int j = 0; j < 8; ++j)
                h[j] = silu_f(__uint_as_float(r[q * 8 + j])) * __uint_as_float(u[q * 8 + j]);
              uint4 w;
              w.x = ptx::pack_bf16(h[0], h[1]);
              w.y = ptx::pack_bf16(h[2], h[3]);
              w.z = ptx::pack_bf16(h[4], h[5]);
              w.w = ptx::pack_bf16(h[6], h[7]);
              dst[q] = w;
            }
          }
        }
      } else if constexpr (EPI == EPI_QKV_ROPE) {
        // The 256 columns of a tile are whole heads (D | 256); rotate-half partners (i, i + D/2)
        // are 32-column chunks c and c + D/64 of the same head.
        const int D = p.head_dim, half = D / 2, per_head = D / 32;
        const int slot = row_ok ? __ldg(p.slots + row) : 0;
        const int64_t blk = slot / p.block_size, off = slot % p.block_size;
        uint32_t u[32];
#pragma unroll 1
        for (int c = 0; c < GEMM_BN / 32; ++c) {
          const int hpos = c % per_head;  // chunk index within its head
          if (hpos >= per_head / 2) continue;
          ptx::tmem_ld_32x32b_x32(tbase + c * 32, r);
          ptx::tmem_ld_32x32b_x32(tbase + (c + per_head / 2) * 32, u);
          ptx::tmem_ld_wait();
          const int col1 = n_blk * GEMM_BN + c * 32;  // first-half column of this chunk
          if (!row_ok || col1 >= p.N) continue;
          const int col2 = col1 + half;
          const int i0 = hpos * 32;                   // rotation index of element 0
          float x1[32], x2[32];
#pragma unroll
          for (int j = 0; j < 32; ++j) {
            x1[j] = __uint_as_float(r[j]);
            x2[j] = __uint_as_float(u[j]);
          }
          if (p.bias) {
#pragma unroll
            for (int j = 0; j < 32; ++j) {
              x1[j] += __ldg(p.bias + col1 + j);
              x2[j] += __ldg(p.bias + col2 + j);
            }
          }
          __nv_bfloat16 *dst1, *dst2;
          if (col1 < p.q_dim + p.kv_dim) {  // q or k: rotate
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
            dst1 = out + col1;
            dst2 = out + col2;
          } else {
            const bool is_k = col1 < p.q_dim + p.kv_dim;
            const int cc = col1 - p.q_dim - (is_k ? 0 : p.kv_dim);
            const int h = cc / D;
            __nv_bfloat16* base = (is_k ? p.kc : p.vc) + ((blk * p.n_kv_heads + h) * p.block_size + off) * D;
            dst1 = base + i0;
            dst2 = base + i0 + half;
          }
          uint4* d1 = reinterpret_cast<uint4*>(dst1);
          uint4* d2 = reinterpret_cast<uint4*>(dst2);
#pragma unroll
          for (int q = 0; q < 4; ++q) {
            uint4 w1, w2;
            w1.x = ptx::pack_bf16(x1[q * 8 + 0], x1[q * 8 + 1]);
            w1.y = ptx::pack_bf16(x1[q * 8 + 2], x1[q * 8 + 3]);
            w1.z = ptx::pack_bf16(x1[q * 8 + 4], x1[q * 8 + 5]);
            w1.w = ptx::pack_bf16(x1[q * 8 + 6], x1[q * 8 + 7]);
            w2.x = ptx::pack_bf16(x2[q * 8 + 0], x2[q * 8 + 1]);
            w2.y = ptx::pack_bf16(x2[q * 8 + 2], x2[q * 8 + 3]);
            w2.z = ptx::pack_bf16(x2[q * 8 + 4], x2[q * 8 + 5]);
            w2.w = ptx::pack_bf16(x2[q * 8 + 6], x2[q * 8 + 7]);
            d1[q] = w1;
            d2[q] = w2;
          }
        }
      } else {  // EPI_ARGMAX
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
      ptx::tc_fence_before();
      __syncwarp();
      if (lane == 0) ptx::mbar_arrive(&tempty[acc]);
      acc ^= 1;
      if (acc == 0) acc_phase ^= 1;
    }
  }
  __syncthreads();
  if (warp == 2) {
    ptx::tc_fence_after();
    ptx::tmem_dealloc(tmem_base, TMEM_COLS);
  }
}

PFN_cuTensorMapEncodeTiled_v12000 g_encode = nullptr;
std::once_flag g_encode_once;

}  // namespace

int make_tmap_bf16(CUtensorMap* map, const void* base, uint64_t rows, uint64_t cols, uint32_t box_rows) {
  std::call_once(g_encode_once, [] {
    void* fn = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &fn, cudaEnableDefault, &q) == cudaSuccess &&
        q == cudaDriverEntryPointSuccess)
      g_encode = reinterpret_cast<PFN_cuTensorMapEncodeTiled_v12000>(fn);
  });
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

int num_sms_of_current_device() {
  int dev = 0, n = 0;
  cudaGetDevice(&dev);
  cudaDeviceGetAttribute(&n, cudaDevAttrMultiProcessorCount, dev);
  return n > 0 ? n : 148;
}

template <int EPI>
static int launch_t(const CUtensorMap& a, const CUtensorMap& b, const GemmArgs& args, cudaStream_t stream,
                    int num_sms) {
  static bool attr_set = false;  // per-process; the attribute is per-function
  if (!attr_set) {
    cudaError_t e = cudaFuncSetAttribute(gemm_tc_kernel<EPI>, cudaFuncAttributeMaxDynamicSharedMemorySize, SMEM_BYTES);
    if (e != cudaSuccess) return set_error(GLLM_ECUDA, "gemm smem attribute: %s", cudaGetErrorString(e));
    attr_set = true;
  }
  const int ntiles = args.num_m_tiles * args.num_n_tiles;
  const int grid = ntiles < num_sms ? ntiles : num_sms;
  if (grid <= 0) return GLLM_OK;
  gemm_tc_kernel<EPI><<<grid, 256, SMEM_BYTES, stream>>>(a, b, args);
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) return set_error(GLLM_ECUDA, "gemm launch: %s", cudaGetErrorString(e));
  return GLLM_OK;
}

int launch_gemm(const CUtensorMap& a, const CUtensorMap& b, GemmEpi epi, const GemmArgs& args0, cudaStream_t stream,
                int num_sms) {
  if (args0.K % GEMM_BK != 0 || args0.M < 0 || args0.N <= 0)
    return set_error(GLLM_EINVAL, "gemm: K %% 64 != 0 or bad M/N (M=%d N=%d K=%d)", args0.M, args0.N, args0.K);
  if (args0.M == 0) return GLLM_OK;
  GemmArgs args = args0;
  args.num_m_tiles = (args.M + GEMM_BM - 1) / GEMM_BM;
  args.num_n_tiles = (args.N + GEMM_BN - 1) / GEMM_BN;
  switch (epi) {
    case EPI_STORE_BF16: return launch_t<EPI_STORE_BF16>(a, b, args, stream, num_sms);
    case EPI_ADD_F32: return launch_t<EPI_ADD_F32>(a, b, args, stream, num_sms);
    case EPI_SILU_MUL: return launch_t<EPI_SILU_MUL>(a, b, args, stream, num_sms);
    case EPI_ARGMAX: return launch_t<EPI_ARGMAX>(a, b, args, stream, num_sms);
    case EPI_QKV_ROPE: return launch_t<EPI_QKV_ROPE>(a, b, args, stream, num_sms);
  }
  return set_error(GLLM_EINVAL, "gemm: unknown epilogue");
}

}  // namespace gllm
