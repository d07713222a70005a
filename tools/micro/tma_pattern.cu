// HBM read bandwidth of the GEMM weight-streaming access pattern: TMA 2-D boxes of 128 rows x 64
// bf16 (128 B per row, rows 2*K bytes apart: each box touches 128 DRAM rows) vs. the same bytes as
// contiguous 1-D bulk copies (a pre-tiled weight layout).  Measurement tool, not product code.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/tma_pattern tools/micro/tma_pattern.cu -lcuda
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void bar_wait(uint64_t* b, uint32_t par) {
  asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared.b64 p, [%0], %1;\n@!p bra W;\n}\n" ::"r"(smem_u32(b)), "r"(par));
}

// mode 0: 2-D tensor boxes (3 per stage: like A 128x64 + B 2 x 128x64 of the GEMM, all from the
// weight matrix here); mode 1: one 48 KB contiguous bulk copy per stage
template <int STAGES>
__global__ void kern(const __grid_constant__ CUtensorMap tm, const uint8_t* base, int mode, int n_tiles, int nk,
                     int ksplit, float* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[STAGES];
  // CTA b: tile (b / ksplit), k range part (b % ksplit)
  const int tile = blockIdx.x / ksplit, part = blockIdx.x % ksplit;
  const int kb0 = part * nk / ksplit, kb1 = (part + 1) * nk / ksplit;
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  const int STAGE = 49152;
  auto issue = [&](int i) {
    const int s = i % STAGES, kb = kb0 + i;
    uint8_t* dst = sm + s * STAGE;
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])), "r"(STAGE));
    if (mode == 0) {
      for (int q = 0; q < 3; ++q) {
        const int row = tile * 384 + q * 128;
        asm volatile(
            "cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
                smem_u32(dst + q * 16384)),
            "l"(&tm), "r"(smem_u32(&bar[s])), "r"(kb * 64), "r"(row)
            : "memory");
      }
    } else {
      const uint8_t* src = base + ((size_t)tile * nk + kb) * STAGE;
      asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       smem_u32(dst)),
                   "l"(src), "r"(STAGE), "r"(smem_u32(&bar[s]))
                   : "memory");
    }
  };
  const int n = kb1 - kb0;
  for (int i = 0; i < STAGES && i < n; ++i) issue(i);
  float acc = 0.f;
  for (int i = 0; i < n; ++i) {
    bar_wait(&bar[i % STAGES], (i / STAGES) & 1);
    acc += *reinterpret_cast<const float*>(sm + (i % STAGES) * STAGE);
    if (i + STAGES < n) issue(i + STAGES);
  }
  sink[blockIdx.x] = acc;
}

// mode 2: 3-D boxes {64, rows, KP k-blocks} (KP x 128 B contiguous per weight row per request), 96 KB
// stages, 2 in flight (the same bytes in flight as 4 x 48 KB); tile = 768 / KP rows
template <int KP>
__global__ void kern_kp(const __grid_constant__ CUtensorMap tm, int n_tiles, int nk, int ksplit, float* sink) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[2];
  constexpr int ROWS = 768 / KP, STAGE = 98304, BOXR = ROWS > 256 ? ROWS / 2 : ROWS;
  const int tile = blockIdx.x / ksplit, part = blockIdx.x % ksplit;
  const int nkp = nk / KP;
  const int kp0 = part * nkp / ksplit, kp1 = (part + 1) * nkp / ksplit;
  if (threadIdx.x == 0) {
    for (int s = 0; s < 2; ++s) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  auto issue = [&](int i) {
    const int s = i % 2, kb = (kp0 + i) * KP;
    uint8_t* dst = sm + s * STAGE;
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])), "r"(STAGE));
    for (int q = 0; q < ROWS / BOXR; ++q)
      asm volatile(
          "cp.async.bulk.tensor.3d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4, %5}], [%2];" ::"r"(
              smem_u32(dst + q * BOXR * KP * 128)),
          "l"(&tm), "r"(smem_u32(&bar[s])), "r"(0), "r"(tile * ROWS + q * BOXR), "r"(kb)
          : "memory");
  };
  const int n = kp1 - kp0;
  for (int i = 0; i < 2 && i < n; ++i) issue(i);
  float acc = 0.f;
  for (int i = 0; i < n; ++i) {
    bar_wait(&bar[i % 2], (i / 2) & 1);
    acc += *reinterpret_cast<const float*>(sm + (i % 2) * STAGE);
    if (i + 2 < n) issue(i + 2);
  }
  sink[blockIdx.x] = acc;
}

int main() {
  PFN_cuTensorMapEncodeTiled_v12000 enc;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  struct Shape { int N, K; const char* name; } shapes[] = {{10240, 8192, "C4 qkv"}, {8192, 8192, "C4 o"}, {8192, 28672, "C4 down"}, {57344, 8192, "C4 gate_up"}};
  float* sink;
  cudaMalloc(&sink, 1 << 20);
  constexpr int ST = 4;
  cudaFuncSetAttribute(kern<ST>, cudaFuncAttributeMaxDynamicSharedMemorySize, ST * 49152);
  for (auto sh : shapes) {
    const size_t bytes = (size_t)sh.N * sh.K * 2;
    uint8_t* w;
    cudaMalloc(&w, bytes);
    cudaMemset(w, 1, bytes);
    CUtensorMap tm;
    cuuint64_t dims[2] = {(cuuint64_t)sh.K, (cuuint64_t)sh.N};
    cuuint64_t str[1] = {(cuuint64_t)sh.K * 2};
    cuuint32_t box[2] = {64, 128}, es[2] = {1, 1};
    enc(&tm, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, w, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    const int n_tiles = sh.N / 384, nk = sh.K / 64;  // 384-row "tiles" = 48 KB per k-block
    for (int mode = 0; mode < 2; ++mode) {
      for (int ks : {1, 2, 3, 4}) {
        const int grid = n_tiles * ks;
        if (grid > 296) continue;
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        kern<ST><<<grid, 32, ST * 49152>>>(tm, w, mode, n_tiles, nk, ks, sink);
        cudaEventRecord(a);
        const int R = 5;
        for (int r = 0; r < R; ++r) kern<ST><<<grid, 32, ST * 49152>>>(tm, w, mode, n_tiles, nk, ks, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        const double moved = (double)n_tiles * 384 * sh.K * 2;
        printf("{\"shape\": \"%s\", \"mode\": \"%s\", \"ksplit\": %d, \"ctas\": %d, \"us\": %.1f, \"GBps\": %.0f}\n", sh.name,
               mode ? "bulk1d" : "tma2d", ks, grid, ms * 1e3 / R, moved * R / (ms * 1e-3) / 1e9);
      }
    }
    for (int KP : {2, 4}) {
      CUtensorMap t3;
      const int ROWS = 768 / KP, BOXR = ROWS > 256 ? ROWS / 2 : ROWS;
      cuuint64_t d3[3] = {64, (cuuint64_t)sh.N, (cuuint64_t)sh.K / 64};
      cuuint64_t s3[2] = {(cuuint64_t)sh.K * 2, 128};
      cuuint32_t b3[3] = {64, (cuuint32_t)BOXR, (cuuint32_t)KP}, e3[3] = {1, 1, 1};
      CUresult rr = enc(&t3, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 3, w, d3, s3, b3, e3, CU_TENSOR_MAP_INTERLEAVE_NONE,
                        CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      if (rr != CUDA_SUCCESS) { printf("# 3d map failed %d\n", (int)rr); continue; }
      auto kfn = KP == 2 ? kern_kp<2> : kern_kp<4>;
      cudaFuncSetAttribute(kfn, cudaFuncAttributeMaxDynamicSharedMemorySize, 2 * 98304);
      const int n_tiles = sh.N / ROWS, nk = sh.K / 64;
      for (int ks : {1, 2, 3, 4}) {
        const int grid = n_tiles * ks;
        if (grid > 296) continue;
        cudaEvent_t a, b;
        cudaEventCreate(&a);
        cudaEventCreate(&b);
        kfn<<<grid, 32, 2 * 98304>>>(t3, n_tiles, nk, ks, sink);
        cudaEventRecord(a);
        const int R = 5;
        for (int r = 0; r < R; ++r) kfn<<<grid, 32, 2 * 98304>>>(t3, n_tiles, nk, ks, sink);
        cudaEventRecord(b);
        cudaEventSynchronize(b);
        float ms;
        cudaEventElapsedTime(&ms, a, b);
        const double moved = (double)n_tiles * ROWS * sh.K * 2;
        printf("{\"shape\": \"%s\", \"mode\": \"tma3d_kp%d\", \"ksplit\": %d, \"ctas\": %d, \"us\": %.1f, \"GBps\": %.0f}\n",
               sh.name, KP, ks, grid, ms * 1e3 / R, moved * R / (ms * 1e-3) / 1e9);
      }
    }
    cudaFree(w);
  }
  printf("# %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
