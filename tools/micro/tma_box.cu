// TMA issue cost vs box size, from L2-resident data: every CTA (one per SM) streams K tiles of
// 128 rows x 128 bf16 (32 KB) as 16-row boxes (16 per tile, the paged-KV prefill pattern) or as
// 128-row boxes (2 per tile), 2-stage ring.  Measurement tool, not product code.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/tma_box tools/micro/tma_box.cu
#include <cuda.h>
#include <cudaTypedefs.h>
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

__global__ void kern(const __grid_constant__ CUtensorMap tm16, const __grid_constant__ CUtensorMap tm128, int rows_total,
                     int big, int iters, long long* cyc, const uint8_t* gbase) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[4];
  if (threadIdx.x == 0) {
    for (int s = 0; s < 4; ++s) asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  if (threadIdx.x != 0) return;
  const int TILE = 32768, NS = 4;
  const long long t0 = clock64();
  auto issue = [&](int i) {
    const int s = i % NS;
    const uint32_t b = smem_u32(&bar[s]);
    asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(b), "r"(TILE));
    const int row0 = ((blockIdx.x * 131 + i * 7) % (rows_total / 128)) * 128;
    for (int at = 0; at < 2; ++at) {
      if (big == 2) {  // 1-D bulk copies of 2 KB (one per 16-row page piece)
        for (int p = 0; p < 8; ++p)
          asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], 2048, [%2];" ::"r"(
                           smem_u32(sm + s * TILE + at * 16384 + p * 2048)),
                       "l"(gbase + ((size_t)(row0 + 16 * p) * 128 + at * 64) * 2), "r"(b) : "memory");
      } else if (big == 3) {  // 1-D bulk copies of 4 KB (a whole page, both 64-column atoms)
        if (at == 0)
          for (int p = 0; p < 8; ++p)
            asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], 4096, [%2];" ::"r"(
                             smem_u32(sm + s * TILE + p * 4096)),
                         "l"(gbase + (size_t)(row0 + 16 * p) * 256), "r"(b) : "memory");
      } else if (big) {
        asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
                         smem_u32(sm + s * TILE + at * 16384)), "l"(&tm128), "r"(b), "r"(at * 64), "r"(row0) : "memory");
      } else {
        for (int p = 0; p < 8; ++p)
          asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1, {%3, %4}], [%2];" ::"r"(
                           smem_u32(sm + s * TILE + at * 16384 + p * 2048)), "l"(&tm16), "r"(b), "r"(at * 64), "r"(row0 + 16 * p) : "memory");
      }
    }
  };
  for (int i = 0; i < NS; ++i) issue(i);
  for (int i = 0; i < iters; ++i) {
    const int s = i % NS;
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared.b64 p, [%0], %1;\n@!p bra W;\n}\n" ::"r"(smem_u32(&bar[s])), "r"((i / NS) & 1));
    if (i + NS < iters) issue(i + NS);
  }
  cyc[blockIdx.x] = clock64() - t0;
}

int main() {
  PFN_cuTensorMapEncodeTiled_v12000 enc;
  cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", (void**)&enc, cudaEnableDefault, &q);
  const int rows = 65536, cols = 128;  // 16 MB: L2 resident
  void* buf;
  cudaMalloc(&buf, (size_t)rows * cols * 2);
  cudaMemset(buf, 0, (size_t)rows * cols * 2);
  CUtensorMap m16, m128;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows}, str[1] = {(cuuint64_t)cols * 2};
  cuuint32_t b16[2] = {64, 16}, b128[2] = {64, 128}, es[2] = {1, 1};
  enc(&m16, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, b16, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  enc(&m128, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, b128, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B,
      CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  long long* cyc;
  cudaMalloc(&cyc, 1024 * 8);
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 4 * 32768);
  const int iters = 400;
  for (int big = 0; big < 4; ++big)
    for (int ctas : {1, 74, 148}) {
      kern<<<ctas, 32, 4 * 32768>>>(m16, m128, rows, big, iters, cyc, (const uint8_t*)buf);
      cudaEvent_t a, b;
      cudaEventCreate(&a);
      cudaEventCreate(&b);
      cudaEventRecord(a);
      kern<<<ctas, 32, 4 * 32768>>>(m16, m128, rows, big, iters, cyc, (const uint8_t*)buf);
      cudaEventRecord(b);
      cudaEventSynchronize(b);
      float ms;
      cudaEventElapsedTime(&ms, a, b);
      long long h[1024];
      cudaMemcpy(h, cyc, ctas * 8, cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < ctas; ++i) avg += h[i];
      avg /= ctas;
      printf("{\"box_rows\": %d, \"ctas\": %d, \"cycles_per_32KB_tile\": %.0f, \"B_per_cycle_per_SM\": %.1f, \"GBps_total\": %.0f}\n",
             big == 0 ? 16 : big == 1 ? 128 : big == 2 ? -2048 : -4096, ctas, avg / iters, 32768.0 * iters / avg, 32768.0 * iters * ctas / (ms * 1e-3) / 1e9);
    }
  printf("# %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
