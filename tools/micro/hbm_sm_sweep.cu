// HBM read bandwidth vs number of active SMs (one CTA per SM streaming its share of a buffer
// through a 4-stage cp.async.bulk ring into shared memory).  Measurement tool, not product code:
// tells whether a GEMM wave that leaves SMs idle still saturates HBM.
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/hbm_sm_sweep tools/micro/hbm_sm_sweep.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int CHUNK, int STAGES>
__global__ void stream_kernel(const uint8_t* __restrict__ src, size_t per_cta, float* sink) {
  extern __shared__ __align__(128) uint8_t sm[];
  __shared__ __align__(8) uint64_t bar[STAGES];
  const uint8_t* base = src + (size_t)blockIdx.x * per_cta;
  const int n = (int)(per_cta / CHUNK);
  if (threadIdx.x == 0) {
    for (int s = 0; s < STAGES; ++s)
      asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar[s])));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  __syncthreads();
  float acc = 0.f;
  if (threadIdx.x == 0) {
    auto issue = [&](int i) {
      const int s = i % STAGES;
      asm volatile("mbarrier.arrive.expect_tx.shared.b64 _, [%0], %1;" ::"r"(smem_u32(&bar[s])), "r"(CHUNK));
      asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                       smem_u32(sm + s * CHUNK)),
                   "l"(base + (size_t)i * CHUNK), "r"(CHUNK), "r"(smem_u32(&bar[s]))
                   : "memory");
    };
    for (int i = 0; i < STAGES && i < n; ++i) issue(i);
    for (int i = 0; i < n; ++i) {
      const int s = i % STAGES;
      const uint32_t par = (i / STAGES) & 1;
      asm volatile(
          "{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared.b64 p, [%0], %1;\n@!p bra W;\n}\n" ::"r"(
              smem_u32(&bar[s])),
          "r"(par));
      acc += *reinterpret_cast<const float*>(sm + s * CHUNK);
      if (i + STAGES < n) issue(i + STAGES);
    }
    sink[blockIdx.x] = acc;
  }
}

int main() {
  const size_t total = size_t(2) << 30;  // 2 GB
  uint8_t* buf;
  float* sink;
  cudaMalloc(&buf, total);
  cudaMemset(buf, 1, total);
  cudaMalloc(&sink, 4096 * 4);
  int nsm = 0;
  cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, 0);
  constexpr int CHUNK = 32768, STAGES = 6;
  cudaFuncSetAttribute(stream_kernel<CHUNK, STAGES>, cudaFuncAttributeMaxDynamicSharedMemorySize, CHUNK * STAGES);
  int counts[] = {8, 16, 32, 48, 64, 76, 96, 112, 128, 148, 296};
  for (int c : counts) {
    const size_t per = (total / c) / CHUNK * CHUNK;
    cudaEvent_t a, b;
    cudaEventCreate(&a);
    cudaEventCreate(&b);
    stream_kernel<CHUNK, STAGES><<<c, 32, CHUNK * STAGES>>>(buf, per, sink);
    cudaEventRecord(a);
    for (int r = 0; r < 3; ++r) stream_kernel<CHUNK, STAGES><<<c, 32, CHUNK * STAGES>>>(buf, per, sink);
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms;
    cudaEventElapsedTime(&ms, a, b);
    const double gbs = 3.0 * per * c / (ms * 1e-3) / 1e9;
    printf("{\"ctas\": %d, \"sms\": %d, \"GBps\": %.1f, \"per_cta_GBps\": %.1f}\n", c, nsm, gbs, gbs / c);
  }
  cudaError_t e = cudaDeviceSynchronize();
  printf("# %s\n", cudaGetErrorString(e));
  return 0;
}
