// tcgen05.mma issue/execute rate per SM for the shapes the kernels use (operands stay in SMEM /
// TMEM, no loads): SS M=128 N=128 / N=256 K-major (the prefill S MMA / the GEMM), TS (A from
// TMEM) M=128 N=128 with an MN-major B (the prefill PV MMA).  Cycles per instruction (K = 16).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/umma_rate tools/micro/umma_rate.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_k(uint32_t addr) {  // K-major SW128
  uint64_t d = 0;
  d |= (uint64_t)((addr & 0x3FFFFu) >> 4);
  d |= (uint64_t)1 << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
__device__ __forceinline__ uint64_t desc_mn(uint32_t addr, uint32_t lbo) {
  uint64_t d = 0;
  d |= (uint64_t)((addr & 0x3FFFFu) >> 4);
  d |= (uint64_t)((lbo >> 4) & 0x3FFFu) << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
__host__ __device__ constexpr uint32_t idesc(int M, int N, bool bmn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((bmn ? 1u : 0u) << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}

__global__ void kern(int mode, int iters, long long* out) {
  extern __shared__ __align__(1024) uint8_t sm[];
  __shared__ uint32_t tslot;
  __shared__ __align__(8) uint64_t bar;
  const int warp = threadIdx.x >> 5;
  if (warp == 0) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], 512;" ::"r"(smem_u32(&tslot)));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared.b64 [%0], 1;" ::"r"(smem_u32(&bar)));
    asm volatile("fence.mbarrier_init.release.cluster;");
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  asm volatile("tcgen05.fence::after_thread_sync;");
  const uint32_t tmem = tslot;
  if (threadIdx.x == 0) {
    const uint32_t a = smem_u32(sm), b = smem_u32(sm + 65536);
    const long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
      const uint32_t acc = i > 0;
      if (mode == 0) {  // SS, M=128 N=128
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(
                         tmem), "l"(desc_k(a + (i & 3) * 32)), "l"(desc_k(b + (i & 3) * 32)), "r"(idesc(128, 128, false)), "r"(acc));
      } else if (mode == 1) {  // SS, M=128 N=256
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(
                         tmem), "l"(desc_k(a + (i & 3) * 32)), "l"(desc_k(b + (i & 3) * 32)), "r"(idesc(128, 256, false)), "r"(acc));
      } else if (mode == 2) {  // TS (A from TMEM cols 256..), B MN-major N=128
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(
                         tmem), "r"(tmem + 256 + (i & 7) * 8), "l"(desc_mn(b + (i & 7) * 2048, 16384)), "r"(idesc(128, 128, true)), "r"(acc));
      } else {  // SS, M=128 N=64
        asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(
                         tmem), "l"(desc_k(a + (i & 3) * 32)), "l"(desc_k(b + (i & 3) * 32)), "r"(idesc(128, 64, false)), "r"(acc));
      }
    }
    asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(smem_u32(&bar)));
    asm volatile("{\n.reg .pred p;\nW: mbarrier.try_wait.parity.shared.b64 p, [%0], 0;\n@!p bra W;\n}\n" ::"r"(smem_u32(&bar)));
    out[blockIdx.x] = clock64() - t0;
  }
  asm volatile("tcgen05.fence::before_thread_sync;");
  __syncthreads();
  if (warp == 0) asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, 512;" ::"r"(tmem));
}

int main() {
  long long* out;
  cudaMalloc(&out, 1024 * 8);
  cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072);
  const char* names[] = {"SS M128 N128 K16 (prefill S)", "SS M128 N256 K16 (GEMM 1-CTA)", "TS M128 N128 K16, B MN-major (prefill PV)", "SS M128 N64 K16"};
  const int iters = 4096;
  for (int mode = 0; mode < 4; ++mode)
    for (int ctas : {1, 148}) {
      kern<<<ctas, 128, 131072>>>(mode, iters, out);
      kern<<<ctas, 128, 131072>>>(mode, iters, out);
      cudaDeviceSynchronize();
      long long h[148];
      cudaMemcpy(h, out, ctas * 8, cudaMemcpyDeviceToHost);
      double avg = 0;
      for (int i = 0; i < ctas; ++i) avg += h[i];
      avg /= ctas;
      printf("{\"mma\": \"%s\", \"ctas\": %d, \"cycles_per_instr\": %.1f}\n", names[mode], ctas, avg / iters);
    }
  printf("# %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
