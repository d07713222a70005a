// tcgen05.mma rate per SM for the shapes the kernels use (operands resident in SMEM / TMEM, no loads),
// issued like the kernels do: one thread, unrolled groups of 8 K=16 steps with precomputed descriptors.
//   CHAINS independent accumulators are interleaved (1 = a dependent accumulation chain).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o tools/micro/umma_rate tools/micro/umma_rate.cu
#include <cuda_runtime.h>
#include <cstdint>
#include <cstdio>

__device__ __forceinline__ uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ uint64_t desc_k(uint32_t addr) {  // K-major SW128
  return (uint64_t)((addr & 0x3FFFFu) >> 4) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) |
         ((uint64_t)2 << 61);
}
__device__ __forceinline__ uint64_t desc_mn(uint32_t addr, uint32_t lbo) {  // MN-major SW128 (V)
  return (uint64_t)((addr & 0x3FFFFu) >> 4) | ((uint64_t)((lbo >> 4) & 0x3FFFu) << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__host__ __device__ constexpr uint32_t idesc(int M, int N, bool bmn) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((bmn ? 1u : 0u) << 16) | ((uint32_t)(N >> 3) << 17) | ((uint32_t)(M >> 4) << 24);
}
__device__ __forceinline__ void mma_ss(uint32_t d, uint64_t a, uint64_t b, uint32_t id, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n}\n" ::"r"(d),
               "l"(a), "l"(b), "r"(id), "r"(acc));
}
__device__ __forceinline__ void mma_ts(uint32_t d, uint32_t a_tmem, uint64_t b, uint32_t id, uint32_t acc) {
  asm volatile("{\n.reg .pred p;\nsetp.ne.b32 p, %4, 0;\ntcgen05.mma.cta_group::1.kind::f16 [%0], [%1], %2, %3, p;\n}\n" ::"r"(d),
               "r"(a_tmem), "l"(b), "r"(id), "r"(acc));
}

template <int N, int CHAINS, bool TS>
__global__ void kern(int groups, long long* out) {
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
    const uint64_t a0 = desc_k(smem_u32(sm)), b0 = desc_k(smem_u32(sm + 65536));
    constexpr uint32_t id = idesc(128, N, TS);
    const long long t0 = clock64();
    for (int g = 0; g < groups; ++g) {
#pragma unroll
      for (int k = 0; k < 8; ++k)
#pragma unroll
        for (int c = 0; c < CHAINS; ++c) {
          const uint32_t d = tmem + c * (N <= 128 ? 128 : 256) % 512;
          if (TS)
            mma_ts(d, tmem + 384 + k * 8, desc_mn(smem_u32(sm + 65536), 16384) + (uint64_t)(k * 128), id, (g | k) ? 1u : 0u);
          else
            mma_ss(d, a0 + (uint64_t)((k & 3) * 2 + (k >> 2) * 1024), b0 + (uint64_t)((k & 3) * 2 + (k >> 2) * 1024), id,
                   (g | k) ? 1u : 0u);
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

// the prefill kernel's per-key-tile MMA sequence with operands resident, no barriers: PV_A (TS, A = P
// aliasing S_A), S_A (SS into S_A), PV_B, S_B.  P_X aliases the first 64 columns of S_X.
__global__ void seq_kern(int iters, int alias, long long* out) {
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
    const uint64_t q = desc_k(smem_u32(sm)), k = desc_k(smem_u32(sm + 65536)), v = desc_mn(smem_u32(sm + 65536), 16384);
    constexpr uint32_t ids = idesc(128, 128, false), ido = idesc(128, 128, true);
    const long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
#pragma unroll
      for (int x = 0; x < 2; ++x) {
        // PV_x: O_x (cols 256 + 128x) += P_x (cols 128x.. or, without aliasing, a separate region) . V
        const uint32_t pa = alias ? tmem + x * 128 : tmem + 448 + x * 32;
#pragma unroll
        for (int kk = 0; kk < 8; ++kk) mma_ts(tmem + 256 + x * 128, pa + kk * (alias ? 8 : 4), v + (uint64_t)(kk * 128), ido, 1u);
#pragma unroll
        for (int ks = 0; ks < 8; ++ks)
          mma_ss(tmem + x * 128, q + (uint64_t)((ks & 3) * 2 + (ks >> 2) * 1024), k + (uint64_t)((ks & 3) * 2 + (ks >> 2) * 1024), ids,
                 ks > 0);
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

void run_seq(int alias) {
  long long* out;
  cudaMalloc(&out, 1024 * 8);
  cudaFuncSetAttribute(seq_kern, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072);
  const int iters = 256;
  seq_kern<<<148, 128, 131072>>>(iters, alias, out);
  seq_kern<<<148, 128, 131072>>>(iters, alias, out);
  cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, out, 148 * 8, cudaMemcpyDeviceToHost);
  double avg = 0;
  for (int i = 0; i < 148; ++i) avg += h[i];
  avg /= 148;
  printf("{\"sequence\": \"PV_A S_A PV_B S_B per key tile, P %s S\", \"cycles_per_key_tile\": %.0f, \"floor\": 2048}\n",
         alias ? "aliasing" : "apart from", avg / iters);
}

template <int N, int CHAINS, bool TS>
void run(const char* name) {
  long long* out;
  cudaMalloc(&out, 1024 * 8);
  cudaFuncSetAttribute(kern<N, CHAINS, TS>, cudaFuncAttributeMaxDynamicSharedMemorySize, 131072);
  const int groups = 512;
  kern<N, CHAINS, TS><<<148, 128, 131072>>>(groups, out);
  kern<N, CHAINS, TS><<<148, 128, 131072>>>(groups, out);
  cudaDeviceSynchronize();
  long long h[148];
  cudaMemcpy(h, out, 148 * 8, cudaMemcpyDeviceToHost);
  double avg = 0;
  for (int i = 0; i < 148; ++i) avg += h[i];
  avg /= 148;
  const double instr = (double)groups * 8 * CHAINS;
  const double floor = 128.0 * N / 256.0;
  printf("{\"mma\": \"%s\", \"cycles_per_instr\": %.1f, \"floor\": %.0f, \"frac_of_floor\": %.2f}\n", name, avg / instr, floor,
         floor / (avg / instr));
  cudaFree(out);
}

int main() {
  run<128, 1, false>("SS M128 N128, 1 chain (prefill S)");
  run<128, 2, false>("SS M128 N128, 2 chains");
  run<256, 1, false>("SS M128 N256, 1 chain (GEMM 1-CTA)");
  run<256, 2, false>("SS M128 N256, 2 chains");
  run<64, 1, false>("SS M128 N64, 1 chain");
  run<128, 1, true>("TS M128 N128 (prefill PV), 1 chain");
  run<128, 2, true>("TS M128 N128, 2 chains");
  run_seq(1);
  run_seq(0);
  printf("# %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
}
