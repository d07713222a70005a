// Bandwidth-bound kernels of the stage forward: O4 weight init,
// slot mapping + RoPE table (O2, a2), embedding gather (a3), RMSNorm statistics and
// the final norm (a4) and the greedy argmax reduction (a11).  RoPE + KV append (a6)
// live in the QKV GEMM epilogue.
#include <cuda_bf16.h>

#include "kernels.cuh"
#include "kvpage.cuh"
#include "launch.cuh"

#include <cstdlib>

namespace gllm {

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  x += 0x9E3779B97F4A7C15ull;
  uint64_t z = x;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// O4: x = (u - 2^23) 2^-23 exactly, then one correctly rounded fp32 multiply by the scale.
__device__ __forceinline__ float o4(uint64_t seed, uint64_t tid, uint64_t i, float scale) {
  const uint64_t u = splitmix64(seed ^ (tid << 40) ^ i) >> 40;
  const float x = (float)((int64_t)u - (int64_t)(1 << 23)) * 0x1p-23f;
  return __fmul_rn(x, scale);
}

__global__ void init_bf16_kernel(__nv_bfloat16* dst, int64_t rows, int64_t cols, uint64_t seed, uint64_t tid,
                                 float scale, int mode, int64_t row_offset, int tiled) {
  const int64_t n = rows * cols;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = i / cols, c = i - r * cols;
    int64_t pr;
    if (mode == 0)
      pr = r + row_offset;
    else
      pr = (r / 128) * 256 + (mode == 2 ? 128 : 0) + (r % 128);
    // tiled: the GEMM weight layout (gemm.cuh, weight_tiled_index): 128-row x 64-column blocks,
    // each 16 KB contiguous, so a B-operand TMA box reads one contiguous run of DRAM
    const int64_t at = tiled ? ((pr >> 7) * (cols >> 6) + (c >> 6)) * 8192 + (pr & 127) * 64 + (c & 63) : pr * cols + c;
    dst[at] = __float2bfloat16_rn(o4(seed, tid, (uint64_t)i, scale));
  }
}

__global__ void init_f32_kernel(float* dst, int64_t n, uint64_t seed, uint64_t tid, float scale) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = __bfloat162float(__float2bfloat16_rn(o4(seed, tid, (uint64_t)i, scale)));
}

__global__ void fill_f32_kernel(float* dst, int64_t n, float v) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    dst[i] = v;
}

// Warm-start KV (O4): K / V of warm request r at position p, kv head h, dim j hold
// element ((r * 2^17 + p) * Hkv + h) * D + j of tensor tid / tid + 1 (scale sqrt(3)), written through
// the sequence's block table.  One CTA per (page, sequence); pages past the context are skipped.
__global__ void fill_warm_kv_kernel(__nv_bfloat16* kc, __nv_bfloat16* vc, const int64_t* __restrict__ req_ids,
                                    const int32_t* __restrict__ ctx, const int32_t* __restrict__ bt, int maxblk,
                                    int Hkv, int D, int bs, uint64_t seed, uint64_t tid) {
  const int seq = blockIdx.y, page = blockIdx.x;
  const int n = ctx[seq];
  const int p0 = page * bs;
  if (p0 >= n) return;
  const int np = min(bs, n - p0);
  const int64_t blk = bt[(int64_t)seq * maxblk + page];
  const uint64_t base = ((uint64_t)req_ids[seq] << 17);
  const int per_pos = Hkv * D;
  for (int e = threadIdx.x; e < np * per_pos; e += blockDim.x) {
    const int o = e / per_pos, hd = e - o * per_pos, h = hd / D, j = hd - h * D;
    const uint64_t i = (base + (uint64_t)(p0 + o)) * (uint64_t)per_pos + (uint64_t)hd;
    const int64_t dst = kv_page_elem(blk * Hkv + h, o, j, D);  // SMEM-ready page layout (kvpage.cuh)
    kc[dst] = __float2bfloat16_rn(o4(seed, tid, i, 1.7320508f));
    vc[dst] = __float2bfloat16_rn(o4(seed, tid + 1, i, 1.7320508f));
  }
}

// One thread per token: slot = bt[seq][pos / bs] * bs + pos % bs, seq found by binary search in cu_q.
// Threads also fill the RoPE table cs[t][i] = (cos, sin)(pos * theta^(-2i/D)) in double precision.
__global__ void prep_kernel(const int32_t* __restrict__ positions, const int32_t* __restrict__ cu_q,
                            const int32_t* __restrict__ bt, int T, int S, int maxblk, int bs, int32_t* slots,
                            float2* cs, int half, double log2_theta) {
  pdl_trigger();
  pdl_wait();
  const int t = blockIdx.x;
  if (t >= T) return;
  const int pos = positions[t];
  if (threadIdx.x == 0) {
    int lo = 0, hi = S;  // largest seq with cu_q[seq] <= t
    while (hi - lo > 1) {
      const int mid = (lo + hi) >> 1;
      if (cu_q[mid] <= t) lo = mid; else hi = mid;
    }
    slots[t] = bt[(int64_t)lo * maxblk + pos / bs] * bs + pos % bs;
  }
  for (int i = threadIdx.x; i < half; i += blockDim.x) {
    const double inv_freq = exp2(-(2.0 * i / (2.0 * half)) * log2_theta);
    double sn, cn;
    sincos((double)pos * inv_freq, &sn, &cn);
    cs[(int64_t)t * half + i] = make_float2((float)cn, (float)sn);
  }
}

__global__ void embed_kernel(const __nv_bfloat16* __restrict__ E, const int32_t* __restrict__ ids, float* x, int H) {
  pdl_trigger();
  pdl_wait();
  const int t = blockIdx.x;
  const __nv_bfloat16* row = E + (int64_t)ids[t] * H;
  float* out = x + (int64_t)t * H;
  for (int c = threadIdx.x * 8; c < H; c += blockDim.x * 8) {
    const uint4 v = *reinterpret_cast<const uint4*>(row + c);
    const __nv_bfloat162* h = reinterpret_cast<const __nv_bfloat162*>(&v);
    float4 a, b;
    float2 f0 = __bfloat1622float2(h[0]), f1 = __bfloat1622float2(h[1]);
    float2 f2 = __bfloat1622float2(h[2]), f3 = __bfloat1622float2(h[3]);
    a = make_float4(f0.x, f0.y, f1.x, f1.y);
    b = make_float4(f2.x, f2.y, f3.x, f3.y);
    *reinterpret_cast<float4*>(out + c) = a;
    *reinterpret_cast<float4*>(out + c + 4) = b;
  }
}

template <int NT>
__device__ __forceinline__ float block_sum(float v, float* red) {
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
  const int w = threadIdx.x >> 5, l = threadIdx.x & 31;
  if (l == 0) red[w] = v;
  __syncthreads();
  float s = 0.f;
#pragma unroll
  for (int i = 0; i < NT / 32; ++i) s += red[i];
  return s;
}

// One CTA of 256 threads per row; fp32 math (a4).
__global__ void __launch_bounds__(256) rmsnorm_kernel(const float* __restrict__ x, const float* __restrict__ g,
                                                      __nv_bfloat16* y, const int32_t* __restrict__ rows, int H,
                                                      float eps) {
  __shared__ float red[8];
  pdl_trigger();
  pdl_wait();
  const int r = blockIdx.x;
  const int src = rows ? rows[r] : r;
  const float* xr = x + (int64_t)src * H;
  float ss = 0.f;
  for (int c = threadIdx.x * 4; c < H; c += 256 * 4) {
    const float4 v = *reinterpret_cast<const float4*>(xr + c);
    ss += v.x * v.x + v.y * v.y + v.z * v.z + v.w * v.w;
  }
  ss = block_sum<256>(ss, red);
  const float inv = rsqrtf(ss / (float)H + eps);
  __nv_bfloat16* yr = y + (int64_t)r * H;
  for (int c = threadIdx.x * 4; c < H; c += 256 * 4) {
    const float4 v = *reinterpret_cast<const float4*>(xr + c);
    const float4 gg = *reinterpret_cast<const float4*>(g + c);
    uint2 o;
    __nv_bfloat162 a = __floats2bfloat162_rn(v.x * inv * gg.x, v.y * inv * gg.y);
    __nv_bfloat162 b = __floats2bfloat162_rn(v.z * inv * gg.z, v.w * inv * gg.w);
    o.x = *reinterpret_cast<uint32_t*>(&a);
    o.y = *reinterpret_cast<uint32_t*>(&b);
    *reinterpret_cast<uint2*>(yr + c) = o;
  }
}

__global__ void __launch_bounds__(256) rms_stats_kernel(const float* __restrict__ x, float* x_copy,
                                                        __nv_bfloat16* xb, float* ss, int H, uint32_t* rel_flag,
                                                        uint32_t rel_val, unsigned* rel_ctr) {
  __shared__ float red[8];
  pdl_trigger();
  pdl_wait();
  const int r = blockIdx.x;
  const float* xr = x + (int64_t)r * H;
  __nv_bfloat16* yr = xb + (int64_t)r * H;
  float acc = 0.f;
  for (int c = threadIdx.x * 4; c < H; c += 256 * 4) {
    const float4 v = *reinterpret_cast<const float4*>(xr + c);
    if (x_copy) *reinterpret_cast<float4*>(x_copy + (int64_t)r * H + c) = v;  // hand-off copy-in
    acc += v.x * v.x + v.y * v.y + v.z * v.z + v.w * v.w;
    uint2 o;
    __nv_bfloat162 a = __floats2bfloat162_rn(v.x, v.y);
    __nv_bfloat162 b = __floats2bfloat162_rn(v.z, v.w);
    o.x = *reinterpret_cast<uint32_t*>(&a);
    o.y = *reinterpret_cast<uint32_t*>(&b);
    *reinterpret_cast<uint2*>(yr + c) = o;
  }
  acc = block_sum<256>(acc, red);  // (its __syncthreads also orders every thread's reads of the row)
  if (threadIdx.x == 0) {
    ss[r] = acc;
    if (rel_flag) {
      // peer-ring credit: the last CTA to finish reading the input slot hands it back to the sender
      __threadfence();
      if (atomicAdd(rel_ctr, 1u) == gridDim.x - 1) {
        *rel_ctr = 0;  // kept zero for the next release (stream order)
        __threadfence_system();
        asm volatile("st.release.sys.global.u32 [%0], %1;" ::"l"(rel_flag), "r"(rel_val) : "memory");
      }
    }
  }
}

__global__ void argmax_reduce_kernel(const float* __restrict__ pv, const int32_t* __restrict__ pi, int rows,
                                     int ntiles, int32_t* out) {
  pdl_trigger();
  pdl_wait();
  const int r = blockIdx.x * (blockDim.x / 32) + (threadIdx.x >> 5);
  const int l = threadIdx.x & 31;
  if (r >= rows) return;
  float best = -INFINITY;
  int bi = 0x7fffffff;
  for (int j = l; j < ntiles; j += 32) {
    const float v = pv[(int64_t)r * ntiles + j];
    const int i = pi[(int64_t)r * ntiles + j];
    if (v > best || (v == best && i < bi)) {
      best = v;
      bi = i;
    }
  }
#pragma unroll
  for (int o = 16; o > 0; o >>= 1) {
    const float v2 = __shfl_xor_sync(0xffffffffu, best, o);
    const int i2 = __shfl_xor_sync(0xffffffffu, bi, o);
    if (v2 > best || (v2 == best && i2 < bi)) {
      best = v2;
      bi = i2;
    }
  }
  if (l == 0) out[r] = bi;
}

int grid_for(int64_t n, int threads) {
  int64_t g = (n + threads - 1) / threads;
  return (int)(g < 148 * 32 ? (g < 1 ? 1 : g) : 148 * 32);
}

}  // namespace

bool pdl_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("GLLM_PDL");  // default on (A/B: profiles/r01/s4b)
    return e == nullptr || e[0] != '0';
  }();
  return on;
}

void launch_init_bf16(__nv_bfloat16* dst, int64_t rows, int64_t cols, uint64_t seed, uint64_t tid, float scale,
                      int mode, int64_t row_offset, cudaStream_t s, int tiled) {
  init_bf16_kernel<<<grid_for(rows * cols, 256), 256, 0, s>>>(dst, rows, cols, seed, tid, scale, mode, row_offset,
                                                               tiled);
}
void launch_init_f32(float* dst, int64_t n, uint64_t seed, uint64_t tid, float scale, cudaStream_t s) {
  init_f32_kernel<<<grid_for(n, 256), 256, 0, s>>>(dst, n, seed, tid, scale);
}
void launch_fill_f32(float* dst, int64_t n, float v, cudaStream_t s) {
  fill_f32_kernel<<<grid_for(n, 256), 256, 0, s>>>(dst, n, v);
}
void launch_fill_warm_kv(__nv_bfloat16* kc, __nv_bfloat16* vc, const int64_t* req_ids, const int32_t* ctx,
                         const int32_t* bt, int n_seqs, int maxblk, int Hkv, int D, int bs, uint64_t seed,
                         uint64_t tid, cudaStream_t s) {
  if (n_seqs == 0 || maxblk == 0) return;
  fill_warm_kv_kernel<<<dim3(maxblk, n_seqs), 256, 0, s>>>(kc, vc, req_ids, ctx, bt, maxblk, Hkv, D, bs, seed, tid);
}
void launch_prep(const int32_t* positions, const int32_t* cu_q, const int32_t* block_table, int T, int S,
                 int maxblk, int block_size, int32_t* slots, float2* rope_cs, int head_dim, float rope_theta,
                 cudaStream_t s) {
  if (T <= 0) return;
  launch_pdl(prep_kernel, dim3(T), dim3(64), 0, s, 1, positions, cu_q, block_table, T, S, maxblk, block_size, slots, rope_cs,
             head_dim / 2, log2((double)rope_theta));
}
void launch_embed(const __nv_bfloat16* E, const int32_t* ids, float* x, int T, int H, cudaStream_t s) {
  if (T <= 0) return;
  launch_pdl(embed_kernel, dim3(T), dim3(128), 0, s, 1, E, ids, x, H);
}
void launch_rmsnorm(const float* x, const float* g, __nv_bfloat16* y, const int32_t* rows, int n, int H, float eps,
                    cudaStream_t s) {
  if (n <= 0) return;
  launch_pdl(rmsnorm_kernel, dim3(n), dim3(256), 0, s, 1, x, g, y, rows, H, eps);
}
void launch_rms_stats(const float* x, float* x_copy, __nv_bfloat16* xb, float* ss, int n, int H, uint32_t* rel_flag,
                      uint32_t rel_val, unsigned* rel_ctr, cudaStream_t s) {
  if (n <= 0) return;
  launch_pdl(rms_stats_kernel, dim3(n), dim3(256), 0, s, 1, x, x_copy, xb, ss, H, rel_flag, rel_val, rel_ctr);
}
void launch_argmax_reduce(const float* part_val, const int32_t* part_idx, int rows, int ntiles, int32_t* out,
                          cudaStream_t s) {
  if (rows <= 0) return;
  launch_pdl(argmax_reduce_kernel, dim3((rows + 3) / 4), dim3(128), 0, s, 1, part_val, part_idx, rows, ntiles, out);
}

}  // namespace gllm
