// Programmatic dependent launch (PDL) for the per-layer kernel chain.
//
// Every hot kernel of the stage forward (prep, embed, norms, GEMMs, stream-K finish, decode and
// prefill attention, argmax) is launched with cudaLaunchAttributeProgrammaticStreamSerialization,
// so its CTAs may become resident while the previous kernel on the stream is still draining. The
// kernel then (1) triggers its own dependents at entry (griddepcontrol.launch_dependents) and
// (2) does only dependency-free setup (mbarrier init, TMEM allocation, tensor-map prefetch)
// before griddepcontrol.wait, which returns once every prerequisite grid has COMPLETED and its
// memory is visible. Every thread that touches global memory executes the wait first, so the
// ordering is the same as a plain stream; only launch latency and prologue overlap the
// predecessor's tail. On by default; GLLM_PDL=0 gives plain stream serialisation (the device-side
// instructions are then no-ops).
#pragma once
#include <cuda_runtime.h>

#include <utility>

namespace gllm {

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

bool pdl_enabled();  // GLLM_PDL (default on), read once per process

// cudaLaunchKernelEx with the PDL attribute (when enabled) and an optional cluster shape.
template <typename... KArgs, typename... Args>
inline cudaError_t launch_pdl(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t stream,
                              int cluster_x, Args&&... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[2];
  int n = 0;
  if (cluster_x > 1) {
    attr[n].id = cudaLaunchAttributeClusterDimension;
    attr[n].val.clusterDim.x = cluster_x;
    attr[n].val.clusterDim.y = 1;
    attr[n].val.clusterDim.z = 1;
    ++n;
  }
  if (pdl_enabled()) {
    attr[n].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[n].val.programmaticStreamSerializationAllowed = 1;
    ++n;
  }
  cfg.attrs = attr;
  cfg.numAttrs = n;
  return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

}  // namespace gllm
