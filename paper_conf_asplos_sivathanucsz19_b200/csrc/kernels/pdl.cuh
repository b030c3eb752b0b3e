// Programmatic dependent launch (PDL) for the kernels of the serial recurrent chains: a kernel
// launched with programmatic stream serialization may be scheduled while its predecessor is still
// running; it runs its prologue (barrier init, TMEM allocation, tensor-map prefetch), then waits in
// griddepcontrol.wait until the predecessor grid has completed and its writes are visible.  Every
// kernel launched this way calls pdl_wait() before its first global-memory access that could
// depend on (or race with) earlier kernels, and pdl_trigger() only after that wait, so when a
// kernel starts, everything two launches back is complete.  ASTRA_PDL=0 disables it (A/B runs).
#pragma once
#include <cuda_runtime.h>
#include <cstdlib>
#include <utility>

#include "../common.h"

namespace astra {

__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ __forceinline__ void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

inline bool pdl_enabled() {
  static const bool on = [] {
    const char* e = std::getenv("ASTRA_PDL");
    return !(e && e[0] == '0');
  }();
  return on;
}

// cudaLaunchKernelEx with the PDL attribute (plus an optional cluster dimension).
template <typename... KArgs, typename... Args>
void launch_pdl(void (*kern)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st, int cluster_x,
                Args&&... args) {
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = st;
  cudaLaunchAttribute attr[2];
  int n = 0;
  if (pdl_enabled()) {
    attr[n].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    attr[n].val.programmaticStreamSerializationAllowed = 1;
    ++n;
  }
  if (cluster_x > 1) {
    attr[n].id = cudaLaunchAttributeClusterDimension;
    attr[n].val.clusterDim.x = cluster_x;
    attr[n].val.clusterDim.y = 1;
    attr[n].val.clusterDim.z = 1;
    ++n;
  }
  cfg.attrs = attr;
  cfg.numAttrs = n;
  CUDA_TRY(cudaLaunchKernelEx(&cfg, kern, std::forward<Args>(args)...));
}

}  // namespace astra
