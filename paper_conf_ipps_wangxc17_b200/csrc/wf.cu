// wf.cu -- translation unit of the wavefront kernels (k_wavefront<float>, <double>).
// Built with -Xptxas -O1 (see wavefront.cuh / DESIGN.md §4.7); everything else in
// libphmm is built at -O3.
#define PHMM_DEFINE_WF
#include "wavefront.cuh"

namespace phmm {

template <typename T>
static void* wf_kernel(bool long_rows) {
  return long_rows ? reinterpret_cast<void*>(k_wavefront<T, true>) : reinterpret_cast<void*>(k_wavefront<T, false>);
}

// Allow every wavefront kernel the device's opt-in maximum of dynamic shared memory once
// (phmm_create), so that launches and occupancy queries need no per-call attribute change.
cudaError_t wf_set_max_smem(int smem_optin) {
  const void* fs[4] = {reinterpret_cast<const void*>(k_wavefront<float, false>),
                       reinterpret_cast<const void*>(k_wavefront<float, true>),
                       reinterpret_cast<const void*>(k_wavefront<double, false>),
                       reinterpret_cast<const void*>(k_wavefront<double, true>)};
  for (const void* f : fs) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

template <typename T>
cudaError_t wf_occupancy(bool long_rows, int warps, size_t smem, int* blocks_per_sm) {
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, wf_kernel<T>(long_rows), warps * 32, smem);
}

template <typename T>
cudaError_t wf_launch(bool long_rows, unsigned grid, int warps, size_t smem, cudaStream_t stream,
                      const WfArgs2<T>& args) {
  if (long_rows) k_wavefront<T, true><<<grid, warps * 32, smem, stream>>>(args);
  else k_wavefront<T, false><<<grid, warps * 32, smem, stream>>>(args);
  return cudaGetLastError();
}

template cudaError_t wf_occupancy<float>(bool, int, size_t, int*);
template cudaError_t wf_occupancy<double>(bool, int, size_t, int*);
template cudaError_t wf_launch<float>(bool, unsigned, int, size_t, cudaStream_t, const WfArgs2<float>&);
template cudaError_t wf_launch<double>(bool, unsigned, int, size_t, cudaStream_t, const WfArgs2<double>&);

}  // namespace phmm

#ifdef PHMM_DBG_TRACE
// debug builds only (not declared in include/phmm.h)
extern "C" int phmm_debug_trace(float* host, int max_steps) {
  int steps = 0;
  cudaMemcpyFromSymbol(&steps, phmm::g_trace_steps, sizeof(int));
  if (steps > max_steps) steps = max_steps;
  cudaMemcpyFromSymbol(host, phmm::g_trace, sizeof(float) * (size_t)steps * 32 * 6);
  return steps;
}
#endif
