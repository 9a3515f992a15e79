// wf.cu -- translation unit of the wavefront kernels (k_wavefront<float>, <double>).
// Built with -Xptxas -O1 (see wavefront.cuh / DESIGN.md §4.6); everything else in
// libphmm is built at -O3.
#define PHMM_DEFINE_WF
#include "wavefront.cuh"

namespace phmm {

template <typename T>
cudaError_t wf_occupancy(int warps, size_t smem, int* blocks_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(k_wavefront<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_wavefront<T>, warps * 32, smem);
}

template <typename T>
cudaError_t wf_launch(unsigned grid, int warps, size_t smem, cudaStream_t stream, const WfArgs2<T>& args) {
  cudaError_t e = cudaFuncSetAttribute(k_wavefront<T>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  k_wavefront<T><<<grid, warps * 32, smem, stream>>>(args);
  return cudaGetLastError();
}

template cudaError_t wf_occupancy<float>(int, size_t, int*);
template cudaError_t wf_occupancy<double>(int, size_t, int*);
template cudaError_t wf_launch<float>(unsigned, int, size_t, cudaStream_t, const WfArgs2<float>&);
template cudaError_t wf_launch<double>(unsigned, int, size_t, cudaStream_t, const WfArgs2<double>&);

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
