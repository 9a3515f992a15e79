// wf32.cu -- translation unit of the FP32 wavefront kernel (k_wavefront_f32).
// Built with -Xptxas -O1 (see wavefront_f32.cuh / DESIGN.md §4.6); everything
// else in libphmm is built at -O3.
#define PHMM_DEFINE_WF32
#include "wavefront_f32.cuh"

namespace phmm {

cudaError_t wf32_occupancy(size_t smem, int* blocks_per_sm) {
  cudaError_t e = cudaFuncSetAttribute(k_wavefront_f32, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
  if (e != cudaSuccess) return e;
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, k_wavefront_f32, F32_WARPS * 32, smem);
}

cudaError_t wf32_launch(unsigned grid, size_t smem, cudaStream_t stream, const F32Args& args) {
  k_wavefront_f32<<<grid, F32_WARPS * 32, smem, stream>>>(args);
  return cudaGetLastError();
}

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
