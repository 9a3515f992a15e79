// wf_long32.cu -- translation unit of the FP32 long-row wavefront kernel
// (k_wavefront<float, true>: rows of >= WF_RESCALE_COLS columns, the ring rescale of
// DESIGN.md §4.5). Built with ptxas -O3: unlike the other wavefront kernels, which are
// faster at -O1 (wf.cu), this one is 2.5 % faster at -O2/-O3 (C4 kernel 8.79 vs 9.01 ms,
// profiles/r02_ab_ptxas_opt.txt). wf.cu reaches it only through these
// functions, so that no other translation unit instantiates it.
#define PHMM_DEFINE_WF
#include "wavefront.cuh"

namespace phmm {

cudaError_t wf_long32_set_max_smem(int smem_optin) {
  return cudaFuncSetAttribute(reinterpret_cast<const void*>(k_wavefront<float, true>),
                              cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
}

cudaError_t wf_long32_occupancy(int warps, size_t smem, int* blocks_per_sm) {
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(
      blocks_per_sm, reinterpret_cast<const void*>(k_wavefront<float, true>), warps * 32, smem);
}

cudaError_t wf_long32_launch(unsigned grid, int warps, size_t smem, cudaStream_t stream, const WfArgs2<float>& args) {
  k_wavefront<float, true><<<grid, warps * 32, smem, stream>>>(args);
  return cudaGetLastError();
}

}  // namespace phmm
