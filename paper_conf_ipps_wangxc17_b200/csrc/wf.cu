// wf.cu -- translation unit of the FP32 short-row wavefront kernel k_wavefront<float, false>
// (the FP32 pass). Built with -Xptxas -O1 (9 % faster than -O2/-O3 for this kernel; DESIGN.md
// §4.7); the FP32 long-row kernel lives in wf_long32.cu and the FP64 kernels in wf_f64.cu
// (both -O3, with 3-group iterations), everything else in libphmm is built at -O3.
#define PHMM_DEFINE_WF
#include "wavefront.cuh"

namespace phmm {

// the FP32 long-row kernel (wf_long32.cu)
cudaError_t wf_long32_set_max_smem(int smem_optin);
cudaError_t wf_long32_occupancy(int warps, size_t smem, int* blocks_per_sm);
cudaError_t wf_long32_launch(unsigned grid, int warps, size_t smem, cudaStream_t stream, const WfArgs2<float>& args);
// the FP64 kernels (wf_f64.cu)
cudaError_t wf_f64_set_max_smem(int smem_optin);

// Allow every wavefront kernel the device's opt-in maximum of dynamic shared memory once
// (phmm_create), so that launches and occupancy queries need no per-call attribute change.
cudaError_t wf_set_max_smem(int smem_optin) {
  cudaError_t e = cudaFuncSetAttribute(reinterpret_cast<const void*>(k_wavefront<float, false>),
                                       cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
  if (e != cudaSuccess) return e;
  e = wf_f64_set_max_smem(smem_optin);
  if (e != cudaSuccess) return e;
  return wf_long32_set_max_smem(smem_optin);
}

template <>
cudaError_t wf_occupancy<float>(bool long_rows, int warps, size_t smem, int* blocks_per_sm) {
  if (long_rows) return wf_long32_occupancy(warps, smem, blocks_per_sm);
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(
      blocks_per_sm, reinterpret_cast<const void*>(k_wavefront<float, false>), warps * 32, smem);
}

template <>
cudaError_t wf_launch<float>(bool long_rows, unsigned grid, int warps, size_t smem, cudaStream_t stream,
                             const WfArgs2<float>& args) {
  if (long_rows) return wf_long32_launch(grid, warps, smem, stream, args);
  k_wavefront<float, false><<<grid, warps * 32, smem, stream>>>(args);
  return cudaGetLastError();
}

}  // namespace phmm
