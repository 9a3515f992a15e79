// wf_f64.cu -- translation unit of the FP64 wavefront kernels k_wavefront<double, *> (the FP64
// underflow rescue and the FP64 pass), built with ptxas -O3 and the long segment of every pass in
// 3-group iterations with the code words in fixed registers (PHMM_UNROLL3_F64): 1-3.5 % faster
// FP64 passes than at -O1 without them (C3 rescue 5.69 -> 5.57-5.59 ms, C4 1.42 -> 1.37 ms;
// profiles/r02_ab_rescue_f64.txt). wf.cu reaches them only through these functions.
#define PHMM_DEFINE_WF
#define PHMM_UNROLL3_F64 1
#include "wavefront.cuh"

namespace phmm {

cudaError_t wf_f64_set_max_smem(int smem_optin) {
  const void* fs[2] = {reinterpret_cast<const void*>(k_wavefront<double, false>),
                       reinterpret_cast<const void*>(k_wavefront<double, true>)};
  for (const void* f : fs) {
    cudaError_t e = cudaFuncSetAttribute(f, cudaFuncAttributeMaxDynamicSharedMemorySize, smem_optin);
    if (e != cudaSuccess) return e;
  }
  return cudaSuccess;
}

template <>
cudaError_t wf_occupancy<double>(bool long_rows, int warps, size_t smem, int* blocks_per_sm) {
  const void* f = long_rows ? reinterpret_cast<const void*>(k_wavefront<double, true>)
                            : reinterpret_cast<const void*>(k_wavefront<double, false>);
  return cudaOccupancyMaxActiveBlocksPerMultiprocessor(blocks_per_sm, f, warps * 32, smem);
}

template <>
cudaError_t wf_launch<double>(bool long_rows, unsigned grid, int warps, size_t smem, cudaStream_t stream,
                              const WfArgs2<double>& args) {
  if (long_rows) k_wavefront<double, true><<<grid, warps * 32, smem, stream>>>(args);
  else k_wavefront<double, false><<<grid, warps * 32, smem, stream>>>(args);
  return cudaGetLastError();
}

}  // namespace phmm
