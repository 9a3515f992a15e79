// bank_counter.cu -- what does l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st count?
//
// The striped C4 wavefront kernel runs every shared-memory instruction at its ideal
// wavefront count (ncu source page: 0 excess wavefronts), yet the aggregate l1tex bank
// conflict counters report a few thousand store "conflicts" per launch
// (profiles/r01_ncu_c4_striped_banks.txt). Two kernels with the SAME conflict-free shared
// stores (each lane one 16-byte STS.128 at a lane-contiguous address, 4 wavefronts per
// instruction), one of them also streaming global loads through L1 the way the wavefront
// kernel's switch events do. If the counter rises only with the global loads, it counts
// contention of the shared stores with L1 fills in the shared data banks, not bank
// conflicts between the lanes of an instruction.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o bank_counter bank_counter.cu
// Run:   ncu --metrics l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum,
//        l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum,smsp__inst_executed_op_shared_st.sum ./bank_counter
#include <cstdio>
#include <cuda_runtime.h>

__global__ void sts_only(int iters, float* sink) {
  __shared__ __align__(16) float4 buf[4 * 32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float4 v = make_float4(lane, 1.f, 2.f, 3.f);
  for (int i = 0; i < iters; ++i) {
    buf[w * 32 + lane] = v;  // 32 lanes x 16 B contiguous: 4 wavefronts, no conflict
    v.x += 1.f;
    __syncwarp();
  }
  if (threadIdx.x == 0) sink[blockIdx.x] = buf[lane].x;
}

__global__ void sts_with_ldg(int iters, const float4* __restrict__ g, size_t n, float* sink) {
  __shared__ __align__(16) float4 buf[4 * 32];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  float4 v = make_float4(lane, 1.f, 2.f, 3.f);
  float acc = 0.f;
  size_t k = ((size_t)blockIdx.x * blockDim.x + threadIdx.x) * 7919u;
  for (int i = 0; i < iters; ++i) {
    buf[w * 32 + lane] = v;
    const float4 x = __ldg(g + (k % n));  // global load through L1 (a miss most of the time)
    k += 104729u;
    acc += x.x;
    v.x += 1.f;
    __syncwarp();
  }
  if (threadIdx.x == 0) sink[blockIdx.x] = buf[lane].x + acc;
}

int main() {
  const size_t n = (size_t)64 << 20;  // 1 GiB of float4
  float4* g;
  float* sink;
  cudaMalloc(&g, n * sizeof(float4));
  cudaMemset(g, 0, n * sizeof(float4));
  cudaMalloc(&sink, 4096 * sizeof(float));
  sts_only<<<592, 128>>>(4096, sink);
  sts_with_ldg<<<592, 128>>>(4096, g, n, sink);
  cudaError_t e = cudaDeviceSynchronize();
  std::printf("%s\n", cudaGetErrorString(e));
  return e == cudaSuccess ? 0 : 1;
}
