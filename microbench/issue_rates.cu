// Issue-rate / pipe-throughput microbenchmarks on sm_100a.
//
// Purpose: measure the per-SM throughput of the instruction classes the PairHMM
// wavefront kernel is built from, so the roofline denominators and the kernel
// layout (scalar FFMA vs packed FFMA2, prior select on ALU vs smem lookup,
// SHFL cost) rest on measurements instead of assumptions.
//
// The paper's own microbenchmarks (Listing 1, PAPER.md L14@19, §II-B) measure
// LATENCY of dependent chains (a *= a; a *= shfl(a)); this file measures
// THROUGHPUT with many independent chains, which is what bounds a batched,
// fully occupied B200. A latency mode (1 warp, 1 dependent chain) is included
// for the Eq. 1-4 style comparison.
//
// Each thread runs ITER iterations of an unrolled body with NCH independent
// chains; thread 0 of each block records clock64() around the loop (after a
// __syncthreads), so ops/clk/SM = (threads/block * ITER * ops_per_iter) / cycles.
// One block per SM, 1024 threads (32 warps) unless stated.
//
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o issue_rates issue_rates.cu
#include <cstdio>
#include <cstdlib>
#include <cstdint>
#include <cuda_runtime.h>

#define CK(x) do { cudaError_t e = (x); if (e != cudaSuccess) { \
  fprintf(stderr, "CUDA %s at %s:%d\n", cudaGetErrorString(e), __FILE__, __LINE__); exit(1);} } while (0)

constexpr int ITER = 4096;

struct Out { unsigned long long cyc; float sink; };

// --- scalar FFMA, 3 register operands, 8 independent chains -----------------
__global__ void k_ffma_rrr(const float* in, Out* out) {
  float b = in[0], c = in[1];
  float a0 = in[2] + threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3,
        a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
    asm volatile("fma.rn.f32 %0, %0, %8, %9;\n\t"
                 "fma.rn.f32 %1, %1, %8, %9;\n\t"
                 "fma.rn.f32 %2, %2, %8, %9;\n\t"
                 "fma.rn.f32 %3, %3, %8, %9;\n\t"
                 "fma.rn.f32 %4, %4, %8, %9;\n\t"
                 "fma.rn.f32 %5, %5, %8, %9;\n\t"
                 "fma.rn.f32 %6, %6, %8, %9;\n\t"
                 "fma.rn.f32 %7, %7, %8, %9;\n\t"
                 : "+f"(a0), "+f"(a1), "+f"(a2), "+f"(a3), "+f"(a4), "+f"(a5), "+f"(a6), "+f"(a7)
                 : "f"(b), "f"(c));
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  if (a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 == 1234.5f) out[blockIdx.x].sink = a0;
}

// --- scalar FFMA with distinct register multiplicands (no operand reuse) ----
__global__ void k_ffma_rrr_distinct(const float* in, Out* out) {
  float b0 = in[0], b1 = in[1], b2 = in[3], b3 = in[4];
  float a0 = in[2] + threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3,
        a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
    asm volatile("fma.rn.f32 %0, %0, %8, %9;\n\t"
                 "fma.rn.f32 %1, %1, %10, %11;\n\t"
                 "fma.rn.f32 %2, %2, %9, %8;\n\t"
                 "fma.rn.f32 %3, %3, %11, %10;\n\t"
                 "fma.rn.f32 %4, %4, %8, %10;\n\t"
                 "fma.rn.f32 %5, %5, %9, %11;\n\t"
                 "fma.rn.f32 %6, %6, %10, %8;\n\t"
                 "fma.rn.f32 %7, %7, %11, %9;\n\t"
                 : "+f"(a0), "+f"(a1), "+f"(a2), "+f"(a3), "+f"(a4), "+f"(a5), "+f"(a6), "+f"(a7)
                 : "f"(b0), "f"(b1), "f"(b2), "f"(b3));
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  if (a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 == 1234.5f) out[blockIdx.x].sink = a0;
}

// --- scalar FFMA with an immediate operand ----------------------------------
__global__ void k_ffma_imm(const float* in, Out* out) {
  float b = in[0];
  float a0 = in[2] + threadIdx.x, a1 = a0 + 1, a2 = a0 + 2, a3 = a0 + 3,
        a4 = a0 + 4, a5 = a0 + 5, a6 = a0 + 6, a7 = a0 + 7;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
    asm volatile("fma.rn.f32 %0, %0, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %1, %1, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %2, %2, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %3, %3, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %4, %4, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %5, %5, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %6, %6, %8, 0f3F000000;\n\t"
                 "fma.rn.f32 %7, %7, %8, 0f3F000000;\n\t"
                 : "+f"(a0), "+f"(a1), "+f"(a2), "+f"(a3), "+f"(a4), "+f"(a5), "+f"(a6), "+f"(a7)
                 : "f"(b));
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  if (a0 + a1 + a2 + a3 + a4 + a5 + a6 + a7 == 1234.5f) out[blockIdx.x].sink = a0;
}

// --- packed FFMA2 / FMUL2 / FADD2, 8 independent chains ----------------------
#define PK(x) (*reinterpret_cast<unsigned long long*>(&(x)))
template <int OP>  // 0 = fma.f32x2, 1 = mul.f32x2, 2 = add.f32x2
__global__ void k_x2(const float* in, Out* out) {
  float2 b = make_float2(in[0], in[3]), c = make_float2(in[1], in[4]);
  float2 a[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = make_float2(in[2] + threadIdx.x + j, in[2] - j);
  unsigned long long B = PK(b), C = PK(c);
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      if (OP == 0) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(PK(a[j])) : "l"(B), "l"(C));
      if (OP == 1) asm volatile("mul.rn.f32x2 %0, %0, %1;" : "+l"(PK(a[j])) : "l"(B));
      if (OP == 2) asm volatile("add.rn.f32x2 %0, %0, %1;" : "+l"(PK(a[j])) : "l"(C));
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  float s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += a[j].x + a[j].y;
  if (s == 1234.5f) out[blockIdx.x].sink = s;
}

// --- the wavefront cell's FP mix: 2 FFMA2 : 1 scalar FMUL, 8 independent chains ---
__global__ void k_x2_fmul(const float* in, Out* out) {
  float2 b = make_float2(in[0], in[3]), c = make_float2(in[1], in[4]);
  float2 a[8];
  float f[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) { a[j] = make_float2(in[2] + threadIdx.x + j, in[2] - j); f[j] = in[0] + j; }
  unsigned long long B = PK(b), C = PK(c);
  const float g = in[3];
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(PK(a[j])) : "l"(B), "l"(C));
      if (j & 1) asm volatile("mul.rn.f32 %0, %0, %1;" : "+f"(f[j]) : "f"(g));
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  float s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += a[j].x + a[j].y + f[j];
  if (s == 1234.5f) out[blockIdx.x].sink = s;
}

// --- FFMA2 interleaved 1:1 with an ALU op (LOP3 / FSEL via predicate / PRMT) --
template <int ALU>  // 0 = lop3, 1 = fsel (setp+selp), 2 = prmt, 3 = mov-free iadd3
__global__ void k_x2_alu(const float* in, Out* out) {
  float2 b = make_float2(in[0], in[3]), c = make_float2(in[1], in[4]);
  float2 a[8];
  unsigned u[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) {
    a[j] = make_float2(in[2] + threadIdx.x + j, in[2] - j);
    u[j] = __float_as_uint(in[5]) + threadIdx.x * 7 + j;
  }
  unsigned long long B = PK(b), C = PK(c);
  unsigned m1 = __float_as_uint(in[6]), m2 = __float_as_uint(in[7]);
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(PK(a[j])) : "l"(B), "l"(C));
      if (ALU == 0) asm volatile("lop3.b32 %0, %0, %1, %2, 0x6a;" : "+r"(u[j]) : "r"(m1), "r"(m2));
      if (ALU == 1) asm volatile("{.reg .pred p; setp.ne.b32 p, %0, %1; selp.b32 %0, %1, %2, p;}" : "+r"(u[j]) : "r"(m1), "r"(m2));
      if (ALU == 2) asm volatile("prmt.b32 %0, %0, %1, %2;" : "+r"(u[j]) : "r"(m1), "r"(m2));
      if (ALU == 3) asm volatile("add.u32 %0, %0, %1;" : "+r"(u[j]) : "r"(m1));
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  float s = 0; unsigned su = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) { s += a[j].x + a[j].y; su ^= u[j]; }
  if (s == 1234.5f || su == 0x12345u) out[blockIdx.x].sink = s + su;
}

// --- ALU-only (LOP3), to get the ALU pipe rate -------------------------------
__global__ void k_lop3(const float* in, Out* out) {
  unsigned u[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) u[j] = __float_as_uint(in[5]) + threadIdx.x * 7 + j;
  unsigned m1 = __float_as_uint(in[6]), m2 = __float_as_uint(in[7]);
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) asm volatile("lop3.b32 %0, %0, %1, %2, 0x6a;" : "+r"(u[j]) : "r"(m1), "r"(m2));
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  unsigned su = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) su ^= u[j];
  if (su == 0x12345u) out[blockIdx.x].sink = su;
}

// --- scalar FFMA interleaved 1:1 with LOP3 (dual pipe co-issue check) -------
__global__ void k_ffma_lop3(const float* in, Out* out) {
  float b = in[0], c = in[1];
  float a[8]; unsigned u[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) { a[j] = in[2] + threadIdx.x + j; u[j] = __float_as_uint(in[5]) + threadIdx.x * 7 + j; }
  unsigned m1 = __float_as_uint(in[6]), m2 = __float_as_uint(in[7]);
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a[j]) : "f"(b), "f"(c));
      asm volatile("lop3.b32 %0, %0, %1, %2, 0x6a;" : "+r"(u[j]) : "r"(m1), "r"(m2));
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  float s = 0; unsigned su = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) { s += a[j]; su ^= u[j]; }
  if (s == 1234.5f || su == 0x12345u) out[blockIdx.x].sink = s + su;
}

// --- SHFL throughput (idx, rotate by one), optionally mixed with FFMA2 ------
template <int WITH_X2>
__global__ void k_shfl(const float* in, Out* out) {
  float v[8];
  float2 a[8];
  float2 b = make_float2(in[0], in[3]), c = make_float2(in[1], in[4]);
#pragma unroll
  for (int j = 0; j < 8; ++j) { v[j] = in[2] + threadIdx.x + j; a[j] = make_float2(v[j], -v[j]); }
  unsigned long long B = PK(b), C = PK(c);
  int src = (threadIdx.x - 1) & 31;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      v[j] = __shfl_sync(0xffffffffu, v[j], src);
      if (WITH_X2) {
#pragma unroll
        for (int r = 0; r < WITH_X2; ++r)
          asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(PK(a[j])) : "l"(B), "l"(C));
      }
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  float s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += v[j] + a[j].x;
  if (s == 1234.5f) out[blockIdx.x].sink = s;
}

// --- LDS.128 throughput (conflict-free), optionally mixed with FFMA2 ---------
template <int WITH_X2>
__global__ void k_lds128(const float* in, Out* out) {
  __shared__ float4 sm[2048];
  for (int i = threadIdx.x; i < 2048; i += blockDim.x) sm[i] = make_float4(in[0] + i, 1, 2, 3);
  float2 b = make_float2(in[0], in[3]), c = make_float2(in[1], in[4]);
  float2 a[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = make_float2(in[2] + threadIdx.x + j, in[2] - j);
  unsigned long long B = PK(b), C = PK(c);
  float4 acc = make_float4(0, 0, 0, 0);
  unsigned idx = threadIdx.x & 31;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 4
  for (int i = 0; i < ITER; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      float4 x = sm[(idx + j * 32 + (i & 7) * 256) & 2047];
      acc.x += x.x; acc.z += x.z; acc.y = __int_as_float(__float_as_int(acc.y) ^ __float_as_int(x.y)); acc.w = __int_as_float(__float_as_int(acc.w) ^ __float_as_int(x.w));
      if (WITH_X2) {
#pragma unroll
        for (int r = 0; r < WITH_X2; ++r)
          asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(PK(a[j])) : "l"(B), "l"(C));
      }
    }
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  float s = acc.x + acc.y + acc.z + acc.w;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += a[j].x;
  if (s == 1234.5f) out[blockIdx.x].sink = s;
}

// --- DFMA throughput ---------------------------------------------------------
__global__ void k_dfma(const float* in, Out* out) {
  double b = in[0], c = in[1];
  double a[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = in[2] + threadIdx.x + j;
  __syncthreads();
  unsigned long long t0 = clock64();
#pragma unroll 2
  for (int i = 0; i < ITER / 8; ++i) {
#pragma unroll
    for (int j = 0; j < 8; ++j) asm volatile("fma.rn.f64 %0, %0, %1, %2;" : "+d"(a[j]) : "d"(b), "d"(c));
  }
  __syncthreads();
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) out[blockIdx.x].cyc = t1 - t0;
  double s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += a[j];
  if (s == 1234.5) out[blockIdx.x].sink = (float)s;
}

// --- latency mode: one warp, one dependent chain (paper Listing 1 style) -----
__global__ void k_lat_ffma(const float* in, Out* out) {
  float a = in[2], b = in[0], c = in[1];
  unsigned long long t0 = clock64();
  for (int i = 0; i < ITER; ++i) asm volatile("fma.rn.f32 %0, %0, %1, %2;" : "+f"(a) : "f"(b), "f"(c));
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) { out[blockIdx.x].cyc = t1 - t0; out[blockIdx.x].sink = a; }
}
__global__ void k_lat_ffma2(const float* in, Out* out) {
  float2 a = make_float2(in[2], in[3]), b = make_float2(in[0], in[3]), c = make_float2(in[1], in[4]);
  unsigned long long B = PK(b), C = PK(c);
  unsigned long long t0 = clock64();
  for (int i = 0; i < ITER; ++i) asm volatile("fma.rn.f32x2 %0, %0, %1, %2;" : "+l"(PK(a)) : "l"(B), "l"(C));
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) { out[blockIdx.x].cyc = t1 - t0; out[blockIdx.x].sink = a.x; }
}
__global__ void k_lat_shfl(const float* in, Out* out) {
  float a = in[2] + threadIdx.x;
  int src = (threadIdx.x - 1) & 31;
  unsigned long long t0 = clock64();
  for (int i = 0; i < ITER; ++i) a = __shfl_sync(0xffffffffu, a, src);
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) { out[blockIdx.x].cyc = t1 - t0; out[blockIdx.x].sink = a; }
}
__global__ void k_lat_lds(const float* in, Out* out) {
  __shared__ unsigned buf[32];
  if (threadIdx.x < 32) buf[threadIdx.x] = (threadIdx.x + 1) & 31;
  __syncthreads();
  unsigned p = (unsigned)in[8];
  unsigned long long t0 = clock64();
  for (int i = 0; i < ITER; ++i) p = buf[p];
  unsigned long long t1 = clock64();
  if (threadIdx.x == 0) { out[blockIdx.x].cyc = t1 - t0; out[blockIdx.x].sink = (float)p; }
}

typedef void (*kfn)(const float*, Out*);

static double run(const char* name, kfn f, int threads, int blocks, double ops_per_thread_iter,
                  double iters, const float* din, Out* dout, int nsm, const char* unit) {
  f<<<blocks, threads>>>(din, dout);  // warm (I$)
  CK(cudaGetLastError());
  CK(cudaDeviceSynchronize());
  f<<<blocks, threads>>>(din, dout);
  CK(cudaDeviceSynchronize());
  Out* h = (Out*)malloc(sizeof(Out) * blocks);
  CK(cudaMemcpy(h, dout, sizeof(Out) * blocks, cudaMemcpyDeviceToHost));
  double cyc = 0;
  for (int i = 0; i < blocks; ++i) cyc += (double)h[i].cyc;
  cyc /= blocks;
  free(h);
  double per_blk = threads * iters * ops_per_thread_iter;
  double rate = per_blk / cyc;  // per block per clock; 1 block per SM
  printf("{\"bench\": \"%s\", \"threads\": %d, \"blocks\": %d, \"cycles\": %.0f, \"per_sm_per_clk\": %.3f, \"unit\": \"%s\"}\n",
         name, threads, blocks, cyc, rate, unit);
  return rate;
}

int main() {
  int dev = 0, nsm = 0;
  CK(cudaSetDevice(dev));
  CK(cudaDeviceGetAttribute(&nsm, cudaDevAttrMultiProcessorCount, dev));
  float hin[16] = {0.999f, 1e-7f, 0.5f, 0.998f, 2e-7f, 3.0f, 1.5f, 2.5f, 0.0f};
  float* din; Out* dout;
  CK(cudaMalloc(&din, sizeof(hin)));
  CK(cudaMemcpy(din, hin, sizeof(hin), cudaMemcpyHostToDevice));
  CK(cudaMalloc(&dout, sizeof(Out) * nsm * 4));
  printf("{\"sm_count\": %d}\n", nsm);
  const int T = 1024, Bk = nsm;
  run("ffma_rrr", k_ffma_rrr, T, Bk, 8, ITER, din, dout, nsm, "fp32 lane-ops (FFMA)");
  run("ffma_rrr_distinct", k_ffma_rrr_distinct, T, Bk, 8, ITER, din, dout, nsm, "fp32 lane-ops (FFMA)");
  run("ffma_imm", k_ffma_imm, T, Bk, 8, ITER, din, dout, nsm, "fp32 lane-ops (FFMA)");
  run("ffma2", k_x2<0>, T, Bk, 16, ITER, din, dout, nsm, "fp32 lane-ops (2 per FFMA2)");
  run("ffma2_8warps", k_x2<0>, 256, Bk, 16, ITER, din, dout, nsm, "fp32 lane-ops (2 per FFMA2), 8 warps/SM");
  run("ffma2_fmul_2to1", k_x2_fmul, T, Bk, 20, ITER, din, dout, nsm, "fp32 lane-ops (8 FFMA2 + 4 FMUL)");
  run("ffma2_fmul_2to1_8warps", k_x2_fmul, 256, Bk, 20, ITER, din, dout, nsm, "fp32 lane-ops, 8 warps/SM");
  run("fmul2", k_x2<1>, T, Bk, 16, ITER, din, dout, nsm, "fp32 lane-ops (2 per FMUL2)");
  run("fadd2", k_x2<2>, T, Bk, 16, ITER, din, dout, nsm, "fp32 lane-ops (2 per FADD2)");
  run("lop3", k_lop3, T, Bk, 8, ITER, din, dout, nsm, "alu lane-ops");
  run("ffma_lop3_1to1", k_ffma_lop3, T, Bk, 16, ITER, din, dout, nsm, "warp-instr*32 (FFMA+LOP3)");
  run("ffma2_lop3_1to1", k_x2_alu<0>, T, Bk, 16, ITER, din, dout, nsm, "warp-instr*32 (FFMA2+LOP3)");
  run("ffma2_setp_selp_1to1", k_x2_alu<1>, T, Bk, 24, ITER, din, dout, nsm, "warp-instr*32 (FFMA2+SETP+SEL)");
  run("ffma2_prmt_1to1", k_x2_alu<2>, T, Bk, 16, ITER, din, dout, nsm, "warp-instr*32 (FFMA2+PRMT)");
  run("ffma2_iadd_1to1", k_x2_alu<3>, T, Bk, 16, ITER, din, dout, nsm, "warp-instr*32 (FFMA2+IADD)");
  run("shfl_idx", k_shfl<0>, T, Bk, 8, ITER, din, dout, nsm, "shfl lane-ops");
  run("shfl_idx_plus_2ffma2", k_shfl<2>, T, Bk, 24, ITER, din, dout, nsm, "warp-instr*32 (1 SHFL + 2 FFMA2)");
  run("shfl_idx_plus_4ffma2", k_shfl<4>, T, Bk, 40, ITER, din, dout, nsm, "warp-instr*32 (1 SHFL + 4 FFMA2)");
  run("lds128", k_lds128<0>, T, Bk, 8, ITER, din, dout, nsm, "LDS.128 lane-ops");
  run("lds128_plus_4ffma2", k_lds128<4>, T, Bk, 8 * 5, ITER, din, dout, nsm, "warp-instr*32 (LDS.128+2 ALU+4 FFMA2; counts 5)");
  run("dfma", k_dfma, T, Bk, 8, ITER / 8, din, dout, nsm, "fp64 lane-ops (DFMA)");
  run("lat_ffma", k_lat_ffma, 32, 1, 1.0 / 32, ITER, din, dout, nsm, "1/latency (per warp-instr)");
  run("lat_ffma2", k_lat_ffma2, 32, 1, 1.0 / 32, ITER, din, dout, nsm, "1/latency");
  run("lat_shfl", k_lat_shfl, 32, 1, 1.0 / 32, ITER, din, dout, nsm, "1/latency");
  run("lat_lds", k_lat_lds, 32, 1, 1.0 / 32, ITER, din, dout, nsm, "1/latency");
  return 0;
}
