// int_peak.cu — measured integer-ALU peak of this B200 ("Integer peak: not in
// MEASURED_PEAKS.json, so measure it with an in-repo microbenchmark (independent IADD3/IMNMX/LOP3
// streams, clocks logged)"). Not part of the product path: tools/int_peak.py and bench.py load it
// to get the denominator of the ALU roofline.
//
// Variant 0 ("alu"): every thread runs NCH independent dependency chains of IADD3 -> LOP3 -> VIMNMX
// (the ALU pipe: rt_SMSP = 2, i.e. 16 lanes/clk per SM sub-partition). Variant 1 ("alu+fma"): the
// same ALU chains interleaved 1:1 with independent IMAD chains (the FMA pipe, another 16 lanes/clk),
// which is the issue bound of 32 thread-instructions/clk per sub-partition. Variant 2 ("isetp"):
// IADD3 -> ISETP + SEL chains (compare-heavy, like the search kernels' threshold tests).
//
// Inline PTX keeps one source instruction per SASS instruction; tools/int_peak.py checks that with
// cuobjdump (the op count per loop trip is read from the SASS, not assumed). The chains are seeded
// from the thread index and stored at the end, so nothing folds.
#include <cstdint>
#include <cuda_runtime.h>

#define NCH 8

__global__ void __launch_bounds__(256) k_int_alu(uint32_t *out, int iters, uint32_t b, uint32_t c, uint32_t d) {
  uint32_t a[NCH];
#pragma unroll
  for (int j = 0; j < NCH; ++j) a[j] = threadIdx.x * (j + 3) + blockIdx.x;
#pragma unroll 1
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
#pragma unroll
      for (int j = 0; j < NCH; ++j) {
        asm volatile("add.u32 %0, %0, %1;" : "+r"(a[j]) : "r"(b));
        asm volatile("xor.b32 %0, %0, %1;" : "+r"(a[j]) : "r"(c));
        asm volatile("min.u32 %0, %0, %1;" : "+r"(a[j]) : "r"(d));
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < NCH; ++j) s ^= a[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void __launch_bounds__(256) k_int_mix(uint32_t *out, int iters, uint32_t b, uint32_t c, uint32_t d) {
  uint32_t a[NCH], m[NCH];
#pragma unroll
  for (int j = 0; j < NCH; ++j) {
    a[j] = threadIdx.x * (j + 3) + blockIdx.x;
    m[j] = threadIdx.x * (j + 5) + 7;
  }
#pragma unroll 1
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
#pragma unroll
      for (int j = 0; j < NCH; ++j) {
        asm volatile("add.u32 %0, %0, %1;" : "+r"(a[j]) : "r"(b));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(m[j]) : "r"(c), "r"(d));
        asm volatile("xor.b32 %0, %0, %1;" : "+r"(a[j]) : "r"(c));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(m[j]) : "r"(d), "r"(b));
        asm volatile("min.u32 %0, %0, %1;" : "+r"(a[j]) : "r"(d));
        asm volatile("mad.lo.u32 %0, %0, %1, %2;" : "+r"(m[j]) : "r"(b), "r"(c));
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < NCH; ++j) s ^= a[j] ^ m[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

__global__ void __launch_bounds__(256) k_int_cmp(uint32_t *out, int iters, uint32_t b, uint32_t c, uint32_t d) {
  uint32_t a[NCH];
#pragma unroll
  for (int j = 0; j < NCH; ++j) a[j] = threadIdx.x * (j + 3) + blockIdx.x;
#pragma unroll 1
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int k = 0; k < 4; ++k) {
#pragma unroll
      for (int j = 0; j < NCH; ++j) {
        asm volatile("add.u32 %0, %0, %1;" : "+r"(a[j]) : "r"(b));
        asm volatile("{ .reg .pred p; setp.lt.u32 p, %0, %1; selp.u32 %0, %0, %2, p; }"
                     : "+r"(a[j]) : "r"(c), "r"(d));
      }
    }
  }
  uint32_t s = 0;
#pragma unroll
  for (int j = 0; j < NCH; ++j) s ^= a[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}

// Source-level integer ops per thread and loop trip (tools/int_peak.py cross-checks with the SASS).
extern "C" int int_peak_ops_per_trip(int variant) {
  return variant == 0 ? 4 * NCH * 3 : variant == 1 ? 4 * NCH * 6 : 4 * NCH * 3;
}

// Runs one variant on `blocks` 256-thread blocks for `iters` loop trips; returns the kernel time in
// ms (CUDA events on the default stream) or a negative value on error.
extern "C" float int_peak_run(int variant, int blocks, int iters) {
  uint32_t *out = nullptr;
  if (cudaMalloc(&out, (size_t)blocks * 256 * sizeof(uint32_t)) != cudaSuccess) return -1.f;
  cudaEvent_t e0, e1;
  cudaEventCreate(&e0);
  cudaEventCreate(&e1);
  auto launch = [&](int it) {
    if (variant == 0) k_int_alu<<<blocks, 256>>>(out, it, 0x9e3779b9u, 0x85ebca6bu, 0xfffffff0u);
    else if (variant == 1) k_int_mix<<<blocks, 256>>>(out, it, 0x9e3779b9u, 0x85ebca6bu, 0xfffffff0u);
    else k_int_cmp<<<blocks, 256>>>(out, it, 0x9e3779b9u, 0x85ebca6bu, 0x12345u);
  };
  launch(16);  // warm-up
  cudaEventRecord(e0);
  launch(iters);
  cudaEventRecord(e1);
  cudaEventSynchronize(e1);
  float ms = -1.f;
  if (cudaGetLastError() == cudaSuccess) cudaEventElapsedTime(&ms, e0, e1);
  cudaEventDestroy(e0);
  cudaEventDestroy(e1);
  cudaFree(out);
  return ms;
}
