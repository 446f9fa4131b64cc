// corunner.cu — a compute-bound background kernel for the co-runner experiment (SURVEY §8(f)
// N3; processor time yielded by waiting nodes can serve other work).
// Each CTA runs `iters` dependent FMA rounds on 8 independent chains per thread; it needs no
// shared memory and few registers, so its CTAs fit beside an executor CTA on the same SM.
#include <cuda_runtime.h>
#include <stdint.h>

__global__ void __launch_bounds__(128) pl_corunner_kernel(uint64_t iters, float* sink) {
  float a[8];
#pragma unroll
  for (int j = 0; j < 8; ++j) a[j] = (float)(threadIdx.x + j);
  for (uint64_t r = 0; r < iters; ++r) {
#pragma unroll
    for (int j = 0; j < 8; ++j) a[j] = fmaf(a[j], 0.999999f, 1e-7f);
  }
  float s = 0;
#pragma unroll
  for (int j = 0; j < 8; ++j) s += a[j];
  if (threadIdx.x == 0) sink[blockIdx.x] = s;   // the result, so a co-resident run can be checked exactly
}

extern "C" int pl_corunner_launch(void* stream, uint32_t n_ctas, uint64_t iters, float* sink) {
  pl_corunner_kernel<<<n_ctas, 128, 0, (cudaStream_t)stream>>>(iters, sink);
  return cudaGetLastError() == cudaSuccess ? 0 : -3;
}
