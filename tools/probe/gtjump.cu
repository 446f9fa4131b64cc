// %globaltimer continuity probe: one thread reads %globaltimer and clock64 back to back for
// `secs` seconds and records every step of the timer larger than 10 us, with the clock64
// cycles elapsed over the same step (a real stall shows cycles ~ 1.965 GHz x step; a timer
// jump shows a large step over few cycles).
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__global__ void k(uint64_t secs, unsigned long long* out, int cap) {
  uint64_t t0 = gt(), prev = t0;
  long long c_prev = clock64();
  int n = 0;
  while (prev - t0 < secs * 1000000000ull) {
    const uint64_t t = gt();
    const long long c = clock64();
    if (t - prev > 10000ull && n < cap) {
      out[2 * n] = t - prev;
      out[2 * n + 1] = (unsigned long long)(c - c_prev);
      out[2 * cap + n] = prev - t0;
      ++n;
    }
    prev = t;
    c_prev = c;
  }
  out[3 * cap] = n;
}
int main(int argc, char** argv) {
  const int cap = 64;
  const uint64_t secs = argc > 1 ? atoi(argv[1]) : 8;
  unsigned long long* d;
  cudaMalloc(&d, (3 * cap + 1) * 8);
  cudaMemset(d, 0, (3 * cap + 1) * 8);
  k<<<1, 1>>>(secs, d, cap);
  unsigned long long h[3 * 64 + 1];
  cudaMemcpy(h, d, sizeof h, cudaMemcpyDeviceToHost);
  printf("%llu steps > 10 us in %llu s\n", h[3 * cap], (unsigned long long)secs);
  for (unsigned long long i = 0; i < h[3 * cap] && i < (unsigned long long)cap; ++i)
    printf("at %.6f s: timer step %llu ns over %llu cycles\n", h[2 * cap + i] * 1e-9, h[2 * i], h[2 * i + 1]);
  return 0;
}
