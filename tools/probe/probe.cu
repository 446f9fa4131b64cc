// Hardware probe for the physical-clock design: %globaltimer resolution,
// __nanosleep accuracy, clock64 rate, cp.async.bulk from host-mapped memory.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
__device__ __forceinline__ uint64_t gtimer() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

__global__ void k_res(uint64_t* out, int n) {
  // record successive distinct globaltimer values
  uint64_t prev = gtimer(); int i = 0;
  long long c0 = clock64();
  while (i < n) { uint64_t t = gtimer(); if (t != prev) { out[i++] = t - prev; prev = t; } }
  long long c1 = clock64();
  out[n] = (uint64_t)(c1 - c0);
}
__global__ void k_rate(uint64_t* out) {
  uint64_t g0 = gtimer(); long long c0 = clock64();
  while (gtimer() - g0 < 2000000ull) {}
  uint64_t g1 = gtimer(); long long c1 = clock64();
  out[0] = g1 - g0; out[1] = c1 - c0;
}
__global__ void k_sleep(uint64_t* out, unsigned ns) {
  for (int r = 0; r < 16; ++r) { uint64_t a = gtimer(); __nanosleep(ns); uint64_t b = gtimer(); out[r] = b - a; }
}
__global__ void k_bulk(const uint32_t* src, uint32_t* dst, int bytes) {
  __shared__ alignas(128) uint32_t buf[1024];
  __shared__ alignas(8) uint64_t bar;
  if (threadIdx.x == 0) {
    uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"(b));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(b), "r"(bytes));
    uint32_t d = (uint32_t)__cvta_generic_to_shared(buf);
    asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                 :: "r"(d), "l"(src), "r"(bytes), "r"(b) : "memory");
    uint32_t ok = 0;
    while (!ok) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], 0; selp.u32 %0,1,0,p; }" : "=r"(ok) : "r"(b));
  }
  __syncthreads();
  for (int i = threadIdx.x; i < bytes / 4; i += blockDim.x) dst[i] = buf[i];
}
int main() {
  cudaDeviceProp p; cudaGetDeviceProperties(&p, 0);
  printf("dev %s sms %d clock %d kHz smemOptin %zu l2 %d\n", p.name, p.multiProcessorCount, p.clockRate, p.sharedMemPerBlockOptin, p.l2CacheSize);
  uint64_t* d; cudaMalloc(&d, 8 * 4096); uint64_t h[4096];
  int n = 64; k_res<<<1,1>>>(d, n); cudaMemcpy(h, d, 8*(n+1), cudaMemcpyDeviceToHost);
  printf("globaltimer deltas:"); for (int i = 0; i < n; ++i) printf(" %llu", (unsigned long long)h[i]); printf("\ncycles for %d ticks: %llu\n", n, (unsigned long long)h[n]);
  k_rate<<<1,1>>>(d); cudaMemcpy(h, d, 16, cudaMemcpyDeviceToHost);
  printf("rate: %llu ns, %llu cycles -> %.1f MHz\n", (unsigned long long)h[0], (unsigned long long)h[1], (double)h[1]/h[0]*1e3);
  for (unsigned ns : {0u, 100u, 500u, 1000u, 5000u}) { k_sleep<<<1,1>>>(d, ns); cudaMemcpy(h, d, 128, cudaMemcpyDeviceToHost);
    printf("nanosleep(%u):", ns); for (int i = 0; i < 16; ++i) printf(" %llu", (unsigned long long)h[i]); printf("\n"); }
  // bulk copy from host-mapped pinned memory
  uint32_t* hp; cudaHostAlloc(&hp, 4096, cudaHostAllocMapped); for (int i = 0; i < 1024; ++i) hp[i] = i * 7 + 1;
  uint32_t* dp; cudaHostGetDevicePointer(&dp, hp, 0);
  uint32_t* dd; cudaMalloc(&dd, 4096); cudaMemset(dd, 0, 4096);
  k_bulk<<<1,128>>>(dp, dd, 4096); cudaError_t e = cudaDeviceSynchronize();
  uint32_t hh[1024]; cudaMemcpy(hh, dd, 4096, cudaMemcpyDeviceToHost); int bad = 0; for (int i = 0; i < 1024; ++i) bad += hh[i] != (uint32_t)(i*7+1);
  printf("bulk from mapped host: err=%s bad=%d\n", cudaGetErrorString(e), bad);
  return 0;
}
