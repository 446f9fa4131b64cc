// Microbenchmark of the executor's per-firing primitives on B200 (clock64 cycles).
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ void bsync(int id, int n) { asm volatile("bar.sync %0, %1;" :: "r"(id), "r"(n) : "memory"); }
__global__ void k(long long* out, int nthreads_bar) {
  __shared__ unsigned long long a64;
  __shared__ unsigned a32;
  __shared__ volatile unsigned flag;
  __shared__ unsigned arr[1024];
  const int tid = threadIdx.x;
  if (tid == 0) { a64 = 0; a32 = 0; flag = 0; }
  __syncthreads();
  const int R = 256;
  long long t0, t1;
  // 1. bar.sync among first nthreads_bar threads
  if (tid < nthreads_bar) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) bsync(1, nthreads_bar);
    t1 = clock64();
    if (tid == 0) out[0] = (t1 - t0) / R;
  }
  __syncthreads();
  // 2. 64-bit smem atomicMax, one lane per warp, 4 warps
  if ((tid & 31) == 0 && tid < 128) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) atomicMax(&a64, (unsigned long long)(r * 4 + tid));
    t1 = clock64();
    if (tid == 0) out[1] = (t1 - t0) / R;
  }
  __syncthreads();
  // 3. 32-bit smem atomicMax
  if ((tid & 31) == 0 && tid < 128) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) atomicMax(&a32, (unsigned)(r * 4 + tid));
    t1 = clock64();
    if (tid == 0) out[2] = (t1 - t0) / R;
  }
  __syncthreads();
  // 4. threadfence_block
  if (tid == 0) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) { arr[r & 1023] = r; __threadfence_block(); }
    t1 = clock64();
    out[3] = (t1 - t0) / R;
    // 5. globaltimer read
    t0 = clock64();
    uint64_t s = 0;
    for (int r = 0; r < R; ++r) s += gt();
    t1 = clock64();
    out[4] = (t1 - t0) / R + (s == 1);
    // 6. clock64 read
    t0 = clock64();
    long long q = 0;
    for (int r = 0; r < R; ++r) q += clock64();
    t1 = clock64();
    out[5] = (t1 - t0) / R + (q == 1);
    // 7. dependent volatile smem load chain
    arr[0] = 0;
    for (int r = 0; r < 1024; ++r) arr[r] = (r + 1) & 1023;
    unsigned x = 0;
    t0 = clock64();
    for (int r = 0; r < R; ++r) x = ((volatile unsigned*)arr)[x];
    t1 = clock64();
    out[6] = (t1 - t0) / R + (x == 12345);
  }
  __syncthreads();
  // 8. ping-pong latency between warp 0 and warp 4 through a volatile smem flag
  if (tid == 0 || tid == 128) {
    const bool ping = tid == 0;
    t0 = clock64();
    for (int r = 0; r < R; ++r) {
      if (ping) { flag = 2 * r + 1; while (flag != 2 * r + 2) {} }
      else { while (flag != 2 * r + 1) {} flag = 2 * r + 2; }
    }
    t1 = clock64();
    if (ping) out[7] = (t1 - t0) / R;
  }
  __syncthreads();
  // 9. warp shuffle scan (5 steps)
  if (tid < 32) {
    unsigned v = tid;
    t0 = clock64();
    for (int r = 0; r < R; ++r) {
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) { unsigned y = __shfl_up_sync(~0u, v, o); if (tid >= o) v += y; }
    }
    t1 = clock64();
    if (tid == 0) out[8] = (t1 - t0) / R + (v == 7);
  }
  // 10. __nanosleep(0) cost
  if (tid == 0) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) __nanosleep(0);
    t1 = clock64();
    out[9] = (t1 - t0) / R;
  }
}
int main() {
  long long* d; cudaMalloc(&d, 16 * 8); long long h[16];
  for (int nb : {32, 128, 512}) {
    cudaMemset(d, 0, 128);
    k<<<1, 512>>>(d, nb); cudaDeviceSynchronize();
    cudaMemcpy(h, d, 128, cudaMemcpyDeviceToHost);
    printf("bar.sync(%d thr): %lld cyc\n", nb, h[0]);
  }
  printf("atomicMax u64 smem (4 warps): %lld\natomicMax u32 smem: %lld\nthreadfence_block+STS: %lld\nglobaltimer: %lld\nclock64: %lld\nvolatile LDS chain: %lld\nsmem flag ping-pong round trip: %lld\nshfl scan 5 steps: %lld\nnanosleep(0): %lld\n",
         h[1], h[2], h[3], h[4], h[5], h[6], h[7], h[8], h[9]);
  return 0;
}
