// Microbenchmark (clock64 cycles, one warp unless noted) of the primitives on the executor's
// per-firing path: fences, %globaltimer, FP64 conversions, REDUX, indirect branch, barriers.
#include <cstdio>
#include <cstdint>
__device__ __forceinline__ uint64_t gt() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }
__device__ __forceinline__ void bsync(int id, int n) { asm volatile("bar.sync %0, %1;" :: "r"(id), "r"(n) : "memory"); }
__device__ __forceinline__ void barv(int id, int n) { asm volatile("bar.arrive %0, %1;" :: "r"(id), "r"(n) : "memory"); }
__device__ int sel_fn(int k, int x);
__global__ void k(long long* out, const int* kinds, double nspu, int64_t tau) {
  __shared__ unsigned arr[1024];
  __shared__ volatile unsigned flag[8];
  const int tid = threadIdx.x, lane = tid & 31, w = tid >> 5;
  const int R = 256;
  long long t0, t1;
  for (int j = tid; j < 1024; j += blockDim.x) arr[j] = (j + 1) & 1023;
  __syncthreads();
  if (tid < 32) {
    // 0: STS + fence.sc.cta
    t0 = clock64();
    for (int r = 0; r < R; ++r) { arr[(r + lane) & 1023] = r; __threadfence_block(); }
    t1 = clock64(); if (!lane) out[0] = (t1 - t0) / R;
    // 1: STS + fence.acq_rel.cta
    t0 = clock64();
    for (int r = 0; r < R; ++r) { arr[(r + lane) & 1023] = r; asm volatile("fence.acq_rel.cta;" ::: "memory"); }
    t1 = clock64(); if (!lane) out[1] = (t1 - t0) / R;
    // 2: globaltimer dependent
    uint64_t s = 0;
    t0 = clock64();
    for (int r = 0; r < R; ++r) s += gt();
    t1 = clock64(); if (!lane) out[2] = (t1 - t0) / R + (s == 1);
    // 3: I2F.F64 -> DMUL -> F2I chain (arrival ns)
    int64_t x = lane;
    t0 = clock64();
    for (int r = 0; r < R; ++r) x = (int64_t)((double)(x * tau) * nspu) & 1023;
    t1 = clock64(); if (!lane) out[3] = (t1 - t0) / R + (x == -5);
    // 4: same in integer
    x = lane;
    t0 = clock64();
    for (int r = 0; r < R; ++r) x = (x * tau + 7) & 1023;
    t1 = clock64(); if (!lane) out[4] = (t1 - t0) / R + (x == -5);
    // 5: reduce_min chain
    unsigned u = lane;
    t0 = clock64();
    for (int r = 0; r < R; ++r) u = __reduce_min_sync(~0u, u + lane) & 1023;
    t1 = clock64(); if (!lane) out[5] = (t1 - t0) / R + (u == 7777);
    // 6: ballot+popc chain
    u = lane;
    t0 = clock64();
    for (int r = 0; r < R; ++r) u = __popc(__ballot_sync(~0u, (u + lane) & 1) & ((1u << lane) - 1)) + u;
    t1 = clock64(); if (!lane) out[6] = (t1 - t0) / R + (u == 7777);
    // 7: switch dispatch (indirect branch) chain
    int y = lane;
    t0 = clock64();
    for (int r = 0; r < R; ++r) y = sel_fn(kinds[r & 7], y);
    t1 = clock64(); if (!lane) out[7] = (t1 - t0) / R + (y == 7777);
    // 8: dependent LDS chain
    u = lane;
    t0 = clock64();
    for (int r = 0; r < R; ++r) u = arr[u];
    t1 = clock64(); if (!lane) out[8] = (t1 - t0) / R + (u == 7777);
    // 9: volatile LDS + STS pair (flag publish/poll)
    t0 = clock64();
    for (int r = 0; r < R; ++r) { flag[0] = r; u += flag[1]; }
    t1 = clock64(); if (!lane) out[9] = (t1 - t0) / R + (u == 7777);
  }
  __syncthreads();
  // 10: 4-warp named barrier round (warps 0,4,8,12 of 16 -> same SMSP)
  if ((w & 3) == 0) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) bsync(1, 128);
    t1 = clock64(); if (tid == 0) out[10] = (t1 - t0) / R;
  }
  __syncthreads();
  // 11: 4-warp barrier, warps 0..3 (4 SMSPs)
  if (w < 4) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) bsync(2, 128);
    t1 = clock64(); if (tid == 0) out[11] = (t1 - t0) / R;
  }
  __syncthreads();
  // 12: leader sync / others arrive + sync next (the B4/B2 pattern), warps 0,4,8,12
  if ((w & 3) == 0) {
    t0 = clock64();
    for (int r = 0; r < R; ++r) {
      if (w == 0) bsync(3, 128); else barv(3, 128);
      bsync(4, 128);
    }
    t1 = clock64(); if (tid == 0) out[12] = (t1 - t0) / R;
  }
  __syncthreads();
  // 13: STS + bar.sync (4 warps) + LDS.128 of the 4 totals (group_scan core)
  if ((w & 3) == 0) {
    unsigned acc = 0;
    t0 = clock64();
    for (int r = 0; r < R; ++r) {
      if (lane == 31) arr[512 + (w >> 2) + 8 * (r & 1)] = acc + r;
      bsync(5, 128);
      const uint4 a = *reinterpret_cast<const uint4*>(&arr[512 + 8 * (r & 1)]);
      acc += a.x + a.y + a.z + a.w;
    }
    t1 = clock64(); if (tid == 0) out[13] = (t1 - t0) / R + (acc == 1);
  }
}
__device__ __noinline__ int sel_fn(int k, int x) {
  switch (k) {
    case 0: return x + 1; case 1: return x ^ 3; case 2: return x * 3; case 3: return x - 7;
    case 4: return x >> 1; case 5: return x + 11; case 6: return x * 5; default: return x | 1;
  }
}
int main() {
  long long* d; cudaMalloc(&d, 32 * 8); long long h[32];
  int* kinds; cudaMalloc(&kinds, 8 * 4); int hk[8] = {3, 3, 3, 3, 3, 3, 3, 3}; cudaMemcpy(kinds, hk, 32, cudaMemcpyHostToDevice);
  cudaMemset(d, 0, 256);
  k<<<1, 512>>>(d, kinds, 1.0, 22); cudaDeviceSynchronize();
  cudaMemcpy(h, d, 256, cudaMemcpyDeviceToHost);
  const char* names[] = {"STS+fence.sc.cta", "STS+fence.acq_rel.cta", "globaltimer read", "I2F.F64*DMUL->F2I chain",
                         "int64 mul chain", "reduce_min chain", "ballot+popc chain", "switch dispatch (noinline)",
                         "dependent LDS", "volatile STS+LDS", "bar.sync 4 warps same SMSP", "bar.sync 4 warps 4 SMSPs",
                         "arrive/sync + sync (B4,B2)", "STS+bar+LDS.128 (scan core)"};
  for (int i = 0; i < 14; ++i) printf("%-32s %lld cyc\n", names[i], h[i]);
  return 0;
}
