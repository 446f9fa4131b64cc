// Latency of warp-collective primitives and branches on B200 (clock64 cycles per op, dependent chain).
#include <cstdio>
#include <cstdint>
__global__ void k(long long* out, int sel, unsigned long long mul) {
  const int lane = threadIdx.x & 31;
  const int R = 512;
  long long t0, t1;
  unsigned v = lane + 1;
  // 0: __reduce_max_sync chain
  t0 = clock64();
  for (int r = 0; r < R; ++r) v = __reduce_max_sync(~0u, v + lane) & 0xffff;
  t1 = clock64();
  if (lane == 0) out[0] = (t1 - t0) / R + (v == 12345);
  // 1: __reduce_add_sync chain
  t0 = clock64();
  for (int r = 0; r < R; ++r) v = __reduce_add_sync(~0u, v) & 0xffff;
  t1 = clock64();
  if (lane == 0) out[1] = (t1 - t0) / R + (v == 12345);
  // 2: ballot + popc chain
  t0 = clock64();
  for (int r = 0; r < R; ++r) v = __popc(__ballot_sync(~0u, (v >> (lane & 7)) & 1)) + v;
  t1 = clock64();
  if (lane == 0) out[2] = (t1 - t0) / R + (v == 12345);
  // 3: shfl chain
  t0 = clock64();
  for (int r = 0; r < R; ++r) v = __shfl_sync(~0u, v, (lane + 1) & 31) + 1;
  t1 = clock64();
  if (lane == 0) out[3] = (t1 - t0) / R + (v == 12345);
  // 4: __all_sync chain
  t0 = clock64();
  for (int r = 0; r < R; ++r) v += __all_sync(~0u, v > 3);
  t1 = clock64();
  if (lane == 0) out[4] = (t1 - t0) / R + (v == 12345);
  // 5: 64-bit multiply chain
  unsigned long long x = mul + lane;
  t0 = clock64();
  for (int r = 0; r < R; ++r) x = x * mul + 1;
  t1 = clock64();
  if (lane == 0) out[5] = (t1 - t0) / R + (x == 12345);
  // 6: dependent uniform branches (data-dependent, warp-uniform)
  unsigned y = sel;
  t0 = clock64();
  for (int r = 0; r < R; ++r) {
    if (y & 1) y = y * 3 + 1; else y = y >> 1;
    y |= 0x10000;
  }
  t1 = clock64();
  if (lane == 0) out[6] = (t1 - t0) / R + (y == 12345);
  // 7: switch via jump table
  unsigned z = sel;
  t0 = clock64();
  for (int r = 0; r < R; ++r) {
    switch ((z >> 3) & 7) {
      case 0: z = z * 5 + 1; break;
      case 1: z = z * 7 + 3; break;
      case 2: z = z ^ 0x1234; break;
      case 3: z = z + 0x777; break;
      case 4: z = z * 11; break;
      case 5: z = z - 3; break;
      case 6: z = z * 13 + 5; break;
      default: z = z ^ 0xffff; break;
    }
  }
  t1 = clock64();
  if (lane == 0) out[7] = (t1 - t0) / R + (z == 12345);
  // 8: divergent if (half the warp)
  unsigned w = lane;
  t0 = clock64();
  for (int r = 0; r < R; ++r) {
    if ((w + r) & 1) w = w * 3 + 1; else w = w + 7;
    w &= 0xffff;
  }
  t1 = clock64();
  if (lane == 0) out[8] = (t1 - t0) / R + (w == 12345);
}
int main() {
  long long* d; cudaMalloc(&d, 16 * 8); long long h[16];
  k<<<1, 32>>>(d, 7, 0x9E3779B97F4A7C15ull); cudaDeviceSynchronize();
  cudaMemcpy(h, d, 128, cudaMemcpyDeviceToHost);
  const char* names[] = {"reduce_max", "reduce_add", "ballot+popc", "shfl", "all_sync", "mul64", "uniform branch", "switch (8-way)", "divergent if"};
  for (int i = 0; i < 9; ++i) printf("%-16s %lld cyc/iter\n", names[i], h[i]);
  return 0;
}
