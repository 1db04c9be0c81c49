// BConv epilogue group body in isolation: W warps/SM each process `iters` groups of 8 targets
// (5 byte planes -> V -> FP64 Barrett -> lazy store), synthetic planes, optional stores.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
typedef unsigned long long u64;
__device__ __forceinline__ double u2d(u64 x) { return __longlong_as_double((long long)(x | 0x4330000000000000ull)) - 4503599627370496.0; }
struct TgtC { double t, tinv; long long off, pad; };
__global__ void k(u64* out, const TgtC* tabg, int iters, int store, int N, unsigned long long* cyc) {
  __shared__ TgtC tab[64];
  if (threadIdx.x < 64) tab[threadIdx.x] = tabg[threadIdx.x];
  __syncthreads();
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  u64* outb = out + (size_t)blockIdx.x * 128 + (warp & 3) * 32 + lane;
  const double kMagic = 6755399441055744.0;
  unsigned long long t0 = clock64();
  uint32_t seed = threadIdx.x * 7919u + blockIdx.x;
  for (int it = 0; it < iters; ++it) {
    const int g = (it * 8 + warp * 8) & 31;
    uint32_t v[40];
#pragma unroll
    for (int x = 0; x < 40; ++x) v[x] = (seed + x * 2654435761u) & 0x3FFFFF;
    seed = seed * 1664525u + 1013904223u;
    double r[8];
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const TgtC& C = tab[g + u];
      const uint32_t* D = &v[5 * u];
      const u64 V = (u64)(D[0] + (D[1] << 8)) + ((u64)D[2] << 16) + ((u64)D[3] << 24) + ((u64)(D[4] & 0x3FFFF) << 32);
      const double Vd = u2d(V);
      const double qf = __dadd_rn(__fma_rn(Vd, C.tinv, kMagic), -kMagic);
      r[u] = __fma_rn(-qf, C.t, Vd);
    }
#pragma unroll
    for (int u = 0; u < 8; ++u) {
      const u64 val = (u64)__double_as_longlong(r[u]);
      if (store) outb[tab[g + u].off] = val; else if (val == 0x1234567ull) outb[0] = val;
    }
  }
  unsigned long long t1 = clock64();
  if (lane == 0 && blockIdx.x == 0) cyc[warp] = t1 - t0;
}
int main() {
  const int N = 65536, sms = 148, iters = 2000;
  u64* out; cudaMalloc(&out, (size_t)64 * N * 8 + 148 * 128 * 8);
  TgtC h[64];
  for (int t = 0; t < 64; ++t) { double q = 68719476731.0 - 2 * t; h[t] = {q, 1.0 / q, (long long)(t % 36) * N, 0}; }
  TgtC* tab; cudaMalloc(&tab, sizeof(h)); cudaMemcpy(tab, h, sizeof(h), cudaMemcpyHostToDevice);
  unsigned long long* cyc; cudaMalloc(&cyc, 64 * 8);
  for (int store = 0; store < 2; ++store)
    for (int w : {4, 8, 16, 24}) {
      k<<<sms, 32 * w>>>(out, tab, 10, store, N, cyc);
      cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
      cudaEventRecord(a); k<<<sms, 32 * w>>>(out, tab, iters, store, N, cyc); cudaEventRecord(b); cudaEventSynchronize(b);
      float ms; cudaEventElapsedTime(&ms, a, b);
      unsigned long long c[64]; cudaMemcpy(c, cyc, 64 * 8, cudaMemcpyDeviceToHost);
      printf("store %d warps/SM %2d: %.3f ms, warp0 %.0f cycles/group, SM: %.1f cycles per group (all warps), err=%s\n", store, w, ms,
             (double)c[0] / iters, (double)c[0] / iters / w, cudaGetErrorString(cudaGetLastError()));
    }
  return 0;
}
