// Throughput probe: DFMA vs IMAD.WIDE vs FFMA vs 64-bit Shoup butterfly vs FP64 butterfly on sm_100a.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
typedef uint64_t u64;
#define ITERS 4096
__global__ void k_dfma(double* out, double a, double b) {
  double x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0+4, x5=x0+5, x6=x0+6, x7=x0+7;
  for (int i = 0; i < ITERS; ++i) {
    x0 = fma(x0, a, b); x1 = fma(x1, a, b); x2 = fma(x2, a, b); x3 = fma(x3, a, b);
    x4 = fma(x4, a, b); x5 = fma(x5, a, b); x6 = fma(x6, a, b); x7 = fma(x7, a, b);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}
__global__ void k_ffma(float* out, float a, float b) {
  float x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0+4, x5=x0+5, x6=x0+6, x7=x0+7;
  for (int i = 0; i < ITERS; ++i) {
    x0 = fmaf(x0, a, b); x1 = fmaf(x1, a, b); x2 = fmaf(x2, a, b); x3 = fmaf(x3, a, b);
    x4 = fmaf(x4, a, b); x5 = fmaf(x5, a, b); x6 = fmaf(x6, a, b); x7 = fmaf(x7, a, b);
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}
__global__ void k_imadw(u64* out, unsigned a, unsigned b) {
  u64 x0 = threadIdx.x, x1 = x0 + 1, x2 = x0 + 2, x3 = x0 + 3, x4 = x0+4, x5=x0+5, x6=x0+6, x7=x0+7;
  for (int i = 0; i < ITERS; ++i) {
    x0 = (u64)(unsigned)x0 * a + x0; x1 = (u64)(unsigned)x1 * a + x1; x2 = (u64)(unsigned)x2 * a + x2; x3 = (u64)(unsigned)x3 * a + x3;
    x4 = (u64)(unsigned)x4 * a + x4; x5 = (u64)(unsigned)x5 * a + x5; x6 = (u64)(unsigned)x6 * a + x6; x7 = (u64)(unsigned)x7 * a + x7;
  }
  out[blockIdx.x * blockDim.x + threadIdx.x] = x0 + x1 + x2 + x3 + x4 + x5 + x6 + x7;
}
// int Shoup CT butterfly with full corrections (current kernel style)
__device__ __forceinline__ u64 shoup(u64 a, u64 w, u64 ws, u64 q) { u64 r = a * w - __umul64hi(a, ws) * q; return r >= q ? r - q : r; }
__global__ void k_bfly_int(u64* out, u64 w, u64 ws, u64 q) {
  u64 x[8]; for (int j = 0; j < 8; ++j) x[j] = threadIdx.x * 8 + j;
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      u64 U = x[j], V = shoup(x[j + 4], w, ws, q);
      u64 s = U + V; x[j] = s >= q ? s - q : s;
      x[j + 4] = U >= V ? U - V : U + q - V;
    }
  }
  u64 s = 0; for (int j = 0; j < 8; ++j) s += x[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
// FP64 lazy butterfly: modmul by w with 6 DP ops, no corrections
__global__ void k_bfly_fp(double* out, double w, double wq, double q) {
  const double M = 6755399441055744.0;  // 1.5 * 2^52
  double x[8]; for (int j = 0; j < 8; ++j) x[j] = threadIdx.x * 8 + j;
  for (int i = 0; i < ITERS / 4; ++i) {
#pragma unroll
    for (int j = 0; j < 4; ++j) {
      double y = x[j + 4];
      double h = y * w, l = fma(y, w, -h);
      double qf = fma(y, wq, M) - M;
      double t = fma(-qf, q, h) + l;
      double U = x[j];
      x[j] = U + t; x[j + 4] = U - t;
    }
  }
  double s = 0; for (int j = 0; j < 8; ++j) s += x[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
int main() {
  int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
  int clk; cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  void* buf; cudaMalloc(&buf, 64 << 20);
  dim3 grid(sms * 8), block(256);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  double thr = (double)grid.x * block.x;
  auto run = [&](const char* name, auto fn, double ops_per_thread) {
    fn(); cudaDeviceSynchronize();
    cudaEventRecord(a); for (int r = 0; r < 5; ++r) fn(); cudaEventRecord(b); cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b); ms /= 5;
    double rate = thr * ops_per_thread / (ms * 1e-3);
    printf("%-12s %8.3f ms  %10.3f Gop/s  %6.1f ops/clk/SM (at %d MHz)\n", name, ms, rate / 1e9, rate / (sms * clk * 1e3), clk / 1000);
  };
  run("dfma", [&] { k_dfma<<<grid, block>>>((double*)buf, 1.0000001, 0.5); }, 8.0 * ITERS);
  run("ffma", [&] { k_ffma<<<grid, block>>>((float*)buf, 1.0000001f, 0.5f); }, 8.0 * ITERS);
  run("imad.wide", [&] { k_imadw<<<grid, block>>>((u64*)buf, 12345u, 7u); }, 8.0 * ITERS);
  run("bfly_int", [&] { k_bfly_int<<<grid, block>>>((u64*)buf, 123456789ull, 1234567891234ull, 68719403009ull); }, 4.0 * ITERS / 4);
  run("bfly_fp64", [&] { k_bfly_fp<<<grid, block>>>((double*)buf, 123456789.0, 123456789.0 / 68719403009.0, 68719403009.0); }, 4.0 * ITERS / 4);
  printf("err: %s\n", cudaGetErrorString(cudaGetLastError()));
}
