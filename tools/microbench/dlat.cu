// FP64 latency / occupancy probe on sm_100a: dependent DFMA chains, varying warps/SM and ILP.
#include <cstdio>
#include <cuda_runtime.h>
template <int ILP>
__global__ void k(double* out, double a, double b, int iters) {
  double x[ILP];
#pragma unroll
  for (int j = 0; j < ILP; ++j) x[j] = threadIdx.x + j;
  for (int i = 0; i < iters; ++i) {
#pragma unroll
    for (int j = 0; j < ILP; ++j) x[j] = fma(x[j], a, b);
  }
  double s = 0;
#pragma unroll
  for (int j = 0; j < ILP; ++j) s += x[j];
  out[blockIdx.x * blockDim.x + threadIdx.x] = s;
}
template <int ILP>
void run(int warps_per_sm, double* buf, int sms, int clk) {
  int iters = 4096;
  dim3 grid(sms), block(32 * warps_per_sm);
  k<ILP><<<grid, block>>>(buf, 1.0000001, 0.5, iters);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  cudaEventRecord(a); k<ILP><<<grid, block>>>(buf, 1.0000001, 0.5, iters); cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  double cycles = ms * 1e-3 * clk * 1e3;
  double ops_per_clk_sm = (double)warps_per_sm * 32 * ILP * iters / cycles;
  double lat = cycles / iters;  // per chain step
  printf("warps/SM %2d ILP %d : %6.1f DFMA/clk/SM, %6.2f cycles per dependent step\n", warps_per_sm, ILP, ops_per_clk_sm, lat);
}
int main() {
  int sms, clk; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0); cudaDeviceGetAttribute(&clk, cudaDevAttrClockRate, 0);
  double* buf; cudaMalloc(&buf, 64 << 20);
  for (int w : {1, 4, 8, 16, 32}) { run<1>(w, buf, sms, clk); run<2>(w, buf, sms, clk); run<4>(w, buf, sms, clk); run<8>(w, buf, sms, clk); }
}
