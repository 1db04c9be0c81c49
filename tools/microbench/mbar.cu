// mbarrier round-trip latency probe (sm_100a): warp-to-warp arrive/wait ping-pong, and
// tcgen05.commit (no MMA) -> wait.
#include <cstdio>
#include <cstdint>
#include "../../paper_conf_isca_jiaodwfcm0z25_b200/csrc/tc.cuh"
using namespace neo;
__global__ void k_pingpong(long long* out, int iters, int use_commit) {
  __shared__ uint64_t a, b;
  __shared__ uint32_t tbase;
  int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (warp == 0) tc::tmem_alloc(&tbase, 32);
  if (threadIdx.x == 0) { tc::mbar_init(&a, 1); tc::mbar_init(&b, 1); }
  tc::fence_before(); __syncthreads(); tc::fence_after();
  long long t0 = clock64();
  for (int i = 0; i < iters; ++i) {
    if (warp == 0 && lane == 0) {
      if (use_commit) tc::commit(&a); else tc::mbar_arrive(&a);
      tc::mbar_wait(&b, i & 1);
    } else if (warp == 1 && lane == 0) {
      tc::mbar_wait(&a, i & 1);
      tc::mbar_arrive(&b);
    }
  }
  long long t1 = clock64();
  __syncthreads();
  if (warp == 0) tc::tmem_dealloc(tbase, 32);
  if (threadIdx.x == 0) out[blockIdx.x] = (t1 - t0) / iters;
}
int main() {
  long long* d; cudaMalloc(&d, 8 * 148); long long h;
  for (int c = 0; c < 2; ++c) {
    k_pingpong<<<1, 64>>>(d, 10000, c); cudaDeviceSynchronize();
    cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
    printf("%s round trip: %lld cycles\n", c ? "commit->wait / arrive->wait" : "arrive->wait x2", h);
  }
  printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
