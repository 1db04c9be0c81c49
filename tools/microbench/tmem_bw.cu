// TMEM read throughput probe (sm_100a): W warps of one CTA per SM repeatedly tcgen05.ld
// 32x32b.xC (each warp its lane quadrant warp % 4), C in {8, 16, 32}; prints bytes per cycle
// per SM.  Used to size the tensor-core NTT's epilogues (20 bytes of TMEM per output element
// per radix-16 stage).
#include <cstdint>
#include <cstdio>

#include "../../paper_conf_isca_jiaodwfcm0z25_b200/csrc/tc.cuh"
using namespace neo;

template <int C>
__device__ __forceinline__ void ld(uint32_t taddr, uint32_t (&v)[C]);
template <>
__device__ __forceinline__ void ld<8>(uint32_t a, uint32_t (&v)[8]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];\n"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]) : "r"(a));
}
template <>
__device__ __forceinline__ void ld<16>(uint32_t a, uint32_t (&v)[16]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x16.b32 {%0,%1,%2,%3,%4,%5,%6,%7,%8,%9,%10,%11,%12,%13,%14,%15}, [%16];\n"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]), "=r"(v[4]), "=r"(v[5]), "=r"(v[6]), "=r"(v[7]),
                   "=r"(v[8]), "=r"(v[9]), "=r"(v[10]), "=r"(v[11]), "=r"(v[12]), "=r"(v[13]), "=r"(v[14]), "=r"(v[15])
                 : "r"(a));
}

template <int C>
__global__ void k_tmem(int iters, unsigned long long* cyc, uint32_t* sink) {
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x >> 5;
    if (warp == 0) tc::tmem_alloc(&tbase, 512);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t t = tbase + ((uint32_t)((warp & 3) * 32) << 16);
    uint32_t acc = 0;
    const unsigned long long t0 = clock64();
    for (int i = 0; i < iters; ++i) {
        uint32_t v[C];
        ld<C>(t + (uint32_t)((i * C + (warp >> 2) * 64) & 511), v);
        tc::tmem_wait_ld();
#pragma unroll
        for (int j = 0; j < C; ++j) acc ^= v[j];
    }
    const unsigned long long t1 = clock64();
    __syncthreads();
    if (threadIdx.x == 0) cyc[blockIdx.x] = t1 - t0;
    sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc(tbase, 512);
}

template <int C>
void run(int warps, unsigned long long* d, uint32_t* s) {
    const int iters = 4096;
    k_tmem<C><<<148, warps * 32>>>(iters, d, s);
    cudaDeviceSynchronize();
    k_tmem<C><<<148, warps * 32>>>(iters, d, s);
    cudaDeviceSynchronize();
    unsigned long long h;
    cudaMemcpy(&h, d, 8, cudaMemcpyDeviceToHost);
    const double bytes = (double)warps * iters * 32 * C * 4;
    printf("{\"cols_per_ld\": %d, \"warps\": %d, \"bytes_per_clk_per_sm\": %.1f}\n", C, warps, bytes / (double)h);
}

int main() {
    unsigned long long* d;
    uint32_t* s;
    cudaMalloc(&d, 148 * 8);
    cudaMalloc(&s, 148 * 1024 * 4);
    for (int w : {4, 8, 16}) {
        run<8>(w, d, s);
        run<16>(w, d, s);
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
