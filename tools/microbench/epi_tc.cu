// Epilogue-1 of the tensor-core NTT in isolation (no MMA, no other roles): W warps per CTA, one
// CTA per SM, each warp repeatedly reads one 4-output group of the 5 byte-accumulators from TMEM
// (5 x tcgen05.ld.32x32b.x4), assembles V, multiplies by a shared-memory twiddle (FP64 mulc) and
// stores the result as the next stage's A-operand bytes (STS.32 + STS.U8), as ntt_tc.cu does.
// Prints cycles per group per warp for variants with parts removed (mode bits: 1 no TMEM load,
// 2 no mulc, 4 no stores).
#include <cstdint>
#include <cstdio>

#include "../../paper_conf_isca_jiaodwfcm0z25_b200/csrc/common.cuh"
#include "../../paper_conf_isca_jiaodwfcm0z25_b200/csrc/tc.cuh"
using namespace neo;

__device__ __forceinline__ void ld4(uint32_t a, uint32_t (&v)[4]) {
    asm volatile("tcgen05.ld.sync.aligned.32x32b.x4.b32 {%0, %1, %2, %3}, [%4];\n"
                 : "=r"(v[0]), "=r"(v[1]), "=r"(v[2]), "=r"(v[3]) : "r"(a));
}
__device__ __forceinline__ double vsum(uint32_t d0, uint32_t d1, uint32_t d2, uint32_t d3, uint32_t d4) {
    const u64 w = (u64)(d0 + (d1 << 8)) + (u64)(d2 + (d3 << 8)) * 65536ull;
    return __dadd_rn(__hiloint2double((int)((uint32_t)(w >> 32) + d4 + 0x43300000u), (int)(uint32_t)w), -kTwo52);
}

__global__ void k_epi(int iters, int mode, unsigned long long* cyc, uint32_t* sink) {
    extern __shared__ __align__(16) uint8_t sm[];
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    TWD* T = reinterpret_cast<TWD*>(sm);
    for (int i = threadIdx.x; i < 256; i += blockDim.x) T[i] = TWD{(double)(1000003 + i), (double)(1000003 + i) / 68718428161.0};
    if (warp == 0) tc::tmem_alloc(&tbase, 256);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t ta = tbase + ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)((warp >> 2) * 80);
    const int pa = 4 * ((warp & 3) >> 1) + (lane & 3), x = 8 * (warp & 1) + (lane >> 2);
    uint8_t* a2p = sm + 4096 + (x >> 3) * 768 + (x & 7) * 16;
    const double q = 68718428161.0, qp52 = q + kTwo52;
    uint32_t acc = 0;
    const unsigned long long t0 = clock64();
    for (int it = 0; it < iters; ++it) {
        const int g = it & 3;
        TWD tw[4];
#pragma unroll
        for (int j = 0; j < 4; ++j) tw[j] = T[pa * 16 + 4 * g + j];
        uint32_t v[5][4];
        if (mode & 1) {
#pragma unroll
            for (int b = 0; b < 5; ++b)
#pragma unroll
                for (int j = 0; j < 4; ++j) v[b][j] = (uint32_t)(lane + b + j + it);
        } else {
#pragma unroll
            for (int b = 0; b < 5; ++b) ld4(ta + (uint32_t)(16 * b + 4 * g), v[b]);
            tc::tmem_wait_ld();
        }
#pragma unroll
        for (int j = 0; j < 4; ++j) {
            const double V = vsum(v[0][j] & 0x3FFFFF, v[1][j] & 0x3FFFFF, v[2][j] & 0x3FFFFF, v[3][j] & 0x3FFFFF, v[4][j] & 0x3FFFF);
            const u64 z = (mode & 2) ? (u64)__double_as_longlong(V)
                                     : (u64)__double_as_longlong(__dadd_rn(mulc(V, tw[j], q), qp52));
            uint8_t* row = a2p + (4 * g + j) * 1536;
            if (mode & 4) {
                acc += (uint32_t)z;
            } else {
                *reinterpret_cast<uint32_t*>(row + (pa >> 2) * 128 + (pa & 3) * 4) = (uint32_t)z;
                row[4 * 128 + pa] = (uint8_t)(z >> 32);
            }
        }
    }
    const unsigned long long t1 = clock64();
    if (lane == 0) cyc[blockIdx.x * 32 + warp] = t1 - t0;
    sink[blockIdx.x * blockDim.x + threadIdx.x] = acc;
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc(tbase, 256);
}

int main() {
    unsigned long long* d;
    uint32_t* s;
    cudaMalloc(&d, 148 * 32 * 8);
    cudaMalloc(&s, 148 * 1024 * 4);
    cudaFuncSetAttribute(k_epi, cudaFuncAttributeMaxDynamicSharedMemorySize, 4096 + 24576 + 1024);
    const int iters = 4096;
    for (int warps : {4, 8, 16}) {
        for (int mode : {0, 1, 2, 4, 7}) {
            k_epi<<<148, warps * 32, 4096 + 24576 + 1024>>>(iters, mode, d, s);
            cudaDeviceSynchronize();
            unsigned long long h[32];
            cudaMemcpy(h, d, 32 * 8, cudaMemcpyDeviceToHost);
            unsigned long long mx = 0;
            for (int w = 0; w < warps; ++w) mx = h[w] > mx ? h[w] : mx;
            printf("{\"warps\": %d, \"mode\": %d, \"cycles_per_group_per_warp\": %.1f, \"sm_cycles_per_element\": %.3f}\n",
                   warps, mode, (double)mx / iters, (double)mx / iters / (warps * 32 * 4));
        }
    }
    printf("err %s\n", cudaGetErrorString(cudaGetLastError()));
}
