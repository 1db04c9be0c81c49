// int8 tensor-core peak of one B200 (sm_100a), measured with the same tcgen05 path the NTT and
// BConv kernels use: tcgen05.mma.cta_group::1.kind::i8 (u8 x u8 -> s32 in TMEM), operands in
// shared memory (SWIZZLE_NONE K-major, the kernels' layout), one persistent CTA per SM, one
// thread issuing back-to-back MMAs into two TMEM accumulators.  No global traffic: this is the
// tensor pipe's throughput for the shape, the denominator of the "int8 tensor fraction" of the
// NTT / BConv kernels.  Shapes: M = 128 and N in {80 (the NTT's), 96, 256}, K = 32 per MMA.
// Output: one JSON line.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 i8peak.cu
#include <cstdint>
#include <cstdio>
#include <vector>

#include "../../paper_conf_isca_jiaodwfcm0z25_b200/csrc/tc.cuh"
using namespace neo;

__global__ void __launch_bounds__(128, 1) k_peak(int n, int iters, unsigned long long* cyc) {
    extern __shared__ __align__(1024) uint8_t sm[];
    __shared__ uint64_t mb[2];
    __shared__ uint32_t tbase;
    const int warp = threadIdx.x >> 5;
    for (int i = threadIdx.x; i < (128 + 256) * 32 / 4; i += blockDim.x) reinterpret_cast<uint32_t*>(sm)[i] = i * 2654435761u;
    if (warp == 0) tc::tmem_alloc(&tbase, 512);
    if (threadIdx.x == 0) {
        tc::mbar_init(&mb[0], 1);
        tc::mbar_init(&mb[1], 1);
    }
    tc::fence_proxy_async();
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t t = tbase;
    if (threadIdx.x == 0) {
        const uint32_t a = tc::smem_u32(sm), b = tc::smem_u32(sm + 128 * 32);
        const uint32_t id = tc::idesc_u8(128, n);
        const uint64_t ad = tc::sdesc(a, 128, 256), bd = tc::sdesc(b, 128, 256);
        const unsigned long long t0 = clock64();
        for (int i = 0; i < iters; ++i) {
            tc::mma_u8(t + (i & 1) * 256, ad, bd, id, i > 1);
            if ((i & 255) == 255) {       // bounded issue queue: wait for the batch before last
                const int k = i >> 8;
                tc::commit(&mb[k & 1]);
                if (k > 0) tc::mbar_wait(&mb[(k - 1) & 1], ((k - 1) >> 1) & 1);
            }
        }
        const int kl = (iters >> 8) - 1;  // iters is a multiple of 256: wait for the last batch
        tc::mbar_wait(&mb[kl & 1], (kl >> 1) & 1);
        cyc[blockIdx.x] = clock64() - t0;
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc(t, 512);
}

int main() {
    int sms = 0, mhz = 0;
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    cudaDeviceGetAttribute(&mhz, cudaDevAttrClockRate, 0);
    unsigned long long* d;
    cudaMalloc(&d, sms * 8);
    cudaFuncSetAttribute(k_peak, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
    printf("{\"sms\": %d, \"shapes\": [", sms);
    const int ns[3] = {80, 96, 256};
    for (int s = 0; s < 3; ++s) {
        const int n = ns[s], iters = 1 << 16;
        k_peak<<<sms, 128, 64 * 1024>>>(n, 1024, d);       // warm-up (multiple of 256)
        cudaEvent_t e0, e1;
        cudaEventCreate(&e0);
        cudaEventCreate(&e1);
        cudaEventRecord(e0);
        k_peak<<<sms, 128, 64 * 1024>>>(n, iters, d);
        cudaEventRecord(e1);
        cudaEventSynchronize(e1);
        float ms = 0;
        cudaEventElapsedTime(&ms, e0, e1);
        std::vector<unsigned long long> c(sms);
        cudaMemcpy(c.data(), d, sms * 8, cudaMemcpyDeviceToHost);
        unsigned long long cmax = 0;
        for (auto x : c) cmax = x > cmax ? x : cmax;
        const double macs = (double)sms * iters * 128.0 * n * 32.0;
        printf("%s{\"M\": 128, \"N\": %d, \"K\": 32, \"ms\": %.4f, \"tops\": %.1f, \"macs_per_clk_per_sm\": %.1f}",
               s ? ", " : "", n, ms, 2.0 * macs / (ms * 1e-3) / 1e12, 128.0 * n * 32.0 * iters / (double)cmax);
    }
    printf("], \"err\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
