// bconv_tc.cu -- BConv (Algorithm 2) as a u8 GEMM on the 5th-gen tensor cores.
//
// Neo recasts BConv as (BS*N x alpha) . (alpha x alpha') (L290, L470) and maps it onto the
// A100 FP64 tensor cores.  On sm_100a the dense int8 path is the fast one, so each 36-bit
// operand is split into 5 bytes with the *constant* side pre-shifted:
//
//   y_i = [c_i qhat_i^-1]_{q_i} = sum_a y_i^(a) 2^(8a)          (bytes of the data, on the fly)
//   C_b[(i,a), t] = byte_b( (2^(8a) qhat_i) mod t )              (host constant, per (l, digit))
//   D_b[m, t]    = sum_(i,a) y_i^(a)[m] C_b[(i,a), t]            (one tcgen05.mma kind::i8 GEMM)
//   out_t[m]     = sum_b 2^(8b) D_b[m, t]  mod t                 (epilogue, FP64)
//
// so sum_b 2^(8b) D_b == sum_i y_i (qhat_i mod t) (mod t): Algorithm 1's result exactly.
// GEMM shape per 128-coefficient tile: M = 128, K = 5*n_in <= 64 (two K=32 MMAs),
// N = 5*n_out rounded up to 16 (<= 256).  A (8 KB) is produced by the CUDA cores into
// shared memory in the SWIZZLE_NONE K-major layout, B (<= 16 KB) is loaded once per CTA,
// the accumulator D lives in TMEM (256 columns) and is drained with tcgen05.ld.
// D_b <= 60 * 255 * 255 < 2^22, so s32 accumulation is exact.
#include "bconv_tc.h"
#include "common.cuh"
#include "tc.cuh"

namespace neo {

constexpr int kTileM = 128;
constexpr int kTmemCols = 256;

template <class LoadB>
__device__ __forceinline__ void bconv_tc_body(const BConvTC& P, const BConvIO& io, LoadB loadB, int N,
                                              int tiles_per_entry, int total_tiles) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t* sA = smem;                     // 128 rows x 64 B
    uint8_t* sB = smem + kTileM * 64;       // ncols rows x 64 B
    __shared__ uint64_t mbar;
    __shared__ uint32_t tmem_base;

    const int tid = threadIdx.x, warp = tid >> 5;
    if (warp == 0) tc::tmem_alloc(&tmem_base, kTmemCols);
    if (tid == 0) tc::mbar_init(&mbar, 1);
    {
        uint4* s = reinterpret_cast<uint4*>(sB);
        for (int e = tid; e < P.ncols * 4; e += kTileM) s[e] = loadB(e);
    }
    tc::fence_proxy_async();
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = tmem_base;
    const uint32_t idesc = tc::idesc_u8(kTileM, P.ncols);
    const uint32_t aaddr = tc::smem_u32(sA), baddr = tc::smem_u32(sB);
    // row m of A at (m/8)*512 + (m%8)*16, K chunk c (16 bytes) at + c*128
    uint8_t* arow = sA + (tid >> 3) * 512 + (tid & 7) * 16;
    uint32_t phase = 0;

    for (int tile = blockIdx.x; tile < total_tiles; tile += gridDim.x) {
        const int b = tile / tiles_per_entry;
        const int m = (tile - b * tiles_per_entry) * kTileM + tid;
        // ---- A row: bytes of y_i = [c_i qhat_i^-1]_{q_i}, y_i occupying bits [40 i, 40 i + 40)
        uint32_t w[16];
#pragma unroll
        for (int k = 0; k < 16; ++k) w[k] = 0;
        const u64* in = io.in + b * io.in_bstride + m;
#pragma unroll
        for (int i = 0; i < 12; ++i) {
            if (i < P.n_in) {
                const double q = P.qin[i];
                const double c = u2d(in[(size_t)io.in_off[i] * N]);
                const u64 y = d2u(canon(mulc(c, P.qhat_inv[i], q), q, P.qinv_in[i]));
                const int bit = 40 * i, wi = bit >> 5, sh = bit & 31;
                w[wi] |= (uint32_t)(y << sh);
                w[wi + 1] |= (uint32_t)(y >> (32 - sh));
                if (sh > 24) w[wi + 2] |= (uint32_t)(y >> (64 - sh));
            }
        }
#pragma unroll
        for (int c = 0; c < 4; ++c)
            *reinterpret_cast<uint4*>(arow + c * 128) = make_uint4(w[4 * c], w[4 * c + 1], w[4 * c + 2], w[4 * c + 3]);
        tc::fence_proxy_async();
        __syncthreads();
        // ---- one thread issues the GEMM: K = 64 as two K = 32 steps (LBO = 128, SBO = 512)
        if (tid == 0) {
            tc::fence_after();
            tc::mma_u8(tmem, tc::sdesc(aaddr, 128, 512), tc::sdesc(baddr, 128, 512), idesc, 0);
            tc::mma_u8(tmem, tc::sdesc(aaddr + 256, 128, 512), tc::sdesc(baddr + 256, 128, 512), idesc, 1);
            tc::commit(&mbar);
        }
        tc::mbar_wait(&mbar, phase);
        phase ^= 1;
        tc::fence_after();
        // ---- epilogue: lane (warp*32 + lane) = row m; columns 5t..5t+4 hold D_0..D_4 of target t
        const uint32_t trow = tmem + ((uint32_t)(warp * 32) << 16);
        u64* outb = io.out + b * io.out_bstride + m;
        for (int g = 0; g < P.n_out; g += 8) {
            uint32_t v[40];
#pragma unroll
            for (int s = 0; s < 5; ++s) {
                uint32_t (&vv)[8] = *reinterpret_cast<uint32_t (*)[8]>(&v[8 * s]);
                tc::tmem_ld8(trow + (uint32_t)(5 * g + 8 * s), vv);
            }
            tc::tmem_wait_ld();
#pragma unroll
            for (int u = 0; u < 8; ++u) {
                const int t = g + u;
                if (t < P.n_out) {
                    const uint32_t* D = &v[5 * u];
                    const u64 lo = (u64)D[0] + ((u64)D[1] << 8) + ((u64)D[2] << 16);     // < 2^39
                    const u64 hi = (u64)D[3] + ((u64)D[4] << 8);                          // < 2^31
                    const double tq = P.t[t];
                    const double r = __dadd_rn(u2d(lo), mulc(u2d(hi), P.c24[t], tq));   // == V (mod t)
                    outb[(size_t)io.out_off[t] * N] = d2u(canon(r, tq, P.tinv[t]));
                }
            }
        }
        tc::fence_before();
        __syncthreads();
    }
    if (warp == 0) tc::tmem_dealloc(tmem, kTmemCols);
}

__global__ void __launch_bounds__(kTileM, 1)
k_bconv_tc_g(const __grid_constant__ BConvTC P, const __grid_constant__ BConvIO io, const uint4* __restrict__ bmat,
             int N, int tiles_per_entry, int total_tiles) {
    bconv_tc_body(P, io, [&](int e) { return bmat[e]; }, N, tiles_per_entry, total_tiles);
}

__global__ void __launch_bounds__(kTileM, 1)
k_bconv_tc_p(const __grid_constant__ BConvTC P, const __grid_constant__ BConvIO io,
             const __grid_constant__ BMatParam B, int N, int tiles_per_entry, int total_tiles) {
    bconv_tc_body(P, io, [&](int e) { return B.d[e]; }, N, tiles_per_entry, total_tiles);
}

size_t bconv_tc_smem(int ncols) { return (size_t)kTileM * 64 + (size_t)ncols * 64; }

cudaError_t launch_bconv_tc(const BConvTC& P, const BConvIO& io, const uint8_t* bmat, const BMatParam* bp, int N,
                            int batch, int num_sms, cudaStream_t st) {
    static bool init = false;
    if (!init) {
        cudaFuncSetAttribute(k_bconv_tc_g, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
        cudaFuncSetAttribute(k_bconv_tc_p, cudaFuncAttributeMaxDynamicSharedMemorySize, 64 * 1024);
        init = true;
    }
    const int tiles_per_entry = N / kTileM;
    const int total = tiles_per_entry * batch;
    int grid = num_sms * 2;
    if (grid > total) grid = total;
    if (bp)
        k_bconv_tc_p<<<grid, kTileM, bconv_tc_smem(P.ncols), st>>>(P, io, *bp, N, tiles_per_entry, total);
    else
        k_bconv_tc_g<<<grid, kTileM, bconv_tc_smem(P.ncols), st>>>(P, io, reinterpret_cast<const uint4*>(bmat), N,
                                                                   tiles_per_entry, total);
    return cudaGetLastError();
}

}  // namespace neo
