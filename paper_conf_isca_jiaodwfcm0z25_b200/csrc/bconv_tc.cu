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
// GEMM shape per 128-coefficient tile: M = 128, K = 5*n_in <= 64 (two K=32 MMAs), and the
// targets split into one or two jobs of N = 5*J <= 128 columns.  A (8 KB) is produced by the
// CUDA cores into shared memory in the SWIZZLE_NONE K-major layout, B (<= 16 KB) is loaded
// once per CTA, the accumulators live in TMEM (4 x 128 columns) and are drained with tcgen05.ld.
// D_b <= 60 * 255 * 255 < 2^22, so s32 accumulation is exact.
#include <cstdlib>

#include "bconv_tc.h"
#include "common.cuh"
#include "tc.cuh"

namespace neo {

constexpr int kTileM = 128;
constexpr int kAStages = 4;                        // A-tile ring
constexpr int kSlots = 4;                          // TMEM accumulator ring (4 x 128 columns)
constexpr int kSlotCols = 128;                     // per half-tile job: N = 5 * J <= 128
constexpr int kInStages = 8;                       // TMA input ring (12 KB each)
constexpr int kEpiWarps = 4 * kSlots;              // one 4-warp set per TMEM slot
constexpr int kThreads = (4 + kEpiWarps + 1) * 32; // producers, epilogue, MMA
constexpr size_t kInBytes = (size_t)BCTC_MAX_IN * kTileM * 8;
constexpr int kMaxJobs = 4;                        // conversions fused into one launch (ModUp digits)
constexpr size_t kBBytes = 2 * kSlotCols * 64;     // two half-matrices per conversion
constexpr size_t kSmemBytes = kAStages * kTileM * 64 + kMaxJobs * kBBytes + kInStages * kInBytes;   // 192 KB
constexpr size_t kSmemAlloc = 200 * 1024;          // > half an SM: one CTA (and 512 TMEM cols) per SM
static_assert(kSmemBytes <= kSmemAlloc, "shared memory plan exceeds the allocation");

// Warp-specialised pipeline, one persistent CTA per SM.  A tile (128 coefficients) is split
// into `nhalf` jobs of J targets (N = 5J <= 128 columns) so that four accumulators fit in TMEM:
//   TMA (warp 0, lane 0): 1-D bulk copies of the n_in input rows of tile i+7 (1 KB each)
//   producers (warps 0-3): y = [c qhat^-1] of one coefficient, split into bytes, write the A
//                          row of A-stage i % 4, arrive full_a
//   MMA (last warp, lane 0): per job q: wait full_a / tmem_empty[q % 4]; two K = 32 MMAs
//                          into slot q % 4; commit -> tmem_full; after the tile's jobs
//                          commit -> empty_a
//   epilogue (4 sets of 4 warps, set e owns TMEM slot e): tcgen05.ld, combine the 5
//                          byte-planes, reduce mod t, store; arrive tmem_empty[e]
// Ring depths 8 (input) / 4 (A) / 4 (TMEM) absorb the mbarrier and TMA round trips.
template <bool kPre, bool kLazy, class LoadB>
__device__ __forceinline__ void bconv_tc_body(const BConvTC* PJ, const BConvIO* IOJ, int njobs, LoadB loadB, int N,
                                              int tiles_per_entry, int batch, int exp,
                                              const CUtensorMap* tmaps = nullptr, const int* use_tmap = nullptr,
                                              unsigned long long* dbg = nullptr) {
    // debug trace (CTA 0 only): [i][0] producer after in_full, [1] producer arrive full_a,
    // [2] MMA after waits, [3] MMA committed, [4] epilogue(set 0/1..) start, [5] epilogue end
    auto T = [&](int i, int ev) {
        if (dbg && blockIdx.x == 0 && i < 62) dbg[i * 8 + ev] = clock64();
    };
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t* sA = smem;                                  // kAStages x (128 rows x 64 B)
    uint8_t* sB0 = smem + kAStages * kTileM * 64;        // kMaxJobs x 2 halves x (128 rows x 64 B)
    u64* sIn = reinterpret_cast<u64*>(sB0 + kMaxJobs * kBBytes);   // kInStages x [n_in][128]
    const int tiles_per_job = tiles_per_entry * batch;
    const int total_tiles = tiles_per_job * njobs;
    auto decode = [&](int tile, int& j, int& b, int& m0) {   // tile -> (conversion, batch entry, first coeff)
        j = tile / tiles_per_job;
        const int r = tile - j * tiles_per_job;
        b = r / tiles_per_entry;
        m0 = (r - b * tiles_per_entry) * kTileM;
    };
    __shared__ uint64_t full_a[kAStages], empty_a[kAStages], tfull[kSlots], tempty[kSlots];
    __shared__ uint64_t in_full[kInStages], in_empty[kInStages];
    __shared__ uint32_t tmem_base;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int G = gridDim.x;
    auto GT = [&](int ev) {      // setup trace (row 63): globaltimer ns of CTA 0 / CTA G-1, thread 0
        if (dbg && tid == 0 && (blockIdx.x == 0 || blockIdx.x == gridDim.x - 1)) {
            unsigned long long t;
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
            dbg[63 * 8 + ev + (blockIdx.x ? 4 : 0)] = t;
            if (!blockIdx.x) dbg[62 * 8 + ev] = clock64();
        }
    };
    GT(0);
    if (warp == 0) tc::tmem_alloc(&tmem_base, kSlots * kSlotCols);
    if (tid == 0) {
        for (int s = 0; s < kAStages; ++s) {
            tc::mbar_init(&full_a[s], 4);                // one arrival per producer warp
            tc::mbar_init(&empty_a[s], 1);
        }
        for (int s = 0; s < kSlots; ++s) {
            tc::mbar_init(&tfull[s], 1);
            tc::mbar_init(&tempty[s], 4);                // one arrival per warp of the set
        }
        for (int s = 0; s < kInStages; ++s) {
            tc::mbar_init(&in_full[s], 1);
            tc::mbar_init(&in_empty[s], 4);
        }
    }
    for (int j = 0; j < njobs; ++j) {
        uint4* s4 = reinterpret_cast<uint4*>(sB0 + j * kBBytes);
        const int n16 = PJ[j].nhalf * kSlotCols * 4;    // 16-byte chunks (halves padded to 128 rows)
        for (int e = tid; e < n16; e += kThreads) s4[e] = loadB(j, e);
    }
    tc::fence_proxy_async();
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    GT(1);
    pdl_wait();            // B matrices / TMEM / barriers were set up while the predecessor drained
    pdl_trigger();
    GT(2);
    const uint32_t tmem = tmem_base;
    const int total_run = (exp & 256) ? 0 : total_tiles;      // exp 256: setup/teardown only

    auto tma_issue = [&](int i) {
        const int tile = blockIdx.x + i * G;
        if (tile >= total_run || (exp & 32)) return;
        const int s = i % kInStages, k = i / kInStages;
        tc::mbar_wait(&in_empty[s], (k & 1) ^ 1);
        int jb, b, m0;
        decode(tile, jb, b, m0);
        const BConvTC& P = PJ[jb];
        const BConvIO& io = IOJ[jb];
        const u64* in = io.in + b * io.in_bstride + m0;
        u64* dst = sIn + (size_t)s * BCTC_MAX_IN * kTileM;
        tc::mbar_arrive_tx(&in_full[s], (uint32_t)P.n_in * kTileM * 8);
        if (use_tmap && use_tmap[jb])      // one instruction for the [n_in][128] box
            tc::tensor_g2s_3d(dst, &tmaps[jb], m0, io.in_off[0], b, &in_full[s]);
        else                               // each 1-D bulk copy costs ~170 issue cycles
            for (int j = 0; j < P.n_in; ++j)
                tc::bulk_g2s(dst + j * kTileM, in + (size_t)io.in_off[j] * N, kTileM * 8, &in_full[s]);
    };

    if (warp < 4) {
        // ------------------------------------------------ producers (+ TMA issue on thread 0)
        if (tid == 0)
            for (int i = 0; i < kInStages - 1; ++i) {
                tma_issue(i);
                if (dbg && blockIdx.x == 0 && i < 3) dbg[62 * 8 + 4 + i] = clock64();
            }
        uint8_t* arow0 = sA + (tid >> 3) * 512 + (tid & 7) * 16;   // row tid of A-stage 0
        int i = 0;
        for (int tile = blockIdx.x; tile < total_run; tile += G, ++i) {
            if (tid == 0) tma_issue(i + kInStages - 1);
            int jb, b, m0;
            decode(tile, jb, b, m0);
            const BConvTC& P = PJ[jb];
            const int si = i % kInStages, ki = i / kInStages;
            if (!(exp & 32)) tc::mbar_wait(&in_full[si], ki & 1);
            if (tid == 0) T(i, 0);
            const u64* src = sIn + (size_t)si * BCTC_MAX_IN * kTileM + tid;
            u64 c[BCTC_MAX_IN];
#pragma unroll
            for (int j = 0; j < BCTC_MAX_IN; ++j) c[j] = (j < P.n_in) ? src[j * kTileM] : 0;
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&in_empty[si]);
            uint32_t w[16];
#pragma unroll
            for (int kk = 0; kk < 16; ++kk) w[kk] = 0;
#pragma unroll
            for (int j = 0; j < BCTC_MAX_IN; ++j) {
                if (j < P.n_in) {
                    const double q = P.qin[j];
                    const u64 y = kPre ? c[j] : d2u(canon(mulc(u2d(c[j]), P.qhat_inv[j], q), q, P.qinv_in[j]));
                    const int bit = 40 * j, wi = bit >> 5, sh = bit & 31;
                    w[wi] |= (uint32_t)(y << sh);
                    w[wi + 1] |= (uint32_t)(y >> (32 - sh));
                    if (sh > 24) w[wi + 2] |= (uint32_t)(y >> (64 - sh));
                }
            }
            const int s = i % kAStages, k = i / kAStages;
            tc::mbar_wait(&empty_a[s], (k & 1) ^ 1);
            uint8_t* arow = arow0 + s * (kTileM * 64);
#pragma unroll
            for (int cc = 0; cc < 4; ++cc)
                *reinterpret_cast<uint4*>(arow + cc * 128) = make_uint4(w[4 * cc], w[4 * cc + 1], w[4 * cc + 2], w[4 * cc + 3]);
            tc::fence_proxy_async();
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&full_a[s]);
            if (tid == 0) T(i, 1);
        }
    } else if (warp < 4 + kEpiWarps) {
        // ------------------------------------------------ epilogue: set e owns TMEM slot e
        const int ew = warp - 4, quarter = ew & 3, e = ew >> 2;
        const int et = quarter * 32 + lane;                  // TMEM lane = A row = coefficient
        const uint32_t trow = tmem + (uint32_t)(e * kSlotCols) + ((uint32_t)(quarter * 32) << 16);
        int q = 0;                                           // job counter of this CTA
        for (int tile = blockIdx.x; tile < total_run; tile += G) {
            int jb, b, m0;
            decode(tile, jb, b, m0);
            const BConvTC& P = PJ[jb];
            for (int h = 0; h < P.nhalf; ++h, ++q) {
                if ((q % kSlots) != e) continue;
                const int k = q / kSlots;
                const BConvIO& io = IOJ[jb];
                const int t0 = h * P.J, t1 = min(t0 + P.J, P.n_out);
                tc::mbar_wait(&tfull[e], k & 1);
                if (lane == 0 && quarter == 0 && h == 0) T(q / P.nhalf, 4);
                tc::fence_after();
                u64* outb = io.out + b * io.out_bstride + m0 + et;
                // 8 targets per group, branch-free so the 8 FP64 chains interleave; the ragged
                // last group re-reads its last valid column and predicates the stores.
                for (int g = t0; g < t1; g += 8) {
                    uint32_t v[40];
#pragma unroll
                    for (int x = 0; x < 5; ++x) {
                        uint32_t (&vv)[8] = *reinterpret_cast<uint32_t (*)[8]>(&v[8 * x]);
                        tc::tmem_ld8(trow + (uint32_t)(5 * (g - t0) + 8 * x), vv);
                    }
                    tc::tmem_wait_ld();
                    double r[8];
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        const int t = min(g + u, t1 - 1);
                        const uint32_t* D = &v[5 * u];
                        const u64 lo = (u64)D[0] + ((u64)D[1] << 8) + ((u64)D[2] << 16);     // < 2^39
                        const u64 hi = (u64)D[3] + ((u64)D[4] << 8);                          // < 2^31
                        const double tq = P.t[t];
                        r[u] = __dadd_rn(u2d(lo), mulc(u2d(hi), P.c24[t], tq));              // == V (mod t)
                        if (!kLazy) r[u] = canon(r[u], tq, P.tinv[t]);
                    }
#pragma unroll
                    for (int u = 0; u < 8; ++u) {
                        const int t = g + u;
                        const u64 val = kLazy ? (u64)__double_as_longlong(r[u]) : d2u(r[u]);
                        if (t < t1) outb[(size_t)io.out_off[t] * N] = val;
                    }
                }
                tc::fence_before();
                __syncwarp();
                if (lane == 0) tc::mbar_arrive(&tempty[e]);
                if (lane == 0 && quarter == 0 && h == P.nhalf - 1) T(q / P.nhalf, 5);
            }
        }
    } else {
        // ------------------------------------------------ MMA issuer
        if (lane == 0) {
            const uint32_t aaddr = tc::smem_u32(sA);
            int i = 0, q = 0;
            for (int tile = blockIdx.x; tile < total_run; tile += G, ++i) {
                const int s = i % kAStages, k = i / kAStages;
                int jb, b, m0;
                decode(tile, jb, b, m0);
                const BConvTC& P = PJ[jb];
                const uint32_t idesc = tc::idesc_u8(kTileM, P.ncols);
                const uint32_t as = aaddr + s * (kTileM * 64);
                tc::mbar_wait(&full_a[s], k & 1);
                T(i, 2);
                for (int h = 0; h < P.nhalf; ++h, ++q) {
                    const int slot = q % kSlots, kq = q / kSlots;
                    tc::mbar_wait(&tempty[slot], (kq & 1) ^ 1);
                    tc::fence_after();
                    const uint32_t acc = tmem + (uint32_t)(slot * kSlotCols);
                    const uint32_t bs = tc::smem_u32(sB0 + jb * kBBytes + h * (kSlotCols * 64));
                    {
                        // K = 64 as two K = 32 steps (LBO = 128 B between K chunks, SBO = 512 B between row groups)
                        tc::mma_u8(acc, tc::sdesc(as, 128, 512), tc::sdesc(bs, 128, 512), idesc, 0);
                        tc::mma_u8(acc, tc::sdesc(as + 256, 128, 512), tc::sdesc(bs + 256, 128, 512), idesc, 1);
                    }
                    tc::commit(&tfull[slot]);
                }
                tc::commit(&empty_a[s]);
                T(i, 3);
            }
        }
        __syncwarp();
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc(tmem, kSlots * kSlotCols);
    GT(3);
}

template <bool kPre, bool kLazy>
__global__ void __launch_bounds__(kThreads, 1)
k_bconv_tc_g(const __grid_constant__ BConvMulti M, int N, int tiles_per_entry, int batch, int exp) {
    bconv_tc_body<kPre, kLazy>(M.P, M.io, M.njobs,
                               [&](int j, int e) { return reinterpret_cast<const uint4*>(M.bmat[j])[e]; }, N,
                               tiles_per_entry, batch, exp, M.tmap, M.use_tmap, M.dbg);
}

__global__ void __launch_bounds__(kThreads, 1)
k_bconv_tc_p(const __grid_constant__ BConvTC P, const __grid_constant__ BConvIO io,
             const __grid_constant__ BMatParam B, int N, int tiles_per_entry, int batch) {
    bconv_tc_body<false, false>(&P, &io, 1, [&](int, int e) { return B.d[e]; }, N, tiles_per_entry, batch, 0);
}

size_t bconv_tc_smem(int) { return kSmemAlloc; }

static void bconv_tc_init() {
    static bool init = false;
    if (!init) {
        cudaFuncSetAttribute(k_bconv_tc_g<false, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemAlloc);
        cudaFuncSetAttribute(k_bconv_tc_g<false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemAlloc);
        cudaFuncSetAttribute(k_bconv_tc_g<true, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemAlloc);
        cudaFuncSetAttribute(k_bconv_tc_g<true, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemAlloc);
        cudaFuncSetAttribute(k_bconv_tc_p, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmemAlloc);
        init = true;
    }
}

// cuTensorMapEncodeTiled through the runtime's driver entry point (no -lcuda link dependency)
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
static EncodeTiledFn encode_tiled() {
    static EncodeTiledFn fn = [] {
        void* p = nullptr;
        cudaDriverEntryPointQueryResult q;
        if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &p, cudaEnableDefault, &q) != cudaSuccess ||
            q != cudaDriverEntryPointSuccess)
            p = nullptr;
        return reinterpret_cast<EncodeTiledFn>(p);
    }();
    return fn;
}

// 3-D map over job j's input: dim0 = coefficient (N), dim1 = limb row, dim2 = batch entry;
// box = one tile {128, n_in, 1}.  Needs the input rows of the job to be consecutive.
static bool make_input_tmap(const BConvTC& P, const BConvIO& io, int N, int batch, CUtensorMap* map) {
    EncodeTiledFn enc = encode_tiled();
    if (!enc || P.n_in < 1) return false;
    for (int i = 1; i < P.n_in; ++i)
        if (io.in_off[i] != io.in_off[0] + i) return false;
    const long long rows = io.in_off[0] + P.n_in;
    if (batch > 1 && rows * N > io.in_bstride) return false;
    if ((reinterpret_cast<uintptr_t>(io.in) & 15) != 0) return false;
    const cuuint64_t dim[3] = {(cuuint64_t)N, (cuuint64_t)rows, (cuuint64_t)batch};
    const cuuint64_t stride[2] = {(cuuint64_t)N * 8, (cuuint64_t)(batch > 1 ? io.in_bstride : rows * N) * 8};
    const cuuint32_t box[3] = {(cuuint32_t)kTileM, (cuuint32_t)P.n_in, 1};
    const cuuint32_t estr[3] = {1, 1, 1};
    return enc(map, CU_TENSOR_MAP_DATA_TYPE_UINT64, 3, const_cast<u64*>(io.in), dim, stride, box, estr,
               CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_NONE, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
               CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE) == CUDA_SUCCESS;
}

cudaError_t launch_bconv_tc(const BConvMulti& M0, int N, int batch, int num_sms, cudaStream_t st) {
    bconv_tc_init();
    BConvMulti M = M0;
    static const bool no_tmap = [] { const char* e = std::getenv("NEO_BCONV_TMAP"); return e && e[0] == '0'; }();
    for (int j = 0; j < 4; ++j) M.use_tmap[j] = (j < M.njobs && !no_tmap) ? make_input_tmap(M.P[j], M.io[j], N, batch, &M.tmap[j]) : 0;
    const int tiles_per_entry = N / kTileM;
    const int total = tiles_per_entry * batch * M.njobs;
    const int grid = num_sms < total ? num_sms : total;
    static const int exp = [] { const char* e = std::getenv("NEO_BCONV_EXP"); return e ? std::atoi(e) : 0; }();
    // exp != 0: timing experiments only (NEO_BCONV_EXP: 32 no TMA, 256 setup/teardown only)
    auto k = M.pre_scaled ? (M.lazy_out ? k_bconv_tc_g<true, true> : k_bconv_tc_g<true, false>)
                          : (M.lazy_out ? k_bconv_tc_g<false, true> : k_bconv_tc_g<false, false>);
    return launch_k(k, dim3(grid), dim3(kThreads), kSmemAlloc, st, M, N, tiles_per_entry, batch, exp);
}

cudaError_t launch_bconv_tc_param(const BConvTC& P, const BConvIO& io, const BMatParam& bp, int N, int batch,
                                  int num_sms, cudaStream_t st) {
    bconv_tc_init();
    const int tiles_per_entry = N / kTileM;
    const int total = tiles_per_entry * batch;
    const int grid = num_sms < total ? num_sms : total;
    return launch_k(k_bconv_tc_p, dim3(grid), dim3(kThreads), kSmemAlloc, st, P, io, bp, N, tiles_per_entry, batch);
}

}  // namespace neo
