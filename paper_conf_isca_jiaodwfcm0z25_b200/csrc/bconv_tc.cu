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
// All moduli are < 2^36, so the top bytes y^(4), C_4 are < 16: D_0..3 < 12 * 1035 * 255 < 2^22,
// D_4 < 12 * 1035 * 15 < 2^18 and V = sum_b 2^(8b) D_b < 2^46.1 + 2^50 < 2^51 is an exact
// double; the epilogue is one integer sum plus one FP64 Barrett step (4 FP64 ops).
// GEMM shape per 128-coefficient tile: M = 128, K = 5*n_in <= 64 (two K=32 MMAs), and the
// targets split into parts of J = 9 (45 columns, padded to 48), all parts of a tile in one
// MMA of N = 48 * parts <= 240.  A (8 KB) is produced by the CUDA cores into shared memory in
// the SWIZZLE_NONE K-major layout, B (<= 15 KB) is loaded once per CTA, the accumulators live
// in TMEM (2 tile slots x 256 columns) and are drained with tcgen05.ld.
// D_b <= 60 * 255 * 255 < 2^22, so s32 accumulation is exact.
#include <cstdlib>

#include "bconv_tc.h"
#include "common.cuh"
#include "tc.cuh"

namespace neo {

constexpr int kTileM = 128;
constexpr int kAStages = 4;                        // A-tile ring
constexpr int kSlots = 2;                          // TMEM accumulator ring: 2 tile slots x 256 columns
constexpr int kSlotCols = 256;                     // a tile's parts at 48-column stride
constexpr int kSets = 4;                           // epilogue sets of 4 warps: set e drains parts q = e (mod 4)
constexpr int kInStages = 8;                       // TMA input ring (12 KB each)
constexpr int kPreIn = kInStages;                  // input stages issued before the setup barrier (2: 4260 KS/s, 8: 4315-4350)
constexpr int kEpiWarps = 4 * kSets;
constexpr int kThreads = (4 + kEpiWarps + 2) * 32; // producers, epilogue, MMA, TMA
constexpr size_t kInBytes = (size_t)BCTC_MAX_IN * kTileM * 8;
constexpr int kMaxJobs = BCTC_MULTI_JOBS;          // conversions fused into one launch (ModUp digits)
constexpr size_t kPartBytes = (size_t)BCTC_PART_ROWS * 64;
constexpr size_t kBAll = BCTC_MULTI_PARTS * kPartBytes;  // all jobs' B, packed (60 KB)
struct JobH {                                      // per-conversion header, staged in smem
    const u64* in;
    u64* out;
    long long in_bs, out_bs;
    int n_in, n_out, nparts, J, ncols, in_off0, use_tmap, boff;   // boff: B offset in parts
};
struct TgtC {                                      // per-target epilogue constants, staged in smem
    double t, tinv;
    long long offb;                                // out_off[t] * N * 8 (bytes)
    long long pad;
};
constexpr int kTgtRow = (BCTC_MAX_PARTS * BCTC_PART_J + 7) / 8 * 8;   // padded: parts need no clamp
constexpr int kMaxSched = 1024;                    // per-CTA tile schedule entries staged in smem
constexpr size_t kTabBytes = kMaxJobs * (sizeof(JobH) + kTgtRow * sizeof(TgtC)) + kMaxSched * 4;
constexpr size_t kSmemBytes = kAStages * kTileM * 64 + kBAll + kInStages * kInBytes + kTabBytes;
constexpr size_t kSmemAlloc = 214 * 1024;          // > half an SM: one CTA (and 512 TMEM cols) per SM
static_assert(kSmemBytes <= kSmemAlloc, "shared memory plan exceeds the allocation");
static_assert(kSlots * kSlotCols == 512, "TMEM plan");

// Warp-specialised pipeline, one persistent CTA per SM:
//   TMA (warp 21, lane 0): one 3-D tensor copy of the [n_in][128] input box of tile i+7
//   producers (warps 0-3): y = [c qhat^-1] of one coefficient (or the pre-scaled input),
//                          split into bytes, write the A row of A-stage i % 4, arrive full_a
//   MMA (warp 20, lane 0): per tile i: wait full_a / tmem_empty[i % 2]; two K = 32 MMAs of
//                          N = 48 * parts into slot i % 2; commit -> tmem_full, commit -> empty_a
//                          (a serial chain of high-latency tcgen05 / mbarrier ops: one MMA pair
//                          per tile instead of one per part halves the thread's time per tile)
//   epilogue (4 sets of 4 warps, set q % 4 drains the q-th part of the CTA): tcgen05.ld of its
//                          32 TMEM lanes x 48 columns, V = sum_b 2^(8b) D_b, one FP64 Barrett
//                          step, store; every warp arrives tmem_empty once per tile
// A tile of 36 targets is 4 parts, one per set.  Per-job / per-target constants and the tile
// schedule are staged in shared memory during setup (register-indexed reads of the large
// parameter block miss the constant cache on the critical path).
template <bool kPre, bool kLazy, class LoadB, bool kCorr = false, int NB = 5>
__device__ __forceinline__ void bconv_tc_body(const BConvTC* PJ, const BConvIO* IOJ, int njobs, LoadB loadB, int N,
                                              int tiles_per_entry, int batch, int exp,
                                              const CUtensorMap* tmaps = nullptr, const int* use_tmap = nullptr,
                                              unsigned long long* dbg = nullptr,
                                              const uint8_t* const* bglob = nullptr) {
    // NEO_BCONV_DBG trace of CTA 0: [i][0..3] producer in / A ready, MMA start / committed,
    // [i][4..5] epilogue part 0 start / last part end; row 60: waiting cycles per barrier
    unsigned long long wacc[6] = {0, 0, 0, 0, 0, 0};
    auto WAIT = [&](uint64_t* bar, uint32_t ph, int k) {
        const unsigned long long t0 = dbg ? clock64() : 0;
        tc::mbar_wait(bar, ph);
        if (dbg) wacc[k] += clock64() - t0;
    };
    auto T = [&](int i, int ev) {
        if (dbg && blockIdx.x == 0 && i < 60) dbg[i * 8 + ev] = clock64();
    };
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t* sA = smem;                                  // kAStages x (128 rows x 64 B)
    uint8_t* sB0 = smem + kAStages * kTileM * 64;        // all jobs' parts x (48 rows x 64 B), packed
    u64* sIn = reinterpret_cast<u64*>(sB0 + kBAll);      // kInStages x [n_in][128]
    JobH* sJob = reinterpret_cast<JobH*>(sIn + kInStages * BCTC_MAX_IN * kTileM);    // [job]
    TgtC* sTgt = reinterpret_cast<TgtC*>(sJob + kMaxJobs);                           // [job][target]
    uint32_t* sSched = reinterpret_cast<uint32_t*>(sTgt + kMaxJobs * kTgtRow);       // [i] -> jb | b | m-tile
    const int tiles_per_job = tiles_per_entry * batch;
    const int total_tiles = tiles_per_job * njobs;
    auto decode = [&](int tile, int& j, int& b, int& m0) {   // tile -> (conversion, batch entry, first coeff)
        j = tile / tiles_per_job;
        const int r = tile - j * tiles_per_job;
        b = r / tiles_per_entry;
        m0 = (r - b * tiles_per_entry) * kTileM;
    };
    auto tile_at = [&](int i, int& j, int& b, int& m0) {   // the CTA's i-th tile, blockIdx.x + i G
        if (i < kMaxSched) {
            const uint32_t w = sSched[i];
            j = w >> 28;
            b = (w >> 16) & 0xFFF;
            m0 = (int)(w & 0xFFFF) * kTileM;
        } else {
            decode(blockIdx.x + i * gridDim.x, j, b, m0);
        }
    };
    __shared__ uint64_t full_a[kAStages], empty_a[kAStages], tfull[kSlots], tempty[kSlots];
    __shared__ uint64_t in_full[kInStages], in_empty[kInStages];
    __shared__ uint32_t tmem_base;
    __shared__ uint64_t bar_b;                           // B matrices landed (bulk copies, bglob != null)

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int G = gridDim.x;
    unsigned long long st0 = dbg ? clock64() : 0, st1 = 0, st2 = 0;   // setup stamps (debug trace, row 61)
    if (bglob && tid == 32 * (4 + kEpiWarps + 1)) {
        // B matrices from device memory: one bulk copy per conversion, issued first so that they
        // land while the rest of the setup runs (only the MMA issuer waits for them)
        uint32_t bytes = 0;
        for (int j = 0; j < njobs; ++j) bytes += (uint32_t)(PJ[j].nparts * kPartBytes);
        tc::mbar_init(&bar_b, 1);
        tc::fence_proxy_async();
        tc::mbar_arrive_tx(&bar_b, bytes);
        for (int j = 0, bo = 0; j < njobs; bo += PJ[j].nparts, ++j)
            tc::bulk_g2s(sB0 + (size_t)bo * kPartBytes, bglob[j], (uint32_t)(PJ[j].nparts * kPartBytes), &bar_b);
    }
    const int total_run = (exp & 256) ? 0 : total_tiles;      // exp 256: setup/teardown only
    // the input ring's first stages are issued before the CTA-wide setup barrier by the TMA thread
    // itself (its barriers initialised here), so the first tiles' HBM latency overlaps the setup
    const int n_pre = (exp & 32) ? 0 : min(kPreIn, (total_run - (int)blockIdx.x + G - 1) / G);
    auto issue_in = [&](int i, int s, int jb, int b, int m0, const BConvIO& io, int n_in, int use_tm, int off0) {
        u64* dst = sIn + (size_t)s * BCTC_MAX_IN * kTileM;
        tc::mbar_arrive_tx(&in_full[s], (uint32_t)n_in * kTileM * 8);
        if (use_tm) {                      // one instruction for the [n_in][128] box
            tc::tensor_g2s_3d(dst, &tmaps[jb], m0, off0, b, &in_full[s]);
        } else {                           // each 1-D bulk copy costs ~170 issue cycles
            const u64* in = io.in + b * io.in_bstride + m0;
            for (int j = 0; j < n_in; ++j)
                tc::bulk_g2s(dst + j * kTileM, in + (size_t)io.in_off[j] * N, kTileM * 8, &in_full[s]);
        }
    };
    if (tid == 32 * (4 + kEpiWarps + 1)) {
        for (int s = 0; s < kInStages; ++s) {
            tc::mbar_init(&in_full[s], 1);
            tc::mbar_init(&in_empty[s], 4);
        }
        tc::fence_proxy_async();
        if (n_pre > 0) pdl_wait();         // the inputs are the predecessor's output
        for (int i = 0; i < n_pre; ++i) {
            int jb, b, m0;
            decode(blockIdx.x + i * G, jb, b, m0);
            issue_in(i, i, jb, b, m0, IOJ[jb], PJ[jb].n_in, use_tmap ? use_tmap[jb] : 0, IOJ[jb].in_off[0]);
        }
    }
    if (warp == 0) tc::tmem_alloc(&tmem_base, kSlots * kSlotCols);
    if (dbg) st1 = clock64();
    if (tid == 0) {
        for (int s = 0; s < kAStages; ++s) {
            tc::mbar_init(&full_a[s], 4);                // one arrival per producer warp
            tc::mbar_init(&empty_a[s], 1);
        }
        for (int s = 0; s < kSlots; ++s) {
            tc::mbar_init(&tfull[s], 1);
            tc::mbar_init(&tempty[s], kEpiWarps);        // one arrival per epilogue warp
        }
    }
    if (!bglob) {
        for (int j = 0, bo = 0; j < njobs; bo += PJ[j].nparts, ++j) {
            uint4* s4 = reinterpret_cast<uint4*>(sB0 + (size_t)bo * kPartBytes);
            const int n16 = PJ[j].nparts * (int)(kPartBytes / 16);
            for (int e = tid; e < n16; e += kThreads) s4[e] = loadB(j, e);
        }
    }
    if (tid < njobs) {
        const BConvTC& P = PJ[tid];
        const BConvIO& io = IOJ[tid];
        int bo = 0;
        for (int j = 0; j < tid; ++j) bo += PJ[j].nparts;
        sJob[tid] = JobH{io.in, io.out, io.in_bstride, io.out_bstride, P.n_in, P.n_out, P.nparts, P.J, P.ncols,
                         io.in_off[0], use_tmap ? use_tmap[tid] : 0, bo};
    }
    for (int x = tid; x < kMaxSched && blockIdx.x + x * G < total_tiles; x += kThreads) {
        int j, b, m0;
        decode(blockIdx.x + x * G, j, b, m0);
        sSched[x] = ((uint32_t)j << 28) | ((uint32_t)b << 16) | (uint32_t)(m0 / kTileM);
    }
    tc::fence_proxy_async();
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    if (dbg) st2 = clock64();
    pdl_wait();            // B matrices / TMEM / barriers were set up while the predecessor drained
    if (dbg && blockIdx.x == 0 && tid == 0) {
        dbg[61 * 8 + 0] = st0;
        dbg[61 * 8 + 1] = st1;
        dbg[61 * 8 + 2] = st2;
        dbg[61 * 8 + 3] = clock64();
    }
    pdl_trigger();
    const uint32_t tmem = tmem_base;

    if (warp < 4) {
        // ------------------------------------------------ producers
        uint8_t* arow0 = sA + (tid >> 3) * 512 + (tid & 7) * 16;   // row tid of A-stage 0
        int i = 0;
        for (int tile = blockIdx.x; tile < total_run; tile += G, ++i) {
            int jb, b, m0;
            tile_at(i, jb, b, m0);
            const int n_in = sJob[jb].n_in;
            const int si = i % kInStages, ki = i / kInStages;
            if (!(exp & 32)) WAIT(&in_full[si], ki & 1, 1);
            if (tid == 0) T(i, 0);
            const u64* src = sIn + (size_t)si * BCTC_MAX_IN * kTileM + tid;
            u64 c[BCTC_MAX_IN];
#pragma unroll
            for (int j = 0; j < BCTC_MAX_IN; ++j) c[j] = (j < n_in) ? src[j * kTileM] : 0;
            __syncwarp();
            if (lane == 0) tc::mbar_arrive(&in_empty[si]);
            uint32_t w[16];
#pragma unroll
            for (int kk = 0; kk < 16; ++kk) w[kk] = 0;
#pragma unroll
            for (int j = 0; j < BCTC_MAX_IN; ++j) {
                if (j < n_in) {
                    u64 y = c[j];
                    if (!kPre) {
                        const BConvTC& P = PJ[jb];
                        const double q = P.qin[j];
                        y = d2u(canon(mulc(u2d(c[j]), P.qhat_inv[j], q), q, P.qinv_in[j]));
                    }
                    const int bit = 40 * j, wi = bit >> 5, sh = bit & 31;
                    w[wi] |= (uint32_t)(y << sh);
                    w[wi + 1] |= (uint32_t)(y >> (32 - sh));
                    if (sh > 24) w[wi + 2] |= (uint32_t)(y >> (64 - sh));
                }
            }
            if (kCorr) {          // centred lift: u = rint(sum_j y_j / q_j) into K column 5 n_in (byte)
                double sacc = 0.0;
#pragma unroll
                for (int j = 0; j < BCTC_MAX_IN; ++j)
                    if (j < n_in) sacc = __fma_rn(u2d(c[j]), PJ[jb].qinv_in[j], sacc);
                const uint32_t u = (uint32_t)__double2int_rn(sacc);
                const int byte = 5 * n_in;
#pragma unroll
                for (int kk = 0; kk < 16; ++kk)
                    if (kk == (byte >> 2)) w[kk] |= u << (8 * (byte & 3));
            }
            const int s = i % kAStages, k = i / kAStages;
            WAIT(&empty_a[s], (k & 1) ^ 1, 2);
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
        // ------------------------------------------------ epilogue: set e drains parts q = e (mod 4)
        // the per-target constants are staged here, off the setup's critical path (the first tile's
        // accumulators are thousands of cycles away); named barrier 1 over the epilogue warps
        for (int x = tid - 128; x < njobs * kTgtRow; x += 32 * kEpiWarps) {
            const int j = x / kTgtRow, t = min(x - j * kTgtRow, PJ[j].n_out - 1);   // pad: repeat the last target
            sTgt[x] = TgtC{PJ[j].t[t], PJ[j].tinv[t], (long long)IOJ[j].out_off[t] * N * 8, 0};
        }
        asm volatile("bar.sync 1, %0;\n" ::"r"(32 * kEpiWarps) : "memory");
        const int ew = warp - 4, quarter = ew & 3, e = ew >> 2;
        const int et = quarter * 32 + lane;                  // TMEM lane = A row = coefficient
        int q = 0, i = 0;                                    // part counter, tile counter of this CTA
        for (int tile = blockIdx.x; tile < total_run; tile += G, ++i) {
            int jb, b, m0;
            tile_at(i, jb, b, m0);
            const JobH& H = sJob[jb];
            const int nparts = H.nparts;
            const int slot = i % kSlots, k = i / kSlots;
            const int p0 = (e - q) & (kSets - 1);            // my first part of this tile
            q += nparts;
            WAIT(&tfull[slot], k & 1, 3);                    // (every warp: orders its arrival below)
            if (lane == 0 && quarter == 0 && e == 0) T(i, 4);
            tc::fence_after();
            char* outb = reinterpret_cast<char*>(H.out + b * H.out_bs + m0 + et);
            if (p0 >= nparts) {
                tc::fence_before();
                __syncwarp();
                if (lane == 0) tc::mbar_arrive(&tempty[slot]);
                continue;
            }
            for (int p = p0; p < nparts; p += kSets) {
                const uint32_t trow = tmem + (uint32_t)(slot * kSlotCols + p * BCTC_PART_ROWS) + ((uint32_t)(quarter * 32) << 16);
                const int t0 = p * H.J, nt = min(H.J, H.n_out - t0);
                uint32_t v[48];
#pragma unroll
                for (int x = 0; x < 6; ++x) {
                    uint32_t (&vv)[8] = *reinterpret_cast<uint32_t (*)[8]>(&v[8 * x]);
                    tc::tmem_ld8(trow + (uint32_t)(8 * x), vv);
                }
                tc::tmem_wait_ld();
                if (p + kSets >= nparts) {                   // my last part: the slot can be refilled
                    tc::fence_before();
                    __syncwarp();
                    if (lane == 0) tc::mbar_arrive(&tempty[slot]);
                }
                const TgtC* tg = sTgt + jb * kTgtRow + t0;
                // V = sum_b 2^(8b) D_b < 2^51 assembled directly as the bits of 2^52 + V:
                // (D0 + 2^8 D1) + 2^16 D2 + 2^24 D3 as a 64-bit word, then D4 and the exponent of
                // 2^52 added to the high word (no carry: hi + D4 < 2^20).
#pragma unroll
                for (int u = 0; u < (NB == 5 ? BCTC_PART_J : BCTC_PART_ROWS / 6); ++u) {
                    const TgtC& C = tg[u];
                    const uint32_t* D = &v[NB * u];
                    u64 w = (u64)(D[0] + (D[1] << 8)) + (u64)D[2] * 65536ull;
                    w += (u64)D[3] * 16777216ull;
                    double r;
                    if (NB == 5) {
                        const double Vd = __dadd_rn(__hiloint2double((int)((uint32_t)(w >> 32) + D[4] + 0x43300000u),
                                                                     (int)(uint32_t)w), -kTwo52);
                        const double qf = __dadd_rn(__fma_rn(Vd, C.tinv, kMagic), -kMagic);
                        r = __fma_rn(-qf, C.t, Vd);                    // V mod t, |r| <= t/2 + 1 (exact)
                    } else {
                        // 48-bit targets: V = sum_b 2^(8b) D_b < 2^62 exactly in 64 bits; the quotient
                        // rint(V / t) < 2^15 from an FP64 estimate (off by < 2^-30), the remainder in
                        // integers: |r| <= t/2 + 1 < 2^48, exact as a double
                        w += ((u64)D[4] << 32) + ((u64)D[5] << 40);
                        const double qf = rint(__dmul_rn(__ull2double_rn(w), C.tinv));
                        r = (double)(long long)(w - (u64)qf * (u64)C.t);
                    }
                    if (!kLazy) r = __dadd_rn(r, r < 0.0 ? C.t : 0.0);
                    const u64 val = kLazy ? (u64)__double_as_longlong(r) : d2u(r);
                    const uint32_t ok = u < nt;
                    asm volatile("{\n\t.reg .pred p;\n\tsetp.ne.u32 p, %2, 0;\n\t@p st.global.u64 [%0], %1;\n\t}"
                                 :: "l"(outb + C.offb), "l"(val), "r"(ok) : "memory");
                }
            }
            if (lane == 0 && quarter == 0 && e == 0) T(i, 5);
        }
    } else if (warp == 4 + kEpiWarps) {
        // ------------------------------------------------ MMA issuer
        if (lane == 0) {
            const uint32_t aaddr = tc::smem_u32(sA);
            if (bglob) tc::mbar_wait(&bar_b, 0);
            int i = 0;
            for (int tile = blockIdx.x; tile < total_run; tile += G, ++i) {
                const int s = i % kAStages, k = i / kAStages;
                int jb, b, m0;
                tile_at(i, jb, b, m0);
                const JobH& H = sJob[jb];
                const uint32_t idesc = tc::idesc_u8(kTileM, H.nparts * BCTC_PART_ROWS);
                const uint32_t as = aaddr + s * (kTileM * 64);
                const int slot = i % kSlots, kq = i / kSlots;
                WAIT(&full_a[s], k & 1, 4);
                T(i, 2);
                WAIT(&tempty[slot], (kq & 1) ^ 1, 5);
                tc::fence_after();
                const uint32_t acc = tmem + (uint32_t)(slot * kSlotCols);
                const uint32_t bs = tc::smem_u32(sB0 + (size_t)H.boff * kPartBytes);
                if (!(exp & 16)) {
                    // K = 64 as two K = 32 steps (LBO = 128 B between K chunks, SBO = 512 B between row groups)
                    tc::mma_u8(acc, tc::sdesc(as, 128, 512), tc::sdesc(bs, 128, 512), idesc, 0);
                    tc::mma_u8(acc, tc::sdesc(as + 256, 128, 512), tc::sdesc(bs + 256, 128, 512), idesc, 1);
                }
                tc::commit(&tfull[slot]);
                tc::commit(&empty_a[s]);
                T(i, 3);
            }
        }
        __syncwarp();
    } else {
        // ------------------------------------------------ TMA issuer (input ring, 7 tiles ahead)
        if (lane == 0) {
            int i = n_pre;
            for (int tile = blockIdx.x + n_pre * G; tile < total_run && !(exp & 32); tile += G, ++i) {
                const int s = i % kInStages, k = i / kInStages;
                WAIT(&in_empty[s], (k & 1) ^ 1, 0);
                int jb, b, m0;
                tile_at(i, jb, b, m0);
                const JobH& H = sJob[jb];
                issue_in(i, s, jb, b, m0, IOJ[jb], H.n_in, H.use_tmap, H.in_off0);
            }
        }
        __syncwarp();
    }
    if (dbg && blockIdx.x == 0) {      // waiting cycles: TMA, producer tid 0, epilogue set 0, MMA
        if (warp == 5 + kEpiWarps && lane == 0) dbg[60 * 8 + 0] = wacc[0];
        if (tid == 0) { dbg[60 * 8 + 1] = wacc[1]; dbg[60 * 8 + 2] = wacc[2]; }
        if (warp == 4 && lane == 0) dbg[60 * 8 + 3] = wacc[3];
        if (warp == 4 + kEpiWarps && lane == 0) { dbg[60 * 8 + 4] = wacc[4]; dbg[60 * 8 + 5] = wacc[5]; }
        if (warp == 4 && lane == 0) dbg[60 * 8 + 6] = clock64();
        if (tid == 0) dbg[60 * 8 + 7] = clock64();
    }
    tc::fence_before();
    __syncthreads();
    if (warp == 0) tc::tmem_dealloc(tmem, kSlots * kSlotCols);
}

template <bool kPre, bool kLazy, bool kCorr = false, int NB = 5>
__global__ void __launch_bounds__(kThreads, 1)
k_bconv_tc_g(const __grid_constant__ BConvMulti M, int N, int tiles_per_entry, int batch, int exp) {
    auto lb = [&](int j, int e) { return reinterpret_cast<const uint4*>(M.bmat[j])[e]; };
    bconv_tc_body<kPre, kLazy, decltype(lb), kCorr, NB>(M.P, M.io, M.njobs, lb, N, tiles_per_entry, batch, exp,
                                                       M.tmap, M.use_tmap, M.dbg, M.bmat);
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
        cudaFuncSetAttribute(k_bconv_tc_g<true, false, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)kSmemAlloc);
        cudaFuncSetAttribute(k_bconv_tc_g<true, true, false, 6>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)kSmemAlloc);
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
    if (M.njobs < 1 || M.njobs > kMaxJobs) return cudaErrorInvalidValue;
    int parts = 0;
    for (int j = 0; j < M.njobs; ++j) parts += M.P[j].nparts;
    if (parts > BCTC_MULTI_PARTS) return cudaErrorInvalidValue;
    for (int j = 0; j < kMaxJobs; ++j) M.use_tmap[j] = (j < M.njobs && !no_tmap) ? make_input_tmap(M.P[j], M.io[j], N, batch, &M.tmap[j]) : 0;
    const int tiles_per_entry = N / kTileM;
    const int total = tiles_per_entry * batch * M.njobs;
    const int grid = num_sms < total ? num_sms : total;
    static const int exp = [] { const char* e = std::getenv("NEO_BCONV_EXP"); return e ? std::atoi(e) : 0; }();
    // exp != 0: timing experiments only (NEO_BCONV_EXP: 32 no TMA, 256 setup/teardown only)
    auto k = M.pre_scaled ? (M.lazy_out ? k_bconv_tc_g<true, true> : k_bconv_tc_g<true, false>)
                          : (M.lazy_out ? k_bconv_tc_g<false, true> : k_bconv_tc_g<false, false>);
    if (M.centred) {                       // KLSS Recover Limbs: pre-scaled input, canonical output only
        if (!M.pre_scaled || M.lazy_out) return cudaErrorInvalidValue;
        k = k_bconv_tc_g<true, false, true>;
    }
    for (int j = 0; j < M.njobs; ++j)
        if ((M.P[j].nb == 6) != (M.P[0].nb == 6)) return cudaErrorInvalidValue;
    if (M.P[0].nb == 6) {                  // 48-bit targets (KLSS ModUp to WordSize_T = 48)
        if (!M.pre_scaled || !M.lazy_out || M.centred) return cudaErrorInvalidValue;
        k = k_bconv_tc_g<true, true, false, 6>;
    }
    // with NEO_PDL=2 the launch may start while its predecessor drains: the setup (TMEM, B matrices,
    // barriers, schedule) runs before griddepcontrol.wait
    return launch_k_pdl(neo_pdl_bconv(), k, dim3(grid), dim3(kThreads), kSmemAlloc, st, M, N, tiles_per_entry, batch,
                        exp);
}

bool bconv_multi_fits(const BConvMulti& M, const BConvTC& P) {
    if (M.njobs >= kMaxJobs) return false;
    int parts = P.nparts;
    for (int j = 0; j < M.njobs; ++j) parts += M.P[j].nparts;
    return parts <= BCTC_MULTI_PARTS;
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
