// ntt.cu -- negacyclic NTT / INTT for N = 2^12 and 2^16 on CUDA cores (sm_100a), FP64.
//
// Transform (the radix-16 "ten-step" NTT of L438-450 computes the same thing): a_hat[i] =
// sum_n a[n] psi^((2i+1)n), natural order in and out (Z6).  Two HBM passes (column pass,
// row pass; ntt_tables.h), each an R x R factorisation held in registers with one
// shared-memory exchange -- the four radix-R matrix stages of Fig. 9 (L448), evaluated with
// radix-2 butterflies.  Residues are FP64 values inside a pass (common.cuh "FP64 residue
// arithmetic"): Neo's observation that the FP64 units beat int8-split arithmetic for
// 36-bit words (L246-256) holds on sm_100a too, but on the CUDA cores, where a lazy FP64
// butterfly costs 8 DFMA-pipe ops and the B200 FP64 pipe runs 63 ops/clk/SM.  Values stay
// lazy (signed, |x| < 16q) inside a pass; the intermediate buffer between the two passes
// holds those doubles; the ABI-facing side of each pass holds canonical uint64.
#include "common.cuh"
#include "ntt_tables.h"
#include "ntt.h"

namespace neo {

// ------------------------------------------------------------------ in-register transforms

// Negacyclic R-point forward NTT (Cooley-Tukey, merged psi): natural in, bit-reversed out.
// tab[k] = rho^bitrev(k) (k = 1..R-1), rho a primitive 2R-th root.  |out| <= |in| + R/2... see DESIGN.
template <int R>
NEO_DEV void neg_fwd(double (&a)[R], const TWD* tab, double q) {
    int t = R;
#pragma unroll
    for (int m = 1; m < R; m <<= 1) {
        t >>= 1;
#pragma unroll
        for (int i = 0; i < m; ++i) {
            const TWD S = tab[m + i];
#pragma unroll
            for (int j = 2 * i * t; j < 2 * i * t + t; ++j) {
                const double U = a[j];
                const double V = mulc(a[j + t], S, q);
                a[j] = __dadd_rn(U, V);
                a[j + t] = __dadd_rn(U, -V);
            }
        }
    }
}

// Negacyclic R-point inverse (Gentleman-Sande, unscaled): bit-reversed in, natural out.
// tab[k] = rho^-bitrev(k).
template <int R>
NEO_DEV void neg_inv(double (&a)[R], const TWD* tab, double q) {
    int t = 1;
#pragma unroll
    for (int m = R; m > 1; m >>= 1) {
        const int h = m >> 1;
#pragma unroll
        for (int i = 0; i < h; ++i) {
            const TWD S = tab[h + i];
            const int j1 = 2 * i * t;
#pragma unroll
            for (int j = j1; j < j1 + t; ++j) {
                const double U = a[j], V = a[j + t];
                a[j] = __dadd_rn(U, V);
                a[j + t] = mulc(__dadd_rn(U, -V), S, q);
            }
        }
        t <<= 1;
    }
}

// Cyclic R-point DFT, decimation in frequency: natural in, bit-reversed out.
// tab[j] = w^j (j < R/2), w a primitive R-th root.
template <int R>
NEO_DEV void cyc_dif(double (&a)[R], const TWD* tab, double q) {
#pragma unroll
    for (int len = R / 2; len >= 1; len >>= 1) {
#pragma unroll
        for (int s = 0; s < R; s += 2 * len) {
#pragma unroll
            for (int j = 0; j < len; ++j) {
                const double U = a[s + j], V = a[s + j + len];
                a[s + j] = __dadd_rn(U, V);
                const double D = __dadd_rn(U, -V);
                a[s + j + len] = (j == 0) ? D : mulc(D, tab[j * (R / (2 * len))], q);
            }
        }
    }
}

// ------------------------------------------------------------------ column pass

constexpr int kCols = 16;     // columns per CTA (column pass)
constexpr int kRows = 16;     // rows per CTA (row pass)

template <int R>
struct ColSmem {
    static constexpr int NS = R + R * R + R / 2;        // neg, tw1, cyc
    static constexpr int NO = 2 * kCols * R;            // outer A, B for this CTA's columns
    static constexpr int XP = R * R + 1;                // odd pitch: conflict-free exchange
    static constexpr size_t bytes = (size_t)(NS + NO) * sizeof(TWD) + (size_t)kCols * XP * sizeof(double);
};

// Forward: src = canonical u64 coefficients, dst = lazy doubles tmp[i1][n2].
// Inverse: src = lazy doubles tmp[i1][n2], dst = canonical u64 coefficients.
template <int R, bool FWD>
__global__ void __launch_bounds__(kCols * R)
k_ntt_col(RowSet rs, NttArgs a) {
    using SM = ColSmem<R>;
    constexpr int C = kCols;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TWD* stab = reinterpret_cast<TWD*>(smem_raw);
    TWD* sA = stab + SM::NS;
    TWD* sB = sA + C * R;
    double* sx = reinterpret_cast<double*>(sB + C * R);

    const int k = blockIdx.y, b = blockIdx.z;
    const int lid = rs.prime[k];
    const ModQ mq = a.mods[lid];
    const double q = mq.qd;
    const TWD* ptab = a.tabd + (size_t)lid * a.tab_stride;
    const u64* __restrict__ src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * a.N;
    u64* __restrict__ dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * a.N;
    const int N2 = a.N2;
    const int tid = threadIdx.x, c = tid % C, r = tid / C;
    const int col0 = blockIdx.x * C;
    const int n2 = col0 + c;

    // element loads first (longest latency), then the constant tables
    double x[R];
    if (FWD) {
#pragma unroll
        for (int na = 0; na < R; ++na) x[na] = u2d(src[(size_t)(R * na + r) * N2 + n2]);
    } else {
        const double* s = reinterpret_cast<const double*>(src);
#pragma unroll
        for (int ib = 0; ib < R; ++ib) x[ib] = s[(size_t)(r + R * ib) * N2 + n2];
    }
    {
        const int off = FWD ? a.L.colf_neg : a.L.coli_neg;         // neg, tw1, cyc contiguous
        for (int e = tid; e < SM::NS; e += blockDim.x) stab[e] = ptab[off + e];
        const int oa = (FWD ? a.L.outf_a : a.L.outi_a) + col0 * R;
        const int ob = (FWD ? a.L.outf_b : a.L.outi_b) + col0 * R;
        for (int e = tid; e < C * R; e += blockDim.x) {
            sA[e] = ptab[oa + e];
            sB[e] = ptab[ob + e];
        }
    }
    __syncthreads();
    const TWD* NEG = stab;
    const TWD* TW1 = stab + R;
    const TWD* CYC = stab + R + R * R;
    double* S = sx + c * SM::XP;

    if (FWD) {
        neg_fwd<R>(x, NEG, q);
#pragma unroll
        for (int ia = 0; ia < R; ++ia) S[ia * R + r] = mulc(x[BitRev<R>::of(ia)], TW1[r * R + ia], q);
        __syncthreads();
#pragma unroll
        for (int nb = 0; nb < R; ++nb) x[nb] = S[r * R + nb];
        cyc_dif<R>(x, CYC, q);
        const TWD ta = sA[c * R + r];
        double* d = reinterpret_cast<double*>(dst);
#pragma unroll
        for (int ib = 0; ib < R; ++ib) {
            const double v = mulc(mulc(x[BitRev<R>::of(ib)], ta, q), sB[c * R + ib], q);
            d[(size_t)(r + R * ib) * N2 + n2] = v;
        }
    } else {
        const TWD ta = sA[c * R + r];
#pragma unroll
        for (int ib = 0; ib < R; ++ib) x[ib] = mulc(mulc(x[ib], ta, q), sB[c * R + ib], q);
        cyc_dif<R>(x, CYC, q);
#pragma unroll
        for (int nb = 0; nb < R; ++nb) S[nb * R + r] = mulc(x[BitRev<R>::of(nb)], TW1[r * R + nb], q);
        __syncthreads();
#pragma unroll
        for (int j = 0; j < R; ++j) x[j] = S[r * R + BitRev<R>::of(j)];
        neg_inv<R>(x, NEG, q);
#pragma unroll
        for (int na = 0; na < R; ++na) dst[(size_t)(R * na + r) * N2 + n2] = d2u(canon(x[na], q, mq.qinv));
    }
}

// ------------------------------------------------------------------ row pass

template <int R>
struct RowSmem {
    static constexpr int NS = R / 2 + R * R;            // cyc, tw2
    static constexpr int XP = R * R + 1;
    static constexpr int TP = kRows + 1;
    static size_t bytes(int N2) {
        size_t xb = (size_t)kRows * XP * sizeof(double), tb = (size_t)N2 * TP * sizeof(double);
        return (size_t)NS * sizeof(TWD) + (xb > tb ? xb : tb);
    }
};

// Forward: src = lazy doubles tmp[i1][n2], dst = canonical u64 a_hat[i1 + N1 i2].
// Inverse: src = canonical u64 a_hat, dst = lazy doubles tmp[i1][n2].
template <int R, bool FWD>
__global__ void __launch_bounds__(kRows * R)
k_ntt_row(RowSet rs, NttArgs a) {
    using SM = RowSmem<R>;
    constexpr int RR = kRows;
    constexpr int TP = SM::TP;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TWD* stab = reinterpret_cast<TWD*>(smem_raw);
    double* sx = reinterpret_cast<double*>(stab + SM::NS);     // exchange, then transpose buffer

    const int k = blockIdx.y, b = blockIdx.z;
    const int lid = rs.prime[k];
    const ModQ mq = a.mods[lid];
    const double q = mq.qd;
    const TWD* ptab = a.tabd + (size_t)lid * a.tab_stride;
    const u64* __restrict__ src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * a.N;
    u64* __restrict__ dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * a.N;
    const int N1 = a.N1, N2 = a.N2;
    const int tid = threadIdx.x, rho = tid / R, r = tid % R;
    const int row0 = blockIdx.x * RR;
    const int i1 = row0 + rho;

    double x[R];
    if (FWD) {
        const double* s = reinterpret_cast<const double*>(src);
#pragma unroll
        for (int na = 0; na < R; ++na) x[na] = s[(size_t)i1 * N2 + R * na + r];
    } else {
        for (int e = tid; e < N2 * RR; e += blockDim.x) {
            const int i2 = e / RR, rr = e % RR;
            sx[i2 * TP + rr] = u2d(src[(size_t)row0 + rr + (size_t)N1 * i2]);
        }
    }
    {
        const int off = FWD ? a.L.rowf_cyc : a.L.rowi_cyc;         // cyc, tw2 contiguous
        for (int e = tid; e < SM::NS; e += blockDim.x) stab[e] = ptab[off + e];
    }
    __syncthreads();
    const TWD* CYC = stab;
    const TWD* TW2 = stab + R / 2;
    double* S = sx + rho * SM::XP;

    if (FWD) {
        cyc_dif<R>(x, CYC, q);
#pragma unroll
        for (int ia = 0; ia < R; ++ia) S[ia * R + r] = mulc(x[BitRev<R>::of(ia)], TW2[r * R + ia], q);
        __syncthreads();
#pragma unroll
        for (int nb = 0; nb < R; ++nb) x[nb] = S[r * R + nb];
        cyc_dif<R>(x, CYC, q);
        __syncthreads();
#pragma unroll
        for (int ib = 0; ib < R; ++ib) sx[(r + R * ib) * TP + rho] = x[BitRev<R>::of(ib)];
        __syncthreads();
        for (int e = tid; e < N2 * RR; e += blockDim.x) {
            const int i2 = e / RR, rr = e % RR;
            dst[(size_t)row0 + rr + (size_t)N1 * i2] = d2u(canon(sx[i2 * TP + rr], q, mq.qinv));
        }
    } else {
#pragma unroll
        for (int ib = 0; ib < R; ++ib) x[ib] = sx[(r + R * ib) * TP + rho];
        cyc_dif<R>(x, CYC, q);
        __syncthreads();
#pragma unroll
        for (int nb = 0; nb < R; ++nb) S[nb * R + r] = mulc(x[BitRev<R>::of(nb)], TW2[r * R + nb], q);
        __syncthreads();
#pragma unroll
        for (int ia = 0; ia < R; ++ia) x[ia] = S[r * R + ia];
        cyc_dif<R>(x, CYC, q);
        double* d = reinterpret_cast<double*>(dst);
#pragma unroll
        for (int na = 0; na < R; ++na) d[(size_t)i1 * N2 + R * na + r] = x[BitRev<R>::of(na)];
    }
}

// ------------------------------------------------------------------ launchers

template <int R, bool FWD>
static cudaError_t launch_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, cudaStream_t st) {
    static bool init = false;
    const size_t smc = ColSmem<R>::bytes, smr = RowSmem<R>::bytes(a.N2);
    if (!init) {
        cudaFuncSetAttribute(k_ntt_col<R, FWD>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smc);
        cudaFuncSetAttribute(k_ntt_row<R, FWD>, cudaFuncAttributeMaxDynamicSharedMemorySize, 160 * 1024);
        init = true;
    }
    if (col) {
        dim3 grid(a.N2 / kCols, rs.n, batch);
        k_ntt_col<R, FWD><<<grid, kCols * R, smc, st>>>(rs, a);
    } else {
        dim3 grid(a.N1 / kRows, rs.n, batch);
        k_ntt_row<R, FWD><<<grid, kRows * R, smr, st>>>(rs, a);
    }
    return cudaGetLastError();
}

cudaError_t ntt_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st) {
    if (rs.n == 0 || batch == 0) return cudaSuccess;
    switch (a.L.R) {
        case 8: return fwd ? launch_pass<8, true>(col, rs, a, batch, st) : launch_pass<8, false>(col, rs, a, batch, st);
        case 16: return fwd ? launch_pass<16, true>(col, rs, a, batch, st) : launch_pass<16, false>(col, rs, a, batch, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace neo
