// ntt.cu -- negacyclic NTT / INTT for N = 2^12 and 2^16 on CUDA cores (sm_100a).
//
// Transform (radix-16 "ten-step" NTT of L438-450 computes the same thing): a_hat[i] =
// sum_n a[n] psi^((2i+1)n), natural order in and out (Z6).  Two HBM passes (column pass,
// row pass; see ntt_tables.h), each an R x R factorisation held in registers with one
// shared-memory exchange -- i.e. four radix-R matrix stages as in Fig. 9 (L448) but with
// radix-2 butterflies inside each R-point stage instead of DFT-matrix products: on sm_100a
// the butterfly form needs fewer int32 ALU instructions than the int8-split DFT GEMM's
// modular epilogue.
#include "common.cuh"
#include "ntt_tables.h"
#include "ntt.h"

namespace neo {

// ------------------------------------------------------------------ in-register transforms

// Negacyclic R-point forward NTT (Cooley-Tukey, merged psi): natural in, bit-reversed out.
// tab[k] = rho^bitrev(k) (k = 1..R-1), rho a primitive 2R-th root.
template <int R>
NEO_DEV void neg_fwd(u64 (&a)[R], const TW* tab, u64 q) {
    int t = R;
#pragma unroll
    for (int m = 1; m < R; m <<= 1) {
        t >>= 1;
#pragma unroll
        for (int i = 0; i < m; ++i) {
            const TW S = tab[m + i];
#pragma unroll
            for (int j = 2 * i * t; j < 2 * i * t + t; ++j) {
                u64 U = a[j];
                u64 V = shoup(a[j + t], S, q);
                a[j] = add_mod(U, V, q);
                a[j + t] = sub_mod(U, V, q);
            }
        }
    }
}

// Negacyclic R-point inverse (Gentleman-Sande, unscaled): bit-reversed in, natural out.
// tab[k] = rho^-bitrev(k).
template <int R>
NEO_DEV void neg_inv(u64 (&a)[R], const TW* tab, u64 q) {
    int t = 1;
#pragma unroll
    for (int m = R; m > 1; m >>= 1) {
        const int h = m >> 1;
#pragma unroll
        for (int i = 0; i < h; ++i) {
            const TW S = tab[h + i];
            const int j1 = 2 * i * t;
#pragma unroll
            for (int j = j1; j < j1 + t; ++j) {
                u64 U = a[j], V = a[j + t];
                a[j] = add_mod(U, V, q);
                a[j + t] = shoup(U + q - V, S, q);
            }
        }
        t <<= 1;
    }
}

// Cyclic R-point DFT, decimation in frequency: natural in, bit-reversed out.
// tab[j] = w^j (j < R/2), w a primitive R-th root.
template <int R>
NEO_DEV void cyc_dif(u64 (&a)[R], const TW* tab, u64 q) {
#pragma unroll
    for (int len = R / 2; len >= 1; len >>= 1) {
#pragma unroll
        for (int s = 0; s < R; s += 2 * len) {
#pragma unroll
            for (int j = 0; j < len; ++j) {
                u64 U = a[s + j], V = a[s + j + len];
                a[s + j] = add_mod(U, V, q);
                if (j == 0)
                    a[s + j + len] = sub_mod(U, V, q);
                else
                    a[s + j + len] = shoup(U + q - V, tab[j * (R / (2 * len))], q);
            }
        }
    }
}

// ------------------------------------------------------------------ column pass

constexpr int kCols = 16;     // columns per CTA (column pass)
constexpr int kRows = 16;     // rows per CTA (row pass)

template <int R>
__global__ void __launch_bounds__(kCols * R)
k_ntt_col(RowSet rs, NttArgs a, int fwd) {
    constexpr int C = kCols;
    constexpr int NS = R + R * R + R / 2;
    constexpr int XP = R * R + 1;                   // odd pitch: conflict-free u64 exchange
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TW* stab = reinterpret_cast<TW*>(smem_raw);
    u64* sx = reinterpret_cast<u64*>(stab + NS);

    const int k = blockIdx.y, b = blockIdx.z;
    const int lid = rs.prime[k];
    const u64 q = a.mods[lid].q;
    const TW* ptab = a.tab + (size_t)lid * a.tab_stride;
    const u64* __restrict__ src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * a.N;
    u64* __restrict__ dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * a.N;
    const int N2 = a.N2;
    const int tid = threadIdx.x, c = tid % C, r = tid / C;
    const int n2 = blockIdx.x * C + c;

    const int off = fwd ? a.L.colf_neg : a.L.coli_neg;   // neg, tw1, cyc are contiguous
    for (int e = tid; e < NS; e += blockDim.x) stab[e] = ptab[off + e];
    __syncthreads();
    const TW* NEG = stab;
    const TW* TW1 = stab + R;
    const TW* CYC = stab + R + R * R;
    u64* S = sx + c * XP;

    u64 x[R], y[R];
    if (fwd) {
#pragma unroll
        for (int na = 0; na < R; ++na) x[na] = src[(size_t)(R * na + r) * N2 + n2];
        neg_fwd<R>(x, NEG, q);
#pragma unroll
        for (int ia = 0; ia < R; ++ia) y[ia] = shoup(x[BitRev<R>::of(ia)], TW1[r * R + ia], q);
#pragma unroll
        for (int ia = 0; ia < R; ++ia) S[ia * R + r] = y[ia];
        __syncthreads();
#pragma unroll
        for (int nb = 0; nb < R; ++nb) x[nb] = S[r * R + nb];
        cyc_dif<R>(x, CYC, q);
        const TW* A = ptab + a.L.outf_a + n2 * R;
        const TW* B = ptab + a.L.outf_b + n2 * R;
        const TW ta = A[r];
#pragma unroll
        for (int ib = 0; ib < R; ++ib) {
            u64 v = shoup(shoup(x[BitRev<R>::of(ib)], ta, q), B[ib], q);
            dst[(size_t)(r + R * ib) * N2 + n2] = v;
        }
    } else {
        const TW* A = ptab + a.L.outi_a + n2 * R;
        const TW* B = ptab + a.L.outi_b + n2 * R;
        const TW ta = A[r];
#pragma unroll
        for (int ib = 0; ib < R; ++ib) {
            u64 v = src[(size_t)(r + R * ib) * N2 + n2];
            x[ib] = shoup(shoup(v, ta, q), B[ib], q);
        }
        cyc_dif<R>(x, CYC, q);
#pragma unroll
        for (int nb = 0; nb < R; ++nb) y[nb] = shoup(x[BitRev<R>::of(nb)], TW1[r * R + nb], q);
#pragma unroll
        for (int nb = 0; nb < R; ++nb) S[nb * R + r] = y[nb];
        __syncthreads();
#pragma unroll
        for (int j = 0; j < R; ++j) x[j] = S[r * R + BitRev<R>::of(j)];
        neg_inv<R>(x, NEG, q);
#pragma unroll
        for (int na = 0; na < R; ++na) dst[(size_t)(R * na + r) * N2 + n2] = x[na];
    }
}

// ------------------------------------------------------------------ row pass

template <int R>
__global__ void __launch_bounds__(kRows * R)
k_ntt_row(RowSet rs, NttArgs a, int fwd) {
    constexpr int RR = kRows;
    constexpr int NS = R / 2 + R * R;
    constexpr int XP = R * R + 1;
    constexpr int TP = RR + 1;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    TW* stab = reinterpret_cast<TW*>(smem_raw);
    u64* sx = reinterpret_cast<u64*>(stab + NS);     // exchange, then transpose buffer

    const int k = blockIdx.y, b = blockIdx.z;
    const int lid = rs.prime[k];
    const u64 q = a.mods[lid].q;
    const TW* ptab = a.tab + (size_t)lid * a.tab_stride;
    const u64* __restrict__ src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * a.N;
    u64* __restrict__ dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * a.N;
    const int N1 = a.N1, N2 = a.N2;
    const int tid = threadIdx.x, rho = tid / R, r = tid % R;
    const int row0 = blockIdx.x * RR;
    const int i1 = row0 + rho;

    const int off = fwd ? a.L.rowf_cyc : a.L.rowi_cyc;   // cyc, tw2 contiguous
    for (int e = tid; e < NS; e += blockDim.x) stab[e] = ptab[off + e];
    const TW* CYC = stab;
    const TW* TW2 = stab + R / 2;
    u64* S = sx + rho * XP;

    u64 x[R], y[R];
    if (fwd) {
        __syncthreads();
#pragma unroll
        for (int na = 0; na < R; ++na) x[na] = src[(size_t)i1 * N2 + R * na + r];
        cyc_dif<R>(x, CYC, q);
#pragma unroll
        for (int ia = 0; ia < R; ++ia) y[ia] = shoup(x[BitRev<R>::of(ia)], TW2[r * R + ia], q);
#pragma unroll
        for (int ia = 0; ia < R; ++ia) S[ia * R + r] = y[ia];
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
            dst[(size_t)row0 + rr + (size_t)N1 * i2] = sx[i2 * TP + rr];
        }
    } else {
        for (int e = tid; e < N2 * RR; e += blockDim.x) {
            const int i2 = e / RR, rr = e % RR;
            sx[i2 * TP + rr] = src[(size_t)row0 + rr + (size_t)N1 * i2];
        }
        __syncthreads();
#pragma unroll
        for (int ib = 0; ib < R; ++ib) x[ib] = sx[(r + R * ib) * TP + rho];
        cyc_dif<R>(x, CYC, q);
#pragma unroll
        for (int nb = 0; nb < R; ++nb) y[nb] = shoup(x[BitRev<R>::of(nb)], TW2[r * R + nb], q);
        __syncthreads();
#pragma unroll
        for (int nb = 0; nb < R; ++nb) S[nb * R + r] = y[nb];
        __syncthreads();
#pragma unroll
        for (int ia = 0; ia < R; ++ia) x[ia] = S[r * R + ia];
        cyc_dif<R>(x, CYC, q);
#pragma unroll
        for (int na = 0; na < R; ++na) dst[(size_t)i1 * N2 + R * na + r] = x[BitRev<R>::of(na)];
    }
}

// ------------------------------------------------------------------ launchers

static size_t col_smem(int R) { return (size_t)(R + R * R + R / 2) * sizeof(TW) + (size_t)kCols * (R * R + 1) * 8; }
static size_t row_smem(int R, int N2) {
    size_t xb = (size_t)kRows * (R * R + 1) * 8, tb = (size_t)N2 * (kRows + 1) * 8;
    return (size_t)(R / 2 + R * R) * sizeof(TW) + (xb > tb ? xb : tb);
}

template <int R>
static cudaError_t launch_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd,
                               cudaStream_t st) {
    static bool init = false;
    size_t sm = col ? col_smem(R) : row_smem(R, a.N2);
    if (!init) {
        cudaFuncSetAttribute(k_ntt_col<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)col_smem(R));
        cudaFuncSetAttribute(k_ntt_row<R>, cudaFuncAttributeMaxDynamicSharedMemorySize, 200 * 1024);
        init = true;
    }
    if (col) {
        dim3 grid(a.N2 / kCols, rs.n, batch);
        k_ntt_col<R><<<grid, kCols * R, sm, st>>>(rs, a, fwd ? 1 : 0);
    } else {
        dim3 grid(a.N1 / kRows, rs.n, batch);
        k_ntt_row<R><<<grid, kRows * R, sm, st>>>(rs, a, fwd ? 1 : 0);
    }
    return cudaGetLastError();
}

cudaError_t ntt_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st) {
    if (rs.n == 0 || batch == 0) return cudaSuccess;
    switch (a.L.R) {
        case 8: return launch_pass<8>(col, rs, a, batch, fwd, st);
        case 16: return launch_pass<16>(col, rs, a, batch, fwd, st);
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace neo
