// klss.cu -- KLSS key-switching kernels (Neo's default method, L155-180; readings K1-K6 in
// DESIGN.md): the inner product over the T basis (Alg. 3 / Alg. 4) and Recover Limbs.
#include <algorithm>

#include "klss.h"

namespace neo {

// 36-bit x 36-bit products as four 18-bit x 18-bit IMADs (32x32->64) into three 64-bit partial
// sums (the CUDA-core BConv's scheme): sum_j x_j e_j = A + 2^18 Bm + 2^36 C exactly.
NEO_DEV void mac18(u64& A, u64& Bm, u64& C, unsigned xl, unsigned xh, unsigned el, unsigned eh) {
    A += (u64)xl * el;
    Bm += (u64)xl * eh + (u64)xh * el;
    C += (u64)xh * eh;
}
NEO_DEV u64 reduce18(u64 A, u64 Bm, u64 C, ModQ m) {       // A, Bm, C < 2^41 (<= 16 terms)
    const u64 t = A + (Bm << 18);
    const u64 lo = t + (C << 36);
    const u64 hi = (C >> 28) + (t < A) + (lo < t);
    return barrett_reduce(hi, lo, m);
}

// IP on CUDA cores (the paper's CUDA-core IP mapping, L488: its beta x beta~ products are far
// too small for a tensor-core tile).  One thread per (coefficient n, T limb k, group i): a warp
// is 32 consecutive coefficients of one group, so every key plane access is a coalesced
// 128-byte (32-bit plane) / 32-byte (8-bit plane) segment, and the 8 group warps of a CTA read
// the same digit values (L1 hits).  The 2 x beta key words of the thread stay in registers
// while the batch is walked: the key (the dominant traffic, 5 bytes per residue) is read once.
constexpr int KLSS_IP_W = 32;

template <int BETA>
__global__ void __launch_bounds__(256, 3)
k_klss_ip(const __grid_constant__ KlssIpArgs A, int batch) {
    pdl_wait();
    const int gi = threadIdx.y;
    if (gi >= A.n_groups) return;
    const int n = blockIdx.x * KLSS_IP_W + threadIdx.x;
    const int k = blockIdx.y, i = A.group[gi];
    const ModQ m = A.mods[A.t0 + k];
    const size_t NK = (size_t)A.alpha_p * A.N;
    const size_t col = (size_t)k * A.N + n;
    unsigned el[2][BETA], eh[2][BETA];
#pragma unroll
    for (int c = 0; c < 2; ++c) {
        const size_t kb = (size_t)(c * A.beta_t + i) * A.dnum * NK + col;
#pragma unroll
        for (int j = 0; j < BETA; ++j) {
            const size_t o = kb + (size_t)j * NK;
            const u64 e = (u64)A.key_lo[o] | ((u64)A.key_hi[o] << 32);
            el[c][j] = (unsigned)(e & 0x3FFFF);
            eh[c][j] = (unsigned)(e >> 18);
        }
    }
    for (int b = 0; b < batch; ++b) {
        const u64* up = A.up + (size_t)b * A.beta * NK + col;
        u64 a0 = 0, a1 = 0, a2 = 0, c0 = 0, c1 = 0, c2 = 0;
#pragma unroll
        for (int j = 0; j < BETA; ++j) {
            const u64 x = up[(size_t)j * NK];
            const unsigned xl = (unsigned)(x & 0x3FFFF), xh = (unsigned)(x >> 18);
            mac18(a0, a1, a2, xl, xh, el[0][j], eh[0][j]);
            mac18(c0, c1, c2, xl, xh, el[1][j], eh[1][j]);
        }
        u64* acc = A.acc + (size_t)(b * 2) * A.beta_t * NK + (size_t)i * NK + col;
        acc[0] = reduce18(a0, a1, a2, m);
        acc[(size_t)A.beta_t * NK] = reduce18(c0, c1, c2, m);
    }
}

// WordSize_T = 48 (Table 4 Set-C, L511): residues and key words < 2^48 split into 24-bit halves,
// so every product is four 24 x 24-bit IMAD.WIDE.U32 multiply-adds into three 64-bit partial sums
// (sum_j x_j e_j = A + 2^24 Bm + 2^48 C, A, C < 12 * 2^48 and Bm < 24 * 2^48: no overflow for
// beta <= 12), and ONE reduction per output: X < 2^101 via an FP64 quotient estimate
// qf = rint(X / t) (|qf - X / t| < 4), the remainder X - qf t exactly in signed 64-bit
// arithmetic (|.| < 5 t < 2^51) and at most four corrections each way.  Karatsuba: the middle
// sum is S - A - C with S = sum (xl + xh)(el + eh) < 12 * 2^50, so three IMAD.WIDE per product.
NEO_DEV void mac24k(u64& A, u64& S, u64& C, unsigned xl, unsigned xh, unsigned xs, unsigned el, unsigned eh,
                    unsigned es) {
    A += (u64)xl * el;
    S += (u64)xs * es;
    C += (u64)xh * eh;
}
NEO_DEV u64 reduce24(u64 A, u64 Bm, u64 C, ModQ m) {
    const double Xd = __fma_rn((double)C, 281474976710656.0, __fma_rn((double)Bm, 16777216.0, (double)A));
    const u64 qf = (u64)rint(Xd * m.qinv);
    long long r = (long long)(A + (Bm << 24) + (C << 48) - qf * m.q);   // low 64 bits; true |r| < 2^51
    const long long q = (long long)m.q;
#pragma unroll
    for (int i = 0; i < 4; ++i) r += (r < 0) ? q : 0;
#pragma unroll
    for (int i = 0; i < 4; ++i) r -= (r >= q) ? q : 0;
    return (u64)r;
}

template <int BETA>
__global__ void __launch_bounds__(256, 3)
k_klss_ip48(const __grid_constant__ KlssIpArgs A, int batch) {
    pdl_wait();
    const int gi = threadIdx.y;
    if (gi >= A.n_groups) return;
    const int n = blockIdx.x * KLSS_IP_W + threadIdx.x;
    const int k = blockIdx.y, i = A.group[gi];
    const ModQ m = A.mods[A.t0 + k];
    const size_t NK = (size_t)A.alpha_p * A.N;
    const size_t col = (size_t)k * A.N + n;
    const uint16_t* hi16 = reinterpret_cast<const uint16_t*>(A.key_hi);
    unsigned el[2][BETA], eh[2][BETA];
#pragma unroll
    for (int c = 0; c < 2; ++c) {
        const size_t kb = (size_t)(c * A.beta_t + i) * A.dnum * NK + col;
#pragma unroll
        for (int j = 0; j < BETA; ++j) {
            const size_t o = kb + (size_t)j * NK;
            const unsigned lo = A.key_lo[o], hi = hi16[o];
            el[c][j] = lo & 0xFFFFFFu;
            eh[c][j] = (lo >> 24) | (hi << 8);
        }
    }
    for (int b = 0; b < batch; ++b) {
        const u64* up = A.up + (size_t)b * A.beta * NK + col;
        u64 x[BETA];
#pragma unroll
        for (int j = 0; j < BETA; ++j) x[j] = up[(size_t)j * NK];
        u64 a0 = 0, s0 = 0, c0 = 0, a1 = 0, s1 = 0, c1 = 0;
#pragma unroll
        for (int j = 0; j < BETA; ++j) {
            const unsigned xl = (unsigned)x[j] & 0xFFFFFFu, xh = (unsigned)(x[j] >> 24);
            mac24k(a0, s0, c0, xl, xh, xl + xh, el[0][j], eh[0][j], el[0][j] + eh[0][j]);
            mac24k(a1, s1, c1, xl, xh, xl + xh, el[1][j], eh[1][j], el[1][j] + eh[1][j]);
        }
        u64* acc = A.acc + (size_t)(b * 2) * A.beta_t * NK + (size_t)i * NK + col;
        acc[0] = reduce24(a0, s0 - a0 - c0, c0, m);
        acc[(size_t)A.beta_t * NK] = reduce24(a1, s1 - a1 - c1, c1, m);
    }
}

// Recover Limbs with 48-bit T primes (reading K4, as k_klss_recover below).

template <int AP>
__global__ void __launch_bounds__(256)
k_klss_recover48(const __grid_constant__ KlssRecArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int gi = blockIdx.y >> 1, c = blockIdx.y & 1, b = blockIdx.z;
    const RecTab& R = *A.tab;
    const int o0 = A.first[gi], no = A.first[gi + 1] - o0;
    // outputs on the FP64 pipe (the y_k on the integer pipe): out_p = sum_k mulc(y_k, [That_k]_p)
    // - mulc(u, [T]_p), each |mulc| <= 0.75 p for |y_k| < 2^48 (common.cuh bound), |sum| < 18 p
    __shared__ TWD tc[KLSS_MAX_OUT_G][AP];                     // this group's ([That_k]_p, /p)
    __shared__ TWD tT[KLSS_MAX_OUT_G];                         // ([T]_p, /p)
    __shared__ double2 tm[KLSS_MAX_OUT_G];                     // (p, 1/p)
    __shared__ int tpos[KLSS_MAX_OUT_G];
    for (int e = threadIdx.x; e < no * AP; e += blockDim.x) {
        const int ro = e / AP, k = e - ro * AP, p = A.out_id[o0 + ro];
        const double pd = (double)A.mods[p].q;
        tc[ro][k] = TWD{(double)R.that_p[p][k].w, (double)R.that_p[p][k].w / pd};
        if (k == 0) {
            tT[ro] = TWD{(double)R.T_p[p].w, (double)R.T_p[p].w / pd};
            tm[ro] = make_double2(pd, 1.0 / pd);
            tpos[ro] = A.out_pos[o0 + ro];
        }
    }
    __syncthreads();
    if (n >= A.N) return;
    const size_t NK = (size_t)AP * A.N;
    const u64* a = A.acc + ((size_t)(b * 2 + c) * A.beta_t + A.group[gi]) * NK + n;
    u64 av[AP];
#pragma unroll
    for (int k = 0; k < AP; ++k) av[k] = a[(size_t)k * A.N];      // all loads in flight first
    double yd[AP];
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < AP; ++k) {
        const u64 y = shoup(av[k], R.that_inv[k], A.mods[A.t0 + k].q);   // y_k = [a_k That_k^-1]_{t_k}
        yd[k] = u2d(y);
        s = __fma_rn(yd[k], R.tinv[k], s);
    }
    const double u = rint(s);
    u64* out = A.rec + (size_t)(b * 2 + c) * A.E * A.N + n;
#pragma unroll 1
    for (int ro = 0; ro < no; ++ro) {
        const double p = tm[ro].x, pinv = tm[ro].y;
        double acc = -mulc(u, tT[ro], p);
#pragma unroll
        for (int k = 0; k < AP; ++k) acc = __dadd_rn(acc, mulc(yd[k], tc[ro][k], p));
        out[(size_t)tpos[ro] * A.N] = d2u(canon(acc, p, pinv));
    }
}

// Recover Limbs: x = the centred lift of acc from T (|x| < T/4 by Eq. 4 + guard bit, K3):
//   y_k = [a_k That_k^-1]_{t_k};  X = sum_k y_k That_k = x + u T exactly, u = rint(sum_k y_k / t_k)
//   (the FP64 sum is within 2^-44 of X / T, and |x / T| < 1/4, so the rounding is exact);
//   out_p = sum_k y_k [That_k]_p - u [T]_p  mod p  = x mod p   (18-bit split products).
template <int AP>
__global__ void __launch_bounds__(256)
k_klss_recover(const __grid_constant__ KlssRecArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int gi = blockIdx.y >> 1, c = blockIdx.y & 1, b = blockIdx.z;
    const RecTab& R = *A.tab;
    const int o0 = A.first[gi], no = A.first[gi + 1] - o0;
    __shared__ uint2 tc[KLSS_MAX_OUT_G][AP];                   // this group's [That_k]_p in 18-bit halves
    __shared__ TW tT[KLSS_MAX_OUT_G];                          // [T]_p
    __shared__ ModQ tm[KLSS_MAX_OUT_G];
    __shared__ int tpos[KLSS_MAX_OUT_G];
    for (int e = threadIdx.x; e < no * AP; e += blockDim.x) {
        const int ro = e / AP, k = e - ro * AP, p = A.out_id[o0 + ro];
        tc[ro][k] = make_uint2(R.that_lo[p][k], R.that_hi[p][k]);
        if (k == 0) {
            tT[ro] = R.T_p[p];
            tm[ro] = A.mods[p];
            tpos[ro] = A.out_pos[o0 + ro];
        }
    }
    __syncthreads();
    if (n >= A.N) return;
    const size_t NK = (size_t)AP * A.N;
    const u64* a = A.acc + ((size_t)(b * 2 + c) * A.beta_t + A.group[gi]) * NK + n;
    u64 av[AP];
#pragma unroll
    for (int k = 0; k < AP; ++k) av[k] = a[(size_t)k * A.N];      // all loads in flight first
    unsigned yl[AP], yh[AP];
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < AP; ++k) {
        const u64 tk = A.mods[A.t0 + k].q;
        const u64 y = shoup(av[k], R.that_inv[k], tk);
        s = __fma_rn((double)y, R.tinv[k], s);
        yl[k] = (unsigned)(y & 0x3FFFF);
        yh[k] = (unsigned)(y >> 18);
    }
    const u64 u = (u64)__double2ll_rn(s);
    u64* out = A.rec + (size_t)(b * 2 + c) * A.E * A.N + n;
#pragma unroll 1
    for (int ro = 0; ro < no; ++ro) {
        u64 a0 = 0, a1 = 0, a2 = 0;
#pragma unroll
        for (int k = 0; k < AP; ++k) {
            const uint2 cc = tc[ro][k];
            mac18(a0, a1, a2, yl[k], yh[k], cc.x, cc.y);
        }
        const ModQ m = tm[ro];
        const u64 r = reduce18(a0, a1, a2, m);
        out[(size_t)tpos[ro] * A.N] = sub_mod(r, shoup(u, tT[ro], m.q), m.q);
    }
}

cudaError_t launch_klss_ip(const KlssIpArgs& A, int batch, cudaStream_t st) {
    const dim3 g(A.N / KLSS_IP_W, A.alpha_p), blk(KLSS_IP_W, 256 / KLSS_IP_W);
    switch (A.beta) {
#define NEO_IP_CASE(B) case B: return launch_k(k_klss_ip<B>, g, blk, 0, st, A, batch);
        NEO_IP_CASE(1) NEO_IP_CASE(2) NEO_IP_CASE(3) NEO_IP_CASE(4) NEO_IP_CASE(5) NEO_IP_CASE(6)
        NEO_IP_CASE(7) NEO_IP_CASE(8) NEO_IP_CASE(9) NEO_IP_CASE(10) NEO_IP_CASE(11) NEO_IP_CASE(12)
#undef NEO_IP_CASE
        default: return cudaErrorInvalidValue;
    }
}
cudaError_t launch_klss_ip48(const KlssIpArgs& A, int batch, cudaStream_t st) {
    const dim3 g(A.N / KLSS_IP_W, A.alpha_p), blk(KLSS_IP_W, 256 / KLSS_IP_W);
    switch (A.beta) {
#define NEO_IP_CASE(B) case B: return launch_k(k_klss_ip48<B>, g, blk, 0, st, A, batch);
        NEO_IP_CASE(1) NEO_IP_CASE(2) NEO_IP_CASE(3) NEO_IP_CASE(4) NEO_IP_CASE(5) NEO_IP_CASE(6)
        NEO_IP_CASE(7) NEO_IP_CASE(8) NEO_IP_CASE(9) NEO_IP_CASE(10) NEO_IP_CASE(11) NEO_IP_CASE(12)
#undef NEO_IP_CASE
        default: return cudaErrorInvalidValue;
    }
}
cudaError_t launch_klss_recover48(const KlssRecArgs& A, int batch, cudaStream_t st) {
    const dim3 g((A.N + 255) / 256, 2 * A.n_groups, batch);
    switch (A.alpha_p) {
#define NEO_REC_CASE(K) case K: return launch_k(k_klss_recover48<K>, g, dim3(256), 0, st, A);
        NEO_REC_CASE(2) NEO_REC_CASE(3) NEO_REC_CASE(4) NEO_REC_CASE(5) NEO_REC_CASE(6) NEO_REC_CASE(7)
        NEO_REC_CASE(8) NEO_REC_CASE(9) NEO_REC_CASE(10) NEO_REC_CASE(11) NEO_REC_CASE(12) NEO_REC_CASE(13)
        NEO_REC_CASE(14) NEO_REC_CASE(15) NEO_REC_CASE(16)
#undef NEO_REC_CASE
        default: return cudaErrorInvalidValue;
    }
}
cudaError_t launch_klss_recover(const KlssRecArgs& A, int batch, cudaStream_t st) {
    const dim3 g((A.N + 255) / 256, 2 * A.n_groups, batch);
    switch (A.alpha_p) {
#define NEO_REC_CASE(K) case K: return launch_k(k_klss_recover<K>, g, dim3(256), 0, st, A);
        NEO_REC_CASE(2) NEO_REC_CASE(3) NEO_REC_CASE(4) NEO_REC_CASE(5) NEO_REC_CASE(6) NEO_REC_CASE(7)
        NEO_REC_CASE(8) NEO_REC_CASE(9) NEO_REC_CASE(10) NEO_REC_CASE(11) NEO_REC_CASE(12) NEO_REC_CASE(13)
        NEO_REC_CASE(14) NEO_REC_CASE(15) NEO_REC_CASE(16)
#undef NEO_REC_CASE
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace neo
