// klss.cu -- KLSS key-switching kernels (Neo's default method, L155-180; readings K1-K6 in
// DESIGN.md): the inner product over the T basis (Alg. 3 / Alg. 4) and Recover Limbs.
#include "klss.h"

namespace neo {

// IP on CUDA cores (the paper's CUDA-core IP mapping, L488: its beta x beta~ products are
// far too small for a tensor-core tile at B = 1).  One thread per (T limb k, coefficient n):
// for each present group i and component c the beta key words stay in registers while the
// batch is walked, so the key is read once per launch (Z21).
__global__ void __launch_bounds__(256)
k_klss_ip(const __grid_constant__ KlssIpArgs A, int batch) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int k = blockIdx.y;
    if (n >= A.N) return;
    const ModQ m = A.mods[A.t0 + k];
    const size_t NK = (size_t)A.alpha_p * A.N;                  // one [alpha'][N] block
    const size_t col = (size_t)k * A.N + n;
    for (int gi = 0; gi < A.n_groups; ++gi) {
        const int i = A.group[gi];
        for (int c = 0; c < 2; ++c) {
            u64 e[KLSS_MAX_BETA];
            const size_t kb = (size_t)(c * A.beta_t + i) * A.dnum * NK + col;
#pragma unroll
            for (int j = 0; j < KLSS_MAX_BETA; ++j) {
                e[j] = 0;
                if (j < A.beta) {
                    const size_t o = kb + (size_t)j * NK;
                    e[j] = (u64)A.key_lo[o] | ((u64)A.key_hi[o] << 32);
                }
            }
            for (int b = 0; b < batch; ++b) {
                const u64* up = A.up + (size_t)b * A.beta * NK + col;
                u64 h = 0, l = 0;                               // < beta 2^72 <= 2^76
#pragma unroll
                for (int j = 0; j < KLSS_MAX_BETA; ++j)
                    if (j < A.beta) mac128(h, l, up[(size_t)j * NK], e[j]);
                A.acc[((size_t)(b * 2 + c) * A.beta_t + i) * NK + col] = barrett_reduce(h, l, m);
            }
        }
    }
}

// Recover Limbs: x = the centred lift of acc from T (|x| < T/4 by Eq. 4 + guard bit, K3):
//   y_k = [a_k That_k^-1]_{t_k};  X = sum_k y_k That_k = x + u T exactly, u = rint(sum_k y_k / t_k)
//   (the FP64 sum is within 2^-44 of X / T, and |x / T| < 1/4, so the rounding is exact);
//   out_p = sum_k y_k [That_k]_p - u [T]_p  mod p  = x mod p.
__global__ void __launch_bounds__(256)
k_klss_recover(const __grid_constant__ KlssRecArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int gi = blockIdx.y >> 1, c = blockIdx.y & 1, b = blockIdx.z;
    if (n >= A.N) return;
    const RecTab& R = *A.tab;
    const size_t NK = (size_t)A.alpha_p * A.N;
    const u64* a = A.acc + ((size_t)(b * 2 + c) * A.beta_t + A.group[gi]) * NK + n;
    u64 y[KLSS_MAX_T];
    double s = 0.0;
#pragma unroll
    for (int k = 0; k < KLSS_MAX_T; ++k) {
        y[k] = 0;
        if (k < A.alpha_p) {
            const u64 tk = A.mods[A.t0 + k].q;
            y[k] = shoup(a[(size_t)k * A.N], R.that_inv[k], tk);
            s = __fma_rn((double)y[k], R.tinv[k], s);
        }
    }
    const u64 u = (u64)__double2ll_rn(s);
    for (int o = A.first[gi]; o < A.first[gi + 1]; ++o) {
        const int p = A.out_id[o];
        const ModQ m = A.mods[p];
        u64 h = 0, l = 0;                                       // < 16 * 2^72
#pragma unroll
        for (int k = 0; k < KLSS_MAX_T; ++k)
            if (k < A.alpha_p) mac128(h, l, y[k], R.that_p[p][k].w);
        const u64 r = barrett_reduce(h, l, m);
        A.rec[((size_t)(b * 2 + c) * A.E + A.out_pos[o]) * A.N + n] = sub_mod(r, shoup(u, R.T_p[p], m.q), m.q);
    }
}

// ModDown difference in coefficient form: (conv - acc_q) mod q_i, canonical.
__global__ void __launch_bounds__(256)
k_klss_diff(const __grid_constant__ KlssDiffArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int i = blockIdx.y, bc = blockIdx.z;
    if (n >= A.N) return;
    const u64 q = A.mods[i].q;
    const size_t o = ((size_t)bc * A.Lq + i) * A.N + n;
    const u64 a = A.rec[((size_t)bc * A.E + i) * A.N + n];      // bc = 2 b + c, position i = q_i
    A.out[o] = sub_mod(A.conv[o], a, q);
}

cudaError_t launch_klss_ip(const KlssIpArgs& A, int batch, cudaStream_t st) {
    return launch_k(k_klss_ip, dim3((A.N + 255) / 256, A.alpha_p), dim3(256), 0, st, A, batch);
}
cudaError_t launch_klss_recover(const KlssRecArgs& A, int batch, cudaStream_t st) {
    return launch_k(k_klss_recover, dim3((A.N + 255) / 256, 2 * A.n_groups, batch), dim3(256), 0, st, A);
}
cudaError_t launch_klss_diff(const KlssDiffArgs& A, int batch, cudaStream_t st) {
    return launch_k(k_klss_diff, dim3((A.N + 255) / 256, A.Lq, 2 * batch), dim3(256), 0, st, A);
}

}  // namespace neo
