// kernels.cu -- BConv (CUDA-core), KeyIP, combine, tensor, automorphism and rescale helpers.
#include "context.h"
#include <algorithm>

#include "kernels.h"

namespace neo {

// ------------------------------------------------------------------ BConv (Algorithm 1)
// CONTROL kernel, off the default path: the CUDA-core form kept for A/B against the tcgen05
// BConv (NEO_BCONV=cuda) and for neo_bconv's generic conversions that have no tensor-core table.
// One thread per coefficient: y_i = [c_i qhat_i^-1]_{q_i} (Shoup), then every output
// out_j = sum_i y_i f_ij mod t_j with y and f split in 18-bit halves so that each MAC is
// four 32x32->64 IMADs into three 64-bit partial sums (12 inputs: < 2^41 each), followed
// by one Barrett reduction of the < 2^77 total.  (L296-319.)
__global__ void __launch_bounds__(256)
k_bconv(BConvTab T, BConvIO io, int N) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int b = blockIdx.y;
    if (n >= N) return;
    unsigned ylo[BC_MAX_IN], yhi[BC_MAX_IN];
    const u64* in = io.in + b * io.in_bstride + n;
#pragma unroll
    for (int i = 0; i < BC_MAX_IN; ++i) {
        if (i < T.n_in) {
            u64 c = in[(size_t)io.in_off[i] * N];
            u64 y = shoup(c, T.qhat_inv[i], T.qin[i]);
            ylo[i] = (unsigned)(y & 0x3FFFF);
            yhi[i] = (unsigned)(y >> 18);
        } else {
            ylo[i] = yhi[i] = 0;
        }
    }
    u64* out = io.out + b * io.out_bstride + n;
    for (int j = 0; j < T.n_out; ++j) {
        u64 A = 0, B = 0, C = 0;
#pragma unroll
        for (int i = 0; i < BC_MAX_IN; ++i) {
            if (i < T.n_in) {
                const unsigned flo = T.f_lo[i][j], fhi = T.f_hi[i][j];
                A += (u64)ylo[i] * flo;
                B += (u64)ylo[i] * fhi + (u64)yhi[i] * flo;
                C += (u64)yhi[i] * fhi;
            }
        }
        u64 t = A + (B << 18);                 // < 2^60
        u64 lo = t + (C << 36);
        u64 hi = (C >> 28) + (lo < t);
        out[(size_t)io.out_off[j] * N] = barrett_reduce(hi, lo, T.tmod[j]);
    }
}

// ------------------------------------------------------------------ KeyIP (Alg. 3)
// acc_c[t] = sum_j dhat_j[t] * evk_{j,c}[t] mod t for c = 0, 1 (L359-382).  One thread per
// (limb, coefficient) holds its 2*beta key words in registers and walks the whole batch, so
// the key is read from HBM once per launch however large the batch (Z21; the CUDA-core IP
// mapping of L488 with the evaluation key reused across the batch).
template <int BETA>
__device__ __forceinline__ void keyip_body(const KeyIPArgs& A, int n, int t, int batch) {
    static_assert(BETA >= 1 && BETA <= KS_MAX_BETA, "beta out of range");
    const ModQ m = A.mods[A.limb[t]];
    u64 e0[BETA], e1[BETA];
    const u64* src[BETA];
    long long sb[BETA];
#pragma unroll
    for (int j = 0; j < BETA; ++j) {
        const size_t o0 = ((size_t)(2 * j) * A.evk_limbs + A.limb[t]) * A.N + n;
        const size_t o1 = o0 + (size_t)A.evk_limbs * A.N;
        e0[j] = (u64)A.evk_lo[o0] | ((u64)A.evk_hi[o0] << 32);
        e1[j] = (u64)A.evk_lo[o1] | ((u64)A.evk_hi[o1] << 32);
        const bool up = A.src_kind[j][t];
        const unsigned nn = (up || !A.galois) ? (unsigned)n      // sigma_g gather (fused HROTATE AUTO)
                            : (unsigned)(((unsigned long long)A.galois * n + (A.galois - 1) / 2) & (A.N - 1));
        src[j] = (up ? A.up : A.d) + (size_t)A.src_off[j][t] * A.N + nn;
        sb[j] = up ? A.up_bstride : A.d_bstride;
    }
    u64* acc = A.acc + (size_t)t * A.N + n;
    for (int b = 0; b < batch; ++b) {
        u64 x[BETA];
#pragma unroll
        for (int j = 0; j < BETA; ++j) x[j] = src[j][b * sb[j]];
        u64 h0 = 0, l0 = 0, h1 = 0, l1 = 0;
#pragma unroll
        for (int j = 0; j < BETA; ++j) {
            mac128(h0, l0, x[j], e0[j]);
            mac128(h1, l1, x[j], e1[j]);
        }
        u64* o = acc + b * A.acc_bstride;
        u64 r0 = barrett_reduce(h0, l0, m), r1 = barrett_reduce(h1, l1, m);
        if (A.accumulate) {
            r0 = add_mod(r0, o[0], m.q);
            r1 = add_mod(r1, o[(size_t)A.acc_cstride], m.q);
        }
        o[0] = r0;
        o[(size_t)A.acc_cstride] = r1;
    }
}

// At beta = 3 (Set-B) the body fits 40 registers without spilling: 6 CTAs per SM instead of
// 5 (48 registers) gives more loads in flight (KeyIP 0.112 -> 0.106 ms per step).  Larger
// beta would spill at that bound and keeps the default.
#ifndef KEYIP_NT
#define KEYIP_NT 128
#endif
template <int BETA>
__global__ void __launch_bounds__(KEYIP_NT, BETA == 3 ? 6 * 256 / KEYIP_NT : 1)
k_keyip(const __grid_constant__ KeyIPArgs A, int batch) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int t = blockIdx.y;
    if (n >= A.N) return;
    keyip_body<BETA>(A, n, t, batch);
}

// ------------------------------------------------------------------ combine (ModDown tail)
// out_c[i] = (acc_c[i] - conv_c[i]) * P^-1 mod q_i  (+ add_c[i]); Fig. 5, Z9.  Off the
// single-GPU path (there the tail is the NTT row pass's epilogue); used by neo_moddown_combine,
// the limb-sharded building block.
__global__ void __launch_bounds__(256)
k_combine(CombineArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int i = blockIdx.y, bc = blockIdx.z, b = bc >> 1, c = bc & 1;
    if (n >= A.N) return;
    const u64 q = A.mods[A.limb[i]].q;
    const size_t row = (size_t)i * A.N + n;
    u64 a = A.acc[b * A.acc_bstride + c * A.acc_cstride + row];
    u64 v = A.conv[(size_t)bc * A.conv_stride + row];
    u64 r = shoup(sub_mod(a, v, q), A.pinv[i], q);
    const u64* add = c ? A.add1 : A.add0;
    if (add) r = add_mod(r, add[b * A.add_bstride + row], q);
    u64* out = c ? A.out1 : A.out0;
    out[b * A.out_bstride + row] = r;
}

// ------------------------------------------------------------------ tensor (HMULT, L132)
__global__ void __launch_bounds__(256)
k_tensor(const u64* __restrict__ cta, const u64* __restrict__ ctb, u64* __restrict__ d,
         const ModQ* __restrict__ mods, int limbs, int N) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int i = blockIdx.y, b = blockIdx.z;
    if (n >= N) return;
    const ModQ m = mods[i];
    const size_t cs = (size_t)limbs * N;             // component stride
    const size_t base = (size_t)b * 2 * cs + (size_t)i * N + n;
    const u64 a0 = cta[base], a1 = cta[base + cs], b0 = ctb[base], b1 = ctb[base + cs];
    const size_t ob = (size_t)b * 3 * cs + (size_t)i * N + n;
    d[ob] = mul_mod(a0, b0, m);
    u64 h = 0, l = 0;
    mac128(h, l, a0, b1);
    mac128(h, l, a1, b0);
    d[ob + cs] = barrett_reduce(h, l, m);
    d[ob + 2 * cs] = mul_mod(a1, b1, m);
}

// Two coefficients per thread with 16-byte accesses; d2 (the key-switch input, read by the INTT
// that follows) is stored L2 evict_last.
__global__ void __launch_bounds__(256)
k_tensor2(const u64* __restrict__ cta, const u64* __restrict__ ctb, u64* __restrict__ d,
          const ModQ* __restrict__ mods, int limbs, int N) {
    pdl_wait();
    const int n = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
    const int i = blockIdx.y, b = blockIdx.z;
    if (n >= N) return;
    const ModQ m = mods[i];
    const size_t cs = (size_t)limbs * N;
    const size_t base = (size_t)b * 2 * cs + (size_t)i * N + n;
    const ulonglong2 A0 = __ldg(reinterpret_cast<const ulonglong2*>(cta + base));
    const ulonglong2 A1 = __ldg(reinterpret_cast<const ulonglong2*>(cta + base + cs));
    const ulonglong2 B0 = __ldg(reinterpret_cast<const ulonglong2*>(ctb + base));
    const ulonglong2 B1 = __ldg(reinterpret_cast<const ulonglong2*>(ctb + base + cs));
    const size_t ob = (size_t)b * 3 * cs + (size_t)i * N + n;
    ulonglong2 r0, r1, r2;
    r0.x = mul_mod(A0.x, B0.x, m);
    r0.y = mul_mod(A0.y, B0.y, m);
    {
        u64 h = 0, l = 0;
        mac128(h, l, A0.x, B1.x);
        mac128(h, l, A1.x, B0.x);
        r1.x = barrett_reduce(h, l, m);
        h = 0; l = 0;
        mac128(h, l, A0.y, B1.y);
        mac128(h, l, A1.y, B0.y);
        r1.y = barrett_reduce(h, l, m);
    }
    r2.x = mul_mod(A1.x, B1.x, m);
    r2.y = mul_mod(A1.y, B1.y, m);
    *reinterpret_cast<ulonglong2*>(d + ob) = r0;
    *reinterpret_cast<ulonglong2*>(d + ob + cs) = r1;
    uint64_t pol;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(pol));
    asm volatile("st.global.L2::cache_hint.v2.u64 [%0], {%1, %2}, %3;\n" ::"l"(d + ob + 2 * cs), "l"(r2.x), "l"(r2.y),
                 "l"(pol) : "memory");
}

// ------------------------------------------------------------------ automorphism (AUTO)
// out[i] = in[(g i + (g-1)/2) mod N]: X -> X^g in the natural-order NTT domain.
#ifndef AUTO_ILP
#define AUTO_ILP 4
#endif
__global__ void __launch_bounds__(256)
k_automorph(const u64* __restrict__ in, u64* __restrict__ out, unsigned g, int N, long long in_bs, long long out_bs) {
    pdl_wait();
    // AUTO_ILP gathers per thread, all issued before the stores (loads in flight per SM).
    const size_t row = (size_t)blockIdx.y * N;
    const u64* src_row = in + blockIdx.z * in_bs + row;
    u64* dst_row = out + blockIdx.z * out_bs + row;
    const int i0 = blockIdx.x * blockDim.x * AUTO_ILP + threadIdx.x;
    u64 v[AUTO_ILP];
#pragma unroll
    for (int k = 0; k < AUTO_ILP; ++k) {
        const int i = i0 + k * blockDim.x;
        const unsigned src = (unsigned)(((unsigned long long)g * i + (g - 1) / 2) & (N - 1));
        if (i < N) v[k] = src_row[src];
    }
#pragma unroll
    for (int k = 0; k < AUTO_ILP; ++k) {
        const int i = i0 + k * blockDim.x;
        if (i < N) dst_row[i] = v[k];
    }
}


// ------------------------------------------------------------------ PMULT / HADD / PADD
// L133-135, two coefficients per thread (16-byte accesses):
//   PMULT (c0 m, c1 m);  HADD (a0 + b0, a1 + b1);  PADD (c0 + m, c1)   (Z1: m joins c0)
__global__ void __launch_bounds__(256)
k_ew(const __grid_constant__ EwArgs A) {
    pdl_wait();
    const int n = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
    const int i = blockIdx.y, b = blockIdx.z;
    if (n >= A.N) return;
    const ModQ m = A.mods[i];
    const size_t cs = (size_t)A.limbs * A.N;
    const size_t ct = (size_t)b * 2 * cs + (size_t)i * A.N + n;
    const size_t pt = (size_t)b * cs + (size_t)i * A.N + n;
    const ulonglong2 x0 = *reinterpret_cast<const ulonglong2*>(A.a + ct);
    const ulonglong2 x1 = *reinterpret_cast<const ulonglong2*>(A.a + ct + cs);
    ulonglong2 y0, y1;
    if (A.op == EW_HADD) {
        const ulonglong2 b0 = *reinterpret_cast<const ulonglong2*>(A.b + ct);
        const ulonglong2 b1 = *reinterpret_cast<const ulonglong2*>(A.b + ct + cs);
        y0 = make_ulonglong2(add_mod(x0.x, b0.x, m.q), add_mod(x0.y, b0.y, m.q));
        y1 = make_ulonglong2(add_mod(x1.x, b1.x, m.q), add_mod(x1.y, b1.y, m.q));
    } else if (A.op == EW_HSUB) {
        const ulonglong2 b0 = *reinterpret_cast<const ulonglong2*>(A.b + ct);
        const ulonglong2 b1 = *reinterpret_cast<const ulonglong2*>(A.b + ct + cs);
        y0 = make_ulonglong2(sub_mod(x0.x, b0.x, m.q), sub_mod(x0.y, b0.y, m.q));
        y1 = make_ulonglong2(sub_mod(x1.x, b1.x, m.q), sub_mod(x1.y, b1.y, m.q));
    } else {
        const ulonglong2 p = *reinterpret_cast<const ulonglong2*>(A.b + pt);
        if (A.op == EW_PMULT) {
            y0 = make_ulonglong2(mul_mod(x0.x, p.x, m), mul_mod(x0.y, p.y, m));
            y1 = make_ulonglong2(mul_mod(x1.x, p.x, m), mul_mod(x1.y, p.y, m));
        } else {
            y0 = make_ulonglong2(add_mod(x0.x, p.x, m.q), add_mod(x0.y, p.y, m.q));
            y1 = x1;
        }
    }
    *reinterpret_cast<ulonglong2*>(A.out + ct) = y0;
    *reinterpret_cast<ulonglong2*>(A.out + ct + cs) = y1;
}

__global__ void __launch_bounds__(256)
k_add_rows(const u64* __restrict__ a, const u64* __restrict__ b, u64* out, const ModQ* __restrict__ mods, int limbs,
           int N) {
    pdl_wait();
    const int n = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
    const int i = blockIdx.y;
    if (n >= N) return;
    const u64 q = mods[i].q;
    const size_t o = ((size_t)blockIdx.z * limbs + i) * N + n;
    const ulonglong2 x = *reinterpret_cast<const ulonglong2*>(a + o), y = *reinterpret_cast<const ulonglong2*>(b + o);
    *reinterpret_cast<ulonglong2*>(out + o) = make_ulonglong2(add_mod(x.x, y.x, q), add_mod(x.y, y.y, q));
}

// ------------------------------------------------------------------ plaintext inner product
// sum_k (c0_k m_k, c1_k m_k) (L133 PMULT + L134 HADD, the diagonal method's inner loop):
// products < 2^72 accumulate exactly in 128 bits (n_terms <= 32: < 2^77), one Barrett
// reduction per output.  Two coefficients per thread, 16-byte accesses; one read of every
// operand and one write, against 2 k launches and k - 1 intermediate ciphertexts unfused.
__global__ void __launch_bounds__(256)
k_pmult_acc(const __grid_constant__ PmaccArgs A) {
    pdl_wait();
    const int n = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
    const int i = blockIdx.y, b = blockIdx.z;
    if (n >= A.N) return;
    const ModQ m = A.mods[i];
    const size_t cs = (size_t)A.limbs * A.N;
    const size_t ct = (size_t)b * 2 * cs + (size_t)i * A.N + n;
    const size_t pt = (A.pt_shared ? 0 : (size_t)b * cs) + (size_t)i * A.N + n;
    u64 h[4] = {0, 0, 0, 0}, l[4] = {0, 0, 0, 0};
#pragma unroll 4
    for (int k = 0; k < A.n_terms; ++k) {
        const ulonglong2 x0 = __ldg(reinterpret_cast<const ulonglong2*>(A.ct[k] + ct));
        const ulonglong2 x1 = __ldg(reinterpret_cast<const ulonglong2*>(A.ct[k] + ct + cs));
        const ulonglong2 p = __ldg(reinterpret_cast<const ulonglong2*>(A.pt[k] + pt));
        mac128(h[0], l[0], x0.x, p.x);
        mac128(h[1], l[1], x0.y, p.y);
        mac128(h[2], l[2], x1.x, p.x);
        mac128(h[3], l[3], x1.y, p.y);
    }
    *reinterpret_cast<ulonglong2*>(A.out + ct) =
        make_ulonglong2(barrett_reduce(h[0], l[0], m), barrett_reduce(h[1], l[1], m));
    *reinterpret_cast<ulonglong2*>(A.out + ct + cs) =
        make_ulonglong2(barrett_reduce(h[2], l[2], m), barrett_reduce(h[3], l[3], m));
}

// ------------------------------------------------------------------ limb-subset element-wise ops
// One thread per (coefficient, row k, batch b); both components in the thread.
__global__ void __launch_bounds__(256)
k_ew_limbs(const __grid_constant__ EwlArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int k = blockIdx.y, b = blockIdx.z;
    if (n >= A.N) return;
    const ModQ m = A.mods[A.lid[k]];
    const size_t cs = (size_t)A.n * A.N;
    const size_t ct = (size_t)b * 2 * cs + (size_t)k * A.N + n;
    if (A.op == EWL_LIFT) {                                  // centred lift from q_src
        const u64 qs = A.mods[A.src].q;
#pragma unroll
        for (int c = 0; c < 2; ++c) {
            const u64 x = A.a[((size_t)b * 2 + c) * A.N + n];
            u64 r;
            if (2 * x > qs) {
                const u64 mm = (qs - x) % m.q;
                r = mm == 0 ? 0 : m.q - mm;
            } else {
                r = x % m.q;
            }
            A.out[ct + c * cs] = r;
        }
        return;
    }
    const u64 a0 = A.a[ct], a1 = A.a[ct + cs];
    if (A.op == EWL_TENSOR) {
        const u64 b0 = A.b[ct], b1 = A.b[ct + cs];
        const size_t ob = (size_t)b * 3 * cs + (size_t)k * A.N + n;
        A.out[ob] = mul_mod(a0, b0, m);
        u64 h = 0, l = 0;
        mac128(h, l, a0, b1);
        mac128(h, l, a1, b0);
        A.out[ob + cs] = barrett_reduce(h, l, m);
        A.out[ob + 2 * cs] = mul_mod(a1, b1, m);
        return;
    }
    u64 y0, y1;
    if (A.op == EWL_HADD || A.op == EWL_HSUB || A.op == EWL_SUBMUL) {
        const u64 b0 = A.b[ct], b1 = A.b[ct + cs];
        if (A.op == EWL_HADD) {
            y0 = add_mod(a0, b0, m.q);
            y1 = add_mod(a1, b1, m.q);
        } else {
            y0 = sub_mod(a0, b0, m.q);
            y1 = sub_mod(a1, b1, m.q);
            if (A.op == EWL_SUBMUL) {
                y0 = shoup(y0, A.scal[k], m.q);
                y1 = shoup(y1, A.scal[k], m.q);
            }
        }
    } else {
        const u64 p = A.b[(size_t)b * cs + (size_t)k * A.N + n];
        if (A.op == EWL_PMULT) {
            y0 = mul_mod(a0, p, m);
            y1 = mul_mod(a1, p, m);
        } else {
            y0 = add_mod(a0, p, m.q);
            y1 = a1;
        }
    }
    A.out[ct] = y0;
    A.out[ct + cs] = y1;
}

// ------------------------------------------------------------------ fused HMULT + Rescale
// One thread per (coefficient, group of kFoldRows rows, bc): c_l once per thread from three
// L2-resident reads, then its rows (a single loop over all l rows per thread was latency-bound
// at 512 CTAs; one row per thread re-read c_l's inputs 35 times: 18.8 / 30 us per step).
constexpr int kFoldRows = 6;
__global__ void __launch_bounds__(256)
k_hmr_fold(const __grid_constant__ HmrFoldArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int i0 = blockIdx.y * kFoldRows, bc = blockIdx.z;
    if (n >= A.N) return;
    const size_t row = (size_t)A.N, base = (size_t)bc * (A.l + 1) * row + n;
    const ModQ ml = A.mods[A.l];
    u64 cv;
    if (A.lazy) cv = d2u(canon(__longlong_as_double((long long)__ldg(A.conv + base + (size_t)A.l * row)), ml.qd, ml.qinv));
    else cv = __ldg(A.conv + base + (size_t)A.l * row);
    const u64 cl = add_mod(shoup(sub_mod(__ldg(A.accl + (size_t)bc * row + n), cv, ml.q), A.pinv_l, ml.q),
                           __ldg(A.dl + (size_t)bc * row + n), ml.q);
    const double cld = u2d(cl);
    const int i1 = min(A.l, i0 + kFoldRows);
    u64* p = A.conv + base + (size_t)i0 * row;
    u64 v[kFoldRows];                                // all rows' loads in flight before the stores
#pragma unroll
    for (int k = 0; k < kFoldRows; ++k)
        if (i0 + k < i1) v[k] = p[(size_t)k * row];
#pragma unroll
    for (int k = 0; k < kFoldRows; ++k) {
        const int i = i0 + k;
        if (i >= i1) break;
        const ModQ m = A.mods[i];
        if (A.lazy) {
            const double z = __dadd_rn(__longlong_as_double((long long)v[k]), mulc(cld, A.pmod[i], m.qd));
            p[(size_t)k * row] = (u64)__double_as_longlong(canon(z, m.qd, m.qinv));
        } else {
            p[(size_t)k * row] = add_mod(v[k], d2u(canon(mulc(cld, A.pmod[i], m.qd), m.qd, m.qinv)), m.q);
        }
    }
}

// c_l only (the fold itself goes into the next NTT's column pass, RowSet::fold): writes
// c_l = ((accl - [conv_l]) P^-1 + dl) mod q_l over accl
__global__ void __launch_bounds__(256)
k_hmr_cl(const __grid_constant__ HmrFoldArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int bc = blockIdx.y;
    if (n >= A.N) return;
    const size_t row = (size_t)A.N, base = (size_t)bc * (A.l + 1) * row + n;
    const ModQ ml = A.mods[A.l];
    u64 cv;
    if (A.lazy) cv = d2u(canon(__longlong_as_double((long long)__ldg(A.conv + base + (size_t)A.l * row)), ml.qd, ml.qinv));
    else cv = __ldg(A.conv + base + (size_t)A.l * row);
    u64* cl = const_cast<u64*>(A.accl) + (size_t)bc * row + n;
    *cl = add_mod(shoup(sub_mod(*cl, cv, ml.q), A.pinv_l, ml.q), __ldg(A.dl + (size_t)bc * row + n), ml.q);
}

// ------------------------------------------------------------------ ModRaise (bootstrapping)
// c in [0, q_0) -> the centred representative in (-q_0/2, q_0/2] reduced mod q_i
__global__ void __launch_bounds__(256)
k_modraise(const u64* __restrict__ coef, u64* __restrict__ out, const ModQ* __restrict__ mods, int limbs, int N) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int i = blockIdx.y, bc = blockIdx.z;
    if (n >= N) return;
    const u64 q0 = mods[0].q, qi = mods[i].q;
    const u64 c = coef[(size_t)bc * N + n];
    u64 r;
    if (2 * c > q0) {                                           // negative: c - q0
        const u64 m = q0 - c;                                   // |value| < q_0 / 2 < q_i
        r = m == 0 ? 0 : qi - (m % qi);
    } else {
        r = c % qi;
    }
    out[((size_t)bc * limbs + i) * N + n] = r;
}

__global__ void __launch_bounds__(256)
k_drop(const u64* __restrict__ in, u64* __restrict__ out, int li, int lo, int N) {
    pdl_wait();
    const int n = 2 * (blockIdx.x * blockDim.x + threadIdx.x);
    const int i = blockIdx.y, bc = blockIdx.z;
    if (n >= N) return;
    *reinterpret_cast<ulonglong2*>(out + ((size_t)bc * lo + i) * N + n) =
        *reinterpret_cast<const ulonglong2*>(in + ((size_t)bc * li + i) * N + n);
}

// ------------------------------------------------------------------ Double Rescale (L138, L151)
// Garner: r = r_l + q_l g, g = [(r_{l-1} - r_l) q_l^-1]_{q_{l-1}}, is x mod q_{l-1} q_l exactly
// (0 <= r < q_{l-1} q_l); corr_i = [r]_{q_i} = r_l + [q_l]_{q_i} g mod q_i.
__global__ void __launch_bounds__(256)
k_ds_corr(const __grid_constant__ DsArgs A) {
    pdl_wait();
    const int n = blockIdx.x * blockDim.x + threadIdx.x;
    const int bc = blockIdx.y;
    if (n >= A.N) return;
    const u64 qm = A.mods[A.l - 1].q;
    const u64 rm = A.last2[(size_t)bc * 2 * A.N + n];
    const u64 rl = A.last2[((size_t)bc * 2 + 1) * A.N + n];
    const u64 rlm = rl >= qm ? rl - qm : rl;                     // r_l < q_l < 2^36 <= 2 q_{l-1}
    const u64 g = shoup(sub_mod(rm, rlm, qm), A.qlinv_m, qm);
    u64* out = A.corr + (size_t)bc * (A.l - 1) * A.N + n;
    for (int i = 0; i + 1 < A.l; ++i) {
        const u64 qi = A.mods[i].q;
        const u64 rli = rl >= qi ? rl - qi : rl;
        out[(size_t)i * A.N] = add_mod(rli, shoup(g, A.ql[i], qi), qi);
    }
}

// ------------------------------------------------------------------ 5-byte key packing
__global__ void __launch_bounds__(256)
k_pack5(const u64* __restrict__ in, uint32_t* __restrict__ lo, uint8_t* __restrict__ hi, size_t n) {
    pdl_wait();
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        const u64 v = in[i];
        lo[i] = (uint32_t)v;
        hi[i] = (uint8_t)(v >> 32);
    }
}

// 6-byte packing (48-bit KLSS T residues): low 32 bits and a 16-bit plane
__global__ void __launch_bounds__(256)
k_pack6(const u64* __restrict__ in, uint32_t* __restrict__ lo, uint16_t* __restrict__ hi, size_t n) {
    pdl_wait();
    for (size_t i = blockIdx.x * (size_t)blockDim.x + threadIdx.x; i < n; i += (size_t)gridDim.x * blockDim.x) {
        const u64 v = in[i];
        lo[i] = (uint32_t)v;
        hi[i] = (uint16_t)(v >> 32);
    }
}

// ------------------------------------------------------------------ 36-bit wire format
// n residues < 2^36 as [4n bytes: u32 low words][n/2 bytes: byte k = hi4(2k) | hi4(2k+1) << 4]
// (4.5 bytes per residue against 8: the host<->device copies of neo_wire_pack / _unpack).
// One thread per 8 residues: 32-byte low-word loads, one 4-byte nibble word.
__global__ void __launch_bounds__(256)
k_wire_unpack(const uint8_t* __restrict__ wire, u64* __restrict__ out, size_t n) {
    pdl_wait();
    const uint4* lo = reinterpret_cast<const uint4*>(wire);
    const uint32_t* hi = reinterpret_cast<const uint32_t*>(wire + 4 * n);
    const size_t groups = n / 8;
    for (size_t g = blockIdx.x * (size_t)blockDim.x + threadIdx.x; g < groups; g += (size_t)gridDim.x * blockDim.x) {
        const uint4 a = lo[2 * g], b = lo[2 * g + 1];
        const uint32_t h = hi[g];
        const uint32_t w[8] = {a.x, a.y, a.z, a.w, b.x, b.y, b.z, b.w};
        ulonglong2* o = reinterpret_cast<ulonglong2*>(out + 8 * g);
#pragma unroll
        for (int k = 0; k < 4; ++k)
            o[k] = make_ulonglong2((u64)w[2 * k] | ((u64)((h >> (8 * k)) & 0xF) << 32),
                                   (u64)w[2 * k + 1] | ((u64)((h >> (8 * k + 4)) & 0xF) << 32));
    }
}
__global__ void __launch_bounds__(256)
k_wire_pack(const u64* __restrict__ in, uint8_t* __restrict__ wire, size_t n) {
    pdl_wait();
    uint4* lo = reinterpret_cast<uint4*>(wire);
    uint32_t* hi = reinterpret_cast<uint32_t*>(wire + 4 * n);
    const size_t groups = n / 8;
    for (size_t g = blockIdx.x * (size_t)blockDim.x + threadIdx.x; g < groups; g += (size_t)gridDim.x * blockDim.x) {
        const ulonglong2* v = reinterpret_cast<const ulonglong2*>(in + 8 * g);
        uint32_t w[8], h = 0;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
            const ulonglong2 x = v[k];
            w[2 * k] = (uint32_t)x.x;
            w[2 * k + 1] = (uint32_t)x.y;
            h |= (uint32_t)(((x.x >> 32) & 0xF) | (((x.y >> 32) & 0xF) << 4)) << (8 * k);
        }
        lo[2 * g] = make_uint4(w[0], w[1], w[2], w[3]);
        lo[2 * g + 1] = make_uint4(w[4], w[5], w[6], w[7]);
        hi[g] = h;
    }
}

// ------------------------------------------------------------------ launchers
cudaError_t launch_wire(bool pack, const void* in, void* out, size_t n, cudaStream_t st) {
    const size_t groups = n / 8;
    const unsigned blocks = (unsigned)std::min<size_t>((groups + 255) / 256, 148 * 16);
    if (pack) return launch_k(k_wire_pack, dim3(blocks), dim3(256), 0, st, (const u64*)in, (uint8_t*)out, n);
    return launch_k(k_wire_unpack, dim3(blocks), dim3(256), 0, st, (const uint8_t*)in, (u64*)out, n);
}
cudaError_t launch_ew(const EwArgs& A, int batch, cudaStream_t st) {
    return launch_k(k_ew, dim3((A.N / 2 + 255) / 256, A.limbs, batch), dim3(256), 0, st, A);
}
cudaError_t launch_add_rows(const u64* a, const u64* b, u64* out, const ModQ* mods, int limbs, int N, int batch,
                            cudaStream_t st) {
    return launch_k(k_add_rows, dim3((N / 2 + 255) / 256, limbs, batch), dim3(256), 0, st, a, b, out, mods, limbs, N);
}
cudaError_t launch_pmult_acc(const PmaccArgs& A, int batch, cudaStream_t st) {
    return launch_k(k_pmult_acc, dim3((A.N / 2 + 255) / 256, A.limbs, batch), dim3(256), 0, st, A);
}
cudaError_t launch_ew_limbs(const EwlArgs& A, int batch, cudaStream_t st) {
    return launch_k(k_ew_limbs, dim3((A.N + 255) / 256, A.n, batch), dim3(256), 0, st, A);
}
cudaError_t launch_hmr_fold(const HmrFoldArgs& A, int bc, cudaStream_t st) {
    return launch_k(k_hmr_fold, dim3((A.N + 255) / 256, (A.l + kFoldRows - 1) / kFoldRows, bc), dim3(256), 0, st, A);
}
cudaError_t launch_hmr_cl(const HmrFoldArgs& A, int bc, cudaStream_t st) {
    return launch_k(k_hmr_cl, dim3((A.N + 255) / 256, bc), dim3(256), 0, st, A);
}
cudaError_t launch_modraise(const u64* coef, u64* out, const ModQ* mods, int limbs, int N, int bc, cudaStream_t st) {
    return launch_k(k_modraise, dim3((N + 255) / 256, limbs, bc), dim3(256), 0, st, coef, out, mods, limbs, N);
}
cudaError_t launch_drop(const u64* in, u64* out, int li, int lo, int N, int batch, cudaStream_t st) {
    return launch_k(k_drop, dim3((N / 2 + 255) / 256, lo, 2 * batch), dim3(256), 0, st, in, out, li, lo, N);
}
cudaError_t launch_ds_corr(const DsArgs& A, int bc, cudaStream_t st) {
    return launch_k(k_ds_corr, dim3((A.N + 255) / 256, bc), dim3(256), 0, st, A);
}
cudaError_t launch_pack5(const u64* in, uint32_t* lo, uint8_t* hi, size_t n, cudaStream_t st) {
    return launch_k(k_pack5, dim3(4096), dim3(256), 0, st, in, lo, hi, n);
}
cudaError_t launch_pack6(const u64* in, uint32_t* lo, uint16_t* hi, size_t n, cudaStream_t st) {
    return launch_k(k_pack6, dim3(4096), dim3(256), 0, st, in, lo, hi, n);
}

static inline dim3 g1(int N) { return dim3((N + 255) / 256); }

cudaError_t launch_bconv(const BConvTab& T, const BConvIO& io, int N, int batch, cudaStream_t st) {
    return launch_k(k_bconv, dim3((N + 255) / 256, batch), dim3(256), 0, st, T, io, N);
}
cudaError_t launch_keyip(const KeyIPArgs& A, int limbs, int batch, cudaStream_t st) {
    const dim3 g((A.N + KEYIP_NT - 1) / KEYIP_NT, limbs);
    switch (A.beta) {
        case 1: return launch_k(k_keyip<1>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 2: return launch_k(k_keyip<2>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 3: return launch_k(k_keyip<3>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 4: return launch_k(k_keyip<4>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 5: return launch_k(k_keyip<5>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 6: return launch_k(k_keyip<6>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 7: return launch_k(k_keyip<7>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 8: return launch_k(k_keyip<8>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 9: return launch_k(k_keyip<9>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 10: return launch_k(k_keyip<10>, g, dim3(KEYIP_NT), 0, st, A, batch);
        case 11: return launch_k(k_keyip<11>, g, dim3(KEYIP_NT), 0, st, A, batch);
        default: return launch_k(k_keyip<12>, g, dim3(KEYIP_NT), 0, st, A, batch);
    }
}
cudaError_t launch_combine(const CombineArgs& A, int limbs, int batch, cudaStream_t st) {
    return launch_k(k_combine, dim3((A.N + 255) / 256, limbs, 2 * batch), dim3(256), 0, st, A);
}
cudaError_t launch_tensor(const u64* a, const u64* b, u64* d, const ModQ* mods, int limbs, int N, int batch,
                          cudaStream_t st) {
    static const bool two = [] { const char* e = std::getenv("NEO_TENSOR2"); return !(e && e[0] == '0'); }();
    if (two && (N % 512) == 0)
        return launch_k(k_tensor2, dim3(N / 512, limbs, batch), dim3(256), 0, st, a, b, d, mods, limbs, N);
    return launch_k(k_tensor, dim3(g1(N).x, limbs, batch), dim3(256), 0, st, a, b, d, mods, limbs, N);
}
cudaError_t launch_automorph(const u64* in, u64* out, unsigned g, int N, int rows, cudaStream_t st, int batch,
                             long long in_bs, long long out_bs) {
    return launch_k(k_automorph, dim3((N + 256 * AUTO_ILP - 1) / (256 * AUTO_ILP), rows, batch), dim3(256), 0, st, in, out, g, N, in_bs, out_bs);
}

}  // namespace neo
