/*
 * oracle_core.c -- CPU ORACLE, TEST INFRASTRUCTURE ONLY.
 *
 * Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference
 * legs may load this library.  It shares no code, header or table with the CUDA path
 * (paper_conf_isca_jiaodwfcm0z25_b200/csrc).
 *
 * Plain, slow, obviously-correct modular loops over 36-bit primes.  Every product is
 * formed exactly in unsigned __int128 and reduced with the C '%' operator.
 * Citations are to /root/reference/PAPER.md lines (L<n>).
 *
 *   or_ntt_def / or_intt_def  definitional negacyclic NTT: a_hat[i] = a(psi^(2i+1))
 *                             (four-step/radix-16 NTT of L438-450 computes exactly this
 *                             transform; natural output order).  O(N^2).
 *   or_ntt_point              one output of the definition (Horner), for sampled checks.
 *   or_ntt_fast / or_intt_fast textbook iterative radix-2 FFT over Z_q (bit-reverse then
 *                             Cooley-Tukey), after the psi^n twist; same transform in
 *                             O(N log N); pinned against or_ntt_def by the tests.
 *   or_negacyclic_mul         schoolbook product in Z_q[X]/(X^N+1) (R_a of Table 1).
 *   or_bconv                  Algorithm 1 (L296-319), literally: for i, for j, for coeff:
 *                             out_j += (c_i * qhat_i^-1 mod q_i) * qhat_i mod p_j.
 *   or_vec_*                  element-wise ModMUL / ModADD (L268, L456).
 *   or_crt_exact              EXACT basis conversion by multi-word big-integer CRT (KLSS key
 *                             decomposition and Recover Limbs, L155-180): x = sum_i y_i qhat_i
 *                             mod Q in [0, Q) (optionally centred to (-Q/2, Q/2]), then x mod t.
 */
#include <stdint.h>
#include <stdlib.h>

typedef unsigned long long u64;
typedef unsigned __int128 u128;

static u64 mulmod(u64 a, u64 b, u64 q) { return (u64)(((u128)a * (u128)b) % q); }
static u64 addmod(u64 a, u64 b, u64 q) { return (u64)(((u128)a + (u128)b) % q); }
static u64 submod(u64 a, u64 b, u64 q) { return (u64)(((u128)a + (u128)q - (u128)(b % q)) % q); }

static u64 powmod(u64 a, u64 e, u64 q) {
    u64 r = 1 % q;
    a %= q;
    while (e) {
        if (e & 1) r = mulmod(r, a, q);
        a = mulmod(a, a, q);
        e >>= 1;
    }
    return r;
}

/* inverse by Fermat's little theorem (q prime) */
static u64 invmod(u64 a, u64 q) { return powmod(a, q - 2, q); }

/* ---------------------------------------------------------------- definition */

/* out[i] = sum_k a[k] * psi^((2i+1)k) mod q, i.e. a evaluated at psi^(2i+1) (Horner). */
u64 or_ntt_point(const u64 *a, int n, u64 q, u64 psi, int i) {
    u64 x = powmod(psi, 2 * (u64)i + 1, q);
    u64 acc = 0;
    for (int k = n - 1; k >= 0; --k) acc = addmod(mulmod(acc, x, q), a[k], q);
    return acc;
}

void or_ntt_def(const u64 *a, u64 *out, int n, u64 q, u64 psi) {
#pragma omp parallel for schedule(static)
    for (int i = 0; i < n; ++i) out[i] = or_ntt_point(a, n, q, psi, i);
}

/* inverse of the definition: a[k] = n^-1 * sum_i a_hat[i] * psi^(-(2i+1)k) */
void or_intt_def(const u64 *ahat, u64 *out, int n, u64 q, u64 psi) {
    u64 psi_inv = invmod(psi, q);
    u64 n_inv = invmod((u64)n % q, q);
#pragma omp parallel for schedule(static)
    for (int k = 0; k < n; ++k) {
        /* sum_i ahat[i] * (psi^-k)^(2i+1) = psi^-k * sum_i ahat[i] * (psi^-2k)^i */
        u64 y = powmod(psi_inv, (u64)k, q);
        u64 y2 = mulmod(y, y, q);
        u64 acc = 0;
        for (int i = n - 1; i >= 0; --i) acc = addmod(mulmod(acc, y2, q), ahat[i], q);
        out[k] = mulmod(mulmod(acc, y, q), n_inv, q);
    }
}

/* ---------------------------------------------------------------- textbook FFT */

static void bit_reverse(u64 *a, int n) {
    for (int i = 1, j = 0; i < n; ++i) {
        int bit = n >> 1;
        for (; j & bit; bit >>= 1) j ^= bit;
        j ^= bit;
        if (i < j) { u64 t = a[i]; a[i] = a[j]; a[j] = t; }
    }
}

/* cyclic DFT over Z_q with root w of order n: A[i] = sum_k a[k] w^(ik) (iterative CT). */
static void cyclic_dft(u64 *a, int n, u64 q, u64 w) {
    bit_reverse(a, n);
    for (int len = 2; len <= n; len <<= 1) {
        u64 wlen = powmod(w, (u64)(n / len), q);
        for (int s = 0; s < n; s += len) {
            u64 x = 1;
            for (int j = 0; j < len / 2; ++j) {
                u64 u = a[s + j];
                u64 v = mulmod(a[s + j + len / 2], x, q);
                a[s + j] = addmod(u, v, q);
                a[s + j + len / 2] = submod(u, v, q);
                x = mulmod(x, wlen, q);
            }
        }
    }
}

/* a_hat[i] = sum_k (a[k] psi^k) (psi^2)^(ik): twist, then cyclic DFT with w = psi^2. */
void or_ntt_fast(u64 *a, int n, u64 q, u64 psi) {
    u64 x = 1;
    for (int k = 0; k < n; ++k) { a[k] = mulmod(a[k], x, q); x = mulmod(x, psi, q); }
    cyclic_dft(a, n, q, mulmod(psi, psi, q));
}

void or_intt_fast(u64 *a, int n, u64 q, u64 psi) {
    u64 psi_inv = invmod(psi, q);
    cyclic_dft(a, n, q, mulmod(psi_inv, psi_inv, q));
    u64 n_inv = invmod((u64)n % q, q);
    u64 x = n_inv;
    for (int k = 0; k < n; ++k) { a[k] = mulmod(a[k], x, q); x = mulmod(x, psi_inv, q); }
}

/* rows independent transforms, row r mod q[r] with psi[r]; inverse != 0 selects INTT. */
void or_ntt_fast_batch(u64 *a, int rows, int n, const u64 *q, const u64 *psi, int inverse) {
#pragma omp parallel for schedule(dynamic, 1)
    for (int r = 0; r < rows; ++r) {
        if (inverse) or_intt_fast(a + (size_t)r * n, n, q[r], psi[r]);
        else         or_ntt_fast(a + (size_t)r * n, n, q[r], psi[r]);
    }
}

/* ---------------------------------------------------------------- ring product */

/* out = a * b in Z_q[X]/(X^n + 1): X^n = -1 wraps with a sign flip. */
void or_negacyclic_mul(const u64 *a, const u64 *b, u64 *out, int n, u64 q) {
#pragma omp parallel for schedule(static)
    for (int k = 0; k < n; ++k) {
        u64 pos = 0, neg = 0;
        for (int i = 0; i <= k; ++i) pos = addmod(pos, mulmod(a[i], b[k - i], q), q);
        for (int i = k + 1; i < n; ++i) neg = addmod(neg, mulmod(a[i], b[n + k - i], q), q);
        out[k] = submod(pos, neg, q);
    }
}

/* ---------------------------------------------------------------- Algorithm 1 */

/* in : [alpha][n]   residues mod q_in[i]
 * out: [alpha_out][n] residues mod t[j]   (overwritten)
 * qhat_inv[i]          = (prod_{i' != i} q_in[i'])^-1 mod q_in[i]
 * qhat_mod_t[i*alpha_out + j] = (prod_{i' != i} q_in[i']) mod t[j]
 * Loop order is Algorithm 1's (i outer, j middle, coefficient inner). */
void or_bconv(const u64 *in, int alpha, u64 *out, int alpha_out, int n,
              const u64 *q_in, const u64 *qhat_inv, const u64 *qhat_mod_t, const u64 *t) {
    for (size_t x = 0; x < (size_t)alpha_out * n; ++x) out[x] = 0;
    for (int i = 0; i < alpha; ++i) {
#pragma omp parallel for schedule(static)
        for (int j = 0; j < alpha_out; ++j) {
            u64 f = qhat_mod_t[(size_t)i * alpha_out + j] % t[j];
            for (int l = 0; l < n; ++l) {
                u64 y = mulmod(in[(size_t)i * n + l], qhat_inv[i], q_in[i]); /* [c_i qhat_i^-1]_{q_i} */
                out[(size_t)j * n + l] = addmod(out[(size_t)j * n + l], mulmod(y, f, t[j]), t[j]);
            }
        }
    }
}

/* ---------------------------------------------------------------- element-wise */

void or_vec_mulmod(const u64 *a, const u64 *b, u64 *out, long n, u64 q) {
#pragma omp parallel for schedule(static)
    for (long k = 0; k < n; ++k) out[k] = mulmod(a[k], b[k], q);
}
void or_vec_addmod(const u64 *a, const u64 *b, u64 *out, long n, u64 q) {
#pragma omp parallel for schedule(static)
    for (long k = 0; k < n; ++k) out[k] = addmod(a[k], b[k], q);
}
void or_vec_submod(const u64 *a, const u64 *b, u64 *out, long n, u64 q) {
#pragma omp parallel for schedule(static)
    for (long k = 0; k < n; ++k) out[k] = submod(a[k], b[k], q);
}
void or_vec_scalar_mulmod(const u64 *a, u64 s, u64 *out, long n, u64 q) {
#pragma omp parallel for schedule(static)
    for (long k = 0; k < n; ++k) out[k] = mulmod(a[k], s, q);
}
/* out = a mod q (inputs are arbitrary u64) */
void or_vec_mod(const u64 *a, u64 *out, long n, u64 q) {
#pragma omp parallel for schedule(static)
    for (long k = 0; k < n; ++k) out[k] = a[k] % q;
}

/* ---------------------------------------------------------------- exact CRT (big integers) */

/* Little-endian multi-word naturals of W <= 8 64-bit words. */
#define CRT_MAXW 8

static int mw_ge(const u64 *a, const u64 *b, int W) {         /* a >= b */
    for (int w = W - 1; w >= 0; --w)
        if (a[w] != b[w]) return a[w] > b[w];
    return 1;
}
static void mw_sub(u64 *a, const u64 *b, int W) {              /* a -= b (a >= b) */
    u64 borrow = 0;
    for (int w = 0; w < W; ++w) {
        u128 d = (u128)a[w] - b[w] - borrow;
        a[w] = (u64)d;
        borrow = (u64)(d >> 64) ? 1 : 0;
    }
}
static u64 mw_mod(const u64 *a, int W, u64 t) {                /* a mod t, Horner over words */
    u128 r = 0;
    for (int w = W - 1; w >= 0; --w) r = ((r << 64) | a[w]) % t;
    return (u64)r;
}

/* in[n_in][n]: residues c_i mod q_i; qhat_inv[i] = (Q/q_i)^-1 mod q_i; qhat[n_in][W] and Q[W]
 * as W-word naturals (n_in * Q < 2^(64 W)); t[n_out].  For every coefficient:
 *   y_i = c_i qhat_inv_i mod q_i,  x = sum_i y_i qhat_i  (exact),  x -= Q while x >= Q,
 *   centred: x > Q/2 -> x - Q (negative);   out[j] = x mod t_j.
 * This is the definition of the CRT lift (no floating point, no approximation). */
void or_crt_exact(const u64 *in, const u64 *q, const u64 *qhat_inv, int n_in, const u64 *qhat,
                  const u64 *Q, int W, const u64 *t, int n_out, u64 *out, int n, int centred) {
#pragma omp parallel for schedule(static)
    for (int k = 0; k < n; ++k) {
        u64 acc[CRT_MAXW + 1] = {0};
        for (int i = 0; i < n_in; ++i) {
            const u64 y = mulmod(in[(size_t)i * n + k], qhat_inv[i], q[i]);
            u64 carry = 0;
            for (int w = 0; w < W; ++w) {
                u128 v = (u128)y * qhat[(size_t)i * W + w] + acc[w] + carry;
                acc[w] = (u64)v;
                carry = (u64)(v >> 64);
            }
            acc[W] += carry;
        }
        u64 Qe[CRT_MAXW + 1];                                  /* Q as W + 1 words */
        for (int w = 0; w < W; ++w) Qe[w] = Q[w];
        Qe[W] = 0;
        while (mw_ge(acc, Qe, W + 1)) mw_sub(acc, Qe, W + 1);  /* at most n_in subtractions */
        int neg = 0;
        if (centred) {                                         /* 2 x > Q  ->  x - Q */
            u64 twice[CRT_MAXW + 1];
            u64 c = 0;
            for (int w = 0; w < W; ++w) {
                twice[w] = (acc[w] << 1) | c;
                c = acc[w] >> 63;
            }
            twice[W] = c;
            if (!mw_ge(Qe, twice, W + 1)) {                    /* Q < 2x */
                u64 m[CRT_MAXW];
                for (int w = 0; w < W; ++w) m[w] = Q[w];
                mw_sub(m, acc, W);                             /* |x - Q| = Q - x */
                for (int w = 0; w < W; ++w) acc[w] = m[w];
                neg = 1;
            }
        }
        for (int j = 0; j < n_out; ++j) {
            const u64 r = mw_mod(acc, W, t[j]);
            out[(size_t)j * n + k] = (neg && r) ? t[j] - r : r;
        }
    }
}

int or_num_threads(void) {
    int t = 1;
#pragma omp parallel
    {
#pragma omp single
        {
#ifdef _OPENMP
            extern int omp_get_num_threads(void);
            t = omp_get_num_threads();
#endif
        }
    }
    return t;
}
