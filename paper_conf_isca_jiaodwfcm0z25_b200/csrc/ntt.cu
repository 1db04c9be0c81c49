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
//
// Both passes are persistent kernels (2 CTAs/SM) that walk their tiles in limb-major order
// through a two-stage cp.async pipeline: tile t+1 (data, per-prime twiddles, the outer
// twist slice) streams into shared memory while tile t is transformed, so HBM traffic
// overlaps the FP64 work.  Tile = 16 columns x N1 rows (column pass) or 16 rows x N2
// (row pass) = 32 KB at N = 2^16; every global access is a full 128-byte segment.
#include <cstdlib>

#include "common.cuh"
#include "ntt.h"
#include "ntt_tables.h"

namespace neo {

// ------------------------------------------------------------------ cp.async
NEO_DEV uint32_t s_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
NEO_DEV void cp16(void* s, const void* g) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s_u32(s)), "l"(g) : "memory");
}
NEO_DEV void cp_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
NEO_DEV void pf_l2(const void* g) { asm volatile("prefetch.global.L2 [%0];\n" ::"l"(g)); }
template <int N>
NEO_DEV void cp_wait() { asm volatile("cp.async.wait_group %0;\n" ::"n"(N) : "memory"); }
// L2 residency of the pass-to-pass intermediate: evict_last stores, and a discard (invalidate
// without write-back) of each 128-byte line once the next pass has read it
NEO_DEV uint64_t l2_keep_policy() {
    uint64_t p;
    asm volatile("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;\n" : "=l"(p));
    return p;
}
NEO_DEV void st_keep(double* a, double v, uint64_t pol) {
    asm volatile("st.global.L2::cache_hint.f64 [%0], %1, %2;\n" ::"l"(a), "d"(v), "l"(pol) : "memory");
}
NEO_DEV void discard_line(const void* a) { asm volatile("discard.global.L2 [%0], 128;\n" ::"l"(a) : "memory"); }

// ------------------------------------------------------------------ in-register transforms

// Negacyclic R-point forward NTT (Cooley-Tukey, merged psi): natural in, bit-reversed out.
// tab[k] = rho^bitrev(k) (k = 1..R-1), rho a primitive 2R-th root.
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

// ------------------------------------------------------------------ tiling

constexpr int kC = 16;   // columns per column-pass tile / rows per row-pass tile

// TileMap: ntt.h

// 16-byte chunk swizzle for [row][16 doubles] tiles read/written column-wise
NEO_DEV int swz(int row, int col) { return row * 16 + ((((col >> 1) ^ (row & 7)) << 1) | (col & 1)); }

// ------------------------------------------------------------------ column pass

template <int R>
struct ColCfg {
    static constexpr int NT = kC * R;
    static constexpr int NS = R + R * R + R / 2;        // neg, tw1, cyc
    static constexpr int NO = 2 * kC * R;               // outer twist A, B for the tile's columns
    static constexpr int XP = R * R + 1;                // odd pitch: conflict-free exchange
    static constexpr int DATA = kC * XP;                // doubles (>= R*R*kC)
    static constexpr size_t STAGE = (size_t)(NS + NO) * sizeof(TWD) + (size_t)DATA * 8;
};

// Forward: src = canonical u64 coefficients, dst = lazy doubles tmp[i1][n2].
// Inverse: src = lazy doubles tmp[i1][n2], dst = canonical u64 coefficients.
template <int R, bool FWD, int STAGES, int MINB>
__global__ void __launch_bounds__(ColCfg<R>::NT, MINB)
k_ntt_col(RowSet rs, NttArgs a, TileMap tm) {
    using CF = ColCfg<R>;
    constexpr int C = kC, NT = CF::NT;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int tid = threadIdx.x, c = tid % C, r = tid / C;
    constexpr int N1 = R * R, N2 = R * R;       // compile-time strides: immediate address offsets
    constexpr long long NN = (long long)N1 * N2;

    auto stage_ptr = [&](int s) { return smem_raw + s * CF::STAGE; };
    auto issue = [&](int t, int s) {
        if (t < tm.total) {
            int b, k, blk;
            tm.decode(t, b, k, blk);
            const int lid = rs.prime[k];
            const TWD* ptab = a.tabd + (size_t)lid * a.tab_stride;
            unsigned char* st = stage_ptr(s);
            TWD* sT = reinterpret_cast<TWD*>(st);
            double* sD = reinterpret_cast<double*>(st + (CF::NS + CF::NO) * sizeof(TWD));
            const int col0 = blk * C;
            const int off = FWD ? a.L.colf_neg : a.L.coli_neg;
            for (int e = tid; e < CF::NS; e += NT) cp16(sT + e, ptab + off + e);
            const int oa = (FWD ? a.L.outf_a : a.L.outi_a) + col0 * R;
            const int ob = (FWD ? a.L.outf_b : a.L.outi_b) + col0 * R;
            for (int e = tid; e < C * R; e += NT) {       // [c][x] in memory -> [x][c] in smem (no conflicts)
                const int cc = e / R, xx = e % R;
                cp16(sT + CF::NS + xx * C + cc, ptab + oa + e);
                cp16(sT + CF::NS + C * R + xx * C + cc, ptab + ob + e);
            }
            const u64* src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN + col0;
            for (int e = tid; e < N1 * (C / 2); e += NT) {
                const int row = e / (C / 2), part = e % (C / 2);
                cp16(sD + row * C + 2 * part, src + (size_t)row * N2 + 2 * part);
            }
        }
        cp_commit();
    };

    // single-stage configurations: pull the CTA's next tile into L2 while this one is
    // transformed, so its cp.async sees L2 rather than HBM latency (one 128-B line per row)
    auto prefetch = [&](int t) {
        if (STAGES == 1 && t < tm.total) {
            int b, k, blk;
            tm.decode(t, b, k, blk);
            const u64* src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN + blk * C;
            for (int row = tid; row < N1; row += NT) pf_l2(src + (size_t)row * N2);
        }
    };

    const int G = gridDim.x;
    int t = blockIdx.x;
    pdl_wait();            // predecessor's writes visible (and its reads done) before any access
    pdl_trigger();         // persistent grid is fully resident: let the next kernel launch now
#pragma unroll
    for (int s = 0; s < STAGES; ++s) issue(t + s * G, s);
    for (int it = 0; t < tm.total; t += G, ++it) {
        const int s = it % STAGES;
        prefetch(t + G);
        cp_wait<STAGES - 1>();
        __syncthreads();
        int b, k, blk;
        tm.decode(t, b, k, blk);
        unsigned char* st = stage_ptr(s);
        const TWD* NEG = reinterpret_cast<const TWD*>(st);
        const double q = NEG[0].w, qinv = NEG[0].wq;      // entry 0 of the table holds (q, 1/q)
        const TWD* TW1 = NEG + R;
        const TWD* CYC = NEG + R + R * R;
        const TWD* sA = NEG + CF::NS;
        const TWD* sB = sA + C * R;
        double* sD = reinterpret_cast<double*>(st + (CF::NS + CF::NO) * sizeof(TWD));
        double* S = sD + c * CF::XP;
        const int n2 = blk * C + c;
        u64* dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * NN;
        double x[R];
        if (FWD) {
            if (rs.src_dead && tid < N1)                   // a dead source (BConv output): drop its lines
                discard_line(rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN + (size_t)tid * N2 + blk * C);
            if (rs.in_lazy) {                              // lazy doubles (BConv outputs), |x| < 2^40
#pragma unroll
                for (int na = 0; na < R; ++na) x[na] = sD[(R * na + r) * C + c];
            } else {
                const u64* d64 = reinterpret_cast<const u64*>(sD);
#pragma unroll
                for (int na = 0; na < R; ++na) x[na] = u2d(d64[(R * na + r) * C + c]);
            }
            if (rs.sub) {                                  // - sub (KLSS ModDown: conv - acc_Q), |x| < 2^40 + q
                const u64* sr = rs.sub + b * rs.sub_bstride + (size_t)k * NN + n2;
                u64 sv[R];
#pragma unroll
                for (int na = 0; na < R; ++na) sv[na] = __ldg(sr + (size_t)(R * na + r) * N2);
#pragma unroll
                for (int na = 0; na < R; ++na) x[na] = __dadd_rn(x[na], -u2d(sv[na]));
            }
            if (rs.fold) {                                 // + [c_l]_{q_i} * (P mod q_i): |x| < 2^40 + q
                const u64* fr = rs.fold + (size_t)b * NN + n2;
                u64 fv[R];
#pragma unroll
                for (int na = 0; na < R; ++na) fv[na] = __ldg(fr + (size_t)(R * na + r) * N2);
                const TWD fw = rs.scale[k];
#pragma unroll
                for (int na = 0; na < R; ++na) x[na] = __dadd_rn(x[na], mulc(u2d(fv[na]), fw, q));
            }
            neg_fwd<R>(x, NEG, q);
            __syncthreads();                               // tile consumed: exchange in place
#pragma unroll
            for (int ia = 0; ia < R; ++ia) S[ia * R + r] = mulc(x[BitRev<R>::of(ia)], TW1[r * R + ia], q);
            __syncthreads();
#pragma unroll
            for (int nb = 0; nb < R; ++nb) x[nb] = S[r * R + nb];
            cyc_dif<R>(x, CYC, q);
            const TWD ta = sA[r * C + c];
            double* dd = reinterpret_cast<double*>(dst);
            if (rs.l2hint == 2) {
                const uint64_t pol = l2_keep_policy();
#pragma unroll
                for (int ib = 0; ib < R; ++ib)
                    st_keep(dd + (size_t)(r + R * ib) * N2 + n2, mulc(mulc(x[BitRev<R>::of(ib)], ta, q), sB[ib * C + c], q),
                            pol);
            } else {
#pragma unroll
                for (int ib = 0; ib < R; ++ib)
                    dd[(size_t)(r + R * ib) * N2 + n2] = mulc(mulc(x[BitRev<R>::of(ib)], ta, q), sB[ib * C + c], q);
            }
        } else {
            if (rs.l2hint && tid < N1)                     // the intermediate's lines of this tile are dead now
                discard_line(rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN + (size_t)tid * N2 + blk * C);
            TWD ta = sA[r * C + c];
            if (rs.has_scale) {                            // fold a per-row constant (e.g. qhat^-1) into the twist
                double w = mulc(ta.w, rs.scale[k], q);
                w = w < 0.0 ? __dadd_rn(w, q) : w;
                ta = TWD{w, __dmul_rn(w, qinv)};
            }
#pragma unroll
            for (int ib = 0; ib < R; ++ib) x[ib] = mulc(mulc(sD[(r + R * ib) * C + c], ta, q), sB[ib * C + c], q);
            cyc_dif<R>(x, CYC, q);
            __syncthreads();
#pragma unroll
            for (int nb = 0; nb < R; ++nb) S[nb * R + r] = mulc(x[BitRev<R>::of(nb)], TW1[r * R + nb], q);
            __syncthreads();
#pragma unroll
            for (int j = 0; j < R; ++j) x[j] = S[r * R + BitRev<R>::of(j)];
            neg_inv<R>(x, NEG, q);
#pragma unroll
            for (int na = 0; na < R; ++na) dst[(size_t)(R * na + r) * N2 + n2] = d2u(canon(x[na], q, qinv));
        }
        __syncthreads();                                   // stage s free
        issue(t + STAGES * G, s);
    }
    cp_wait<0>();
}

// ------------------------------------------------------------------ row pass

template <int R>
struct RowCfg {
    static constexpr int NT = kC * R;
    static constexpr int NS = R / 2 + R * R;            // cyc, tw2
    static constexpr int EP = R + 1;                    // exchange: element (ia, nb) at ia + EP*nb
    static constexpr int XP = R * EP + 1;               // per-row region, odd
    static constexpr int N2 = R * R;
    static constexpr int DATA = (kC * XP > N2 * kC) ? kC * XP : N2 * kC;
    static constexpr size_t STAGE = (size_t)NS * sizeof(TWD) + (size_t)DATA * 8;
};

// Forward: src = lazy doubles tmp[i1][n2], dst = canonical u64 a_hat[i1 + N1 i2].
// Inverse: src = canonical u64 a_hat, dst = lazy doubles tmp[i1][n2].
template <int R, bool FWD, int STAGES, int MINB, bool EPI>
__global__ void __launch_bounds__(RowCfg<R>::NT, MINB)
k_ntt_row(RowSet rs, NttArgs a, TileMap tm, const __grid_constant__ RowEpi ep) {
    using CF = RowCfg<R>;
    constexpr int RR = kC, NT = CF::NT, N2 = CF::N2;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int tid = threadIdx.x, rho = tid / R, r = tid % R;
    constexpr int N1 = R * R;                   // compile-time strides: immediate address offsets
    constexpr long long NN = (long long)N1 * N1;

    auto stage_ptr = [&](int s) { return smem_raw + s * CF::STAGE; };
    auto issue = [&](int t, int s) {
        if (t < tm.total) {
            int b, k, blk;
            tm.decode(t, b, k, blk);
            const int lid = rs.prime[k];
            const TWD* ptab = a.tabd + (size_t)lid * a.tab_stride;
            unsigned char* st = stage_ptr(s);
            TWD* sT = reinterpret_cast<TWD*>(st);
            double* sD = reinterpret_cast<double*>(st + CF::NS * sizeof(TWD));
            const int off = FWD ? a.L.rowf_cyc : a.L.rowi_cyc;   // cyc, then tw2 [r][x] -> [x][r]
            for (int e = tid; e < CF::NS; e += NT) {
                int d = e;
                if (e >= R / 2) {
                    const int f = e - R / 2;
                    d = R / 2 + (f % R) * R + f / R;
                }
                cp16(sT + d, ptab + off + e);
            }
            const int row0 = blk * RR;
            const u64* src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN;
            if (FWD) {   // 16 contiguous rows
                const u64* g = src + (size_t)row0 * N2;
                for (int e = tid; e < RR * N2 / 2; e += NT) cp16(sD + 2 * e, g + 2 * e);
            } else {     // 128-byte segments a_hat[row0 .. row0+15 + N1 i2], swizzled
                for (int e = tid; e < N2 * 8; e += NT) {
                    const int i2 = e >> 3, p = e & 7;
                    cp16(sD + i2 * 16 + ((p ^ (i2 & 7)) << 1), src + row0 + (size_t)N1 * i2 + 2 * p);
                }
            }
        }
        cp_commit();
    };

    // L2 prefetch of the CTA's next tile (single-stage configurations) and of the fused
    // ModDown tail's acc / add rows of this tile (consumed only after the transform)
    auto prefetch = [&](int t, bool epi_rows) {
        if (t >= tm.total) return;
        int b, k, blk;
        tm.decode(t, b, k, blk);
        const int row0 = blk * RR;
        if (epi_rows) {
            const int bb = b >> 1, cc = b & 1;
            const u64* accr = ep.acc + bb * ep.acc_b + cc * ep.acc_c + (size_t)k * NN + row0;
            const u64* addr = cc ? ep.add1 : ep.add0;
            for (int i2 = tid; i2 < N2; i2 += NT) {
                if (ep.acc) pf_l2(accr + (size_t)N1 * i2);
                if (addr && !(cc == 0 && ep.add_galois))
                    pf_l2(addr + bb * ep.add_b + (size_t)k * NN + row0 + (size_t)N1 * i2);
            }
        } else if (STAGES == 1) {
            const u64* src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN;
            if (FWD)
                for (int e = tid; e < RR * N2 / 16; e += NT) pf_l2(src + (size_t)row0 * N2 + 16 * e);
            else
                for (int i2 = tid; i2 < N2; i2 += NT) pf_l2(src + row0 + (size_t)N1 * i2);
        }
    };

    const int G = gridDim.x;
    int t = blockIdx.x;
    pdl_wait();            // predecessor's writes visible (and its reads done) before any access
    pdl_trigger();         // persistent grid is fully resident: let the next kernel launch now
#pragma unroll
    for (int s = 0; s < STAGES; ++s) issue(t + s * G, s);
    for (int it = 0; t < tm.total; t += G, ++it) {
        const int s = it % STAGES;
        if (EPI) prefetch(t, true);
        prefetch(t + G, false);
        cp_wait<STAGES - 1>();
        __syncthreads();
        int b, k, blk;
        tm.decode(t, b, k, blk);
        unsigned char* st = stage_ptr(s);
        const TWD* CYC = reinterpret_cast<const TWD*>(st);
        const double q = CYC[0].w, qinv = CYC[0].wq;      // entry 0 of the table holds (q, 1/q)
        const TWD* TW2 = CYC + R / 2;
        double* sD = reinterpret_cast<double*>(st + CF::NS * sizeof(TWD));
        double* S = sD + rho * CF::XP;
        const int row0 = blk * RR, i1 = row0 + rho;
        u64* dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * NN;
        double x[R];
        if (FWD) {
            if (rs.l2hint)                                 // the intermediate's lines of this tile are dead now
                for (int e = tid; e < RR * N2 / 16; e += NT)
                    discard_line(rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN + (size_t)row0 * N2 + 16 * e);
#pragma unroll
            for (int na = 0; na < R; ++na) x[na] = sD[rho * N2 + R * na + r];
            cyc_dif<R>(x, CYC, q);
            __syncthreads();
#pragma unroll
            for (int ia = 0; ia < R; ++ia) S[ia + CF::EP * r] = mulc(x[BitRev<R>::of(ia)], TW2[ia * R + r], q);
            __syncthreads();
#pragma unroll
            for (int nb = 0; nb < R; ++nb) x[nb] = S[r + CF::EP * nb];
            cyc_dif<R>(x, CYC, q);
            __syncthreads();
            u64* T = reinterpret_cast<u64*>(sD);
#pragma unroll
            for (int ib = 0; ib < R; ++ib) T[swz(r + R * ib, rho)] = d2u(canon(x[BitRev<R>::of(ib)], q, qinv));
            __syncthreads();
            if (!EPI && rs.dst_keep) {
                const uint64_t pol = l2_keep_policy();
                for (int e = tid; e < N2 * 8; e += NT) {
                    const int i2 = e >> 3, p = e & 7;
                    const uint4 v = *reinterpret_cast<const uint4*>(T + i2 * 16 + ((p ^ (i2 & 7)) << 1));
                    asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;\n"
                                 ::"l"(dst + row0 + (size_t)N1 * i2 + 2 * p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w),
                                   "l"(pol) : "memory");
                }
            } else if (!EPI) {
                for (int e = tid; e < N2 * 8; e += NT) {
                    const int i2 = e >> 3, p = e & 7;
                    const uint4 v = *reinterpret_cast<const uint4*>(T + i2 * 16 + ((p ^ (i2 & 7)) << 1));
                    *reinterpret_cast<uint4*>(dst + row0 + (size_t)N1 * i2 + 2 * p) = v;
                }
            } else {      // fused ModDown tail (a10): out = (acc - conv) P^-1 (+ add)
                const int bb = b >> 1, cc = b & 1;
                const u64 qq = d2u(q);
                const TW pinv = ep.pinv[k];
                const u64* accr = ep.acc + bb * ep.acc_b + cc * ep.acc_c + (size_t)k * NN;
                const u64* addr = cc ? ep.add1 : ep.add0;
                if (addr) addr += bb * ep.add_b + (size_t)k * NN;
                u64* outr = (cc ? ep.out1 : ep.out0) + bb * ep.out_b + (size_t)k * NN;
                // 8 chunks of 2 coefficients per thread, in two rounds of 4 whose global loads are
                // all issued before any of their results is used (the loads' L2 latency overlaps)
                constexpr int U = 4;
                static_assert((N2 * 8) % (NT * U) == 0, "epilogue rounds");
                const bool gat = cc == 0 && ep.add_galois;
#pragma unroll 1
                for (int e0 = tid; e0 < N2 * 8; e0 += NT * U) {
                    uint4 av[U], dv[U];
                    size_t pos[U];
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        const int e = e0 + u * NT, i2 = e >> 3, p = e & 7;
                        pos[u] = row0 + (size_t)N1 * i2 + 2 * p;
                        av[u] = ep.acc ? __ldg(reinterpret_cast<const uint4*>(accr + pos[u]))
                                       : make_uint4(0u, 0u, 0u, 0u);        // acc = 0 (KLSS ModDown)
                        dv[u] = make_uint4(0u, 0u, 0u, 0u);
                        if (addr) {
                            if (gat) {                                       // sigma_g(c0), gathered
                                const unsigned gg = ep.add_galois, msk = (unsigned)NN - 1;
                                const unsigned s0 = (unsigned)(((unsigned long long)gg * pos[u] + (gg - 1) / 2) & msk);
                                const u64 x0 = __ldg(addr + s0), x1 = __ldg(addr + ((s0 + gg) & msk));
                                dv[u] = make_uint4((unsigned)x0, (unsigned)(x0 >> 32), (unsigned)x1, (unsigned)(x1 >> 32));
                            } else {
                                dv[u] = __ldg(reinterpret_cast<const uint4*>(addr + pos[u]));
                            }
                        }
                    }
#pragma unroll
                    for (int u = 0; u < U; ++u) {
                        const int e = e0 + u * NT, i2 = e >> 3, p = e & 7;
                        const uint4 v = *reinterpret_cast<const uint4*>(T + i2 * 16 + ((p ^ (i2 & 7)) << 1));
                        u64 r0 = shoup(sub_mod(((u64)av[u].y << 32) | av[u].x, ((u64)v.y << 32) | v.x, qq), pinv, qq);
                        u64 r1 = shoup(sub_mod(((u64)av[u].w << 32) | av[u].z, ((u64)v.w << 32) | v.z, qq), pinv, qq);
                        r0 = add_mod(r0, ((u64)dv[u].y << 32) | dv[u].x, qq);       // add = 0 when absent
                        r1 = add_mod(r1, ((u64)dv[u].w << 32) | dv[u].z, qq);
                        if (ep.has_post) {                       // fused Rescale: x q_l^-1 (uniform branch)
                            const TW post = ep.post[k];
                            r0 = shoup(r0, post, qq);
                            r1 = shoup(r1, post, qq);
                        }
                        *reinterpret_cast<uint4*>(outr + pos[u]) =
                            make_uint4((unsigned)r0, (unsigned)(r0 >> 32), (unsigned)r1, (unsigned)(r1 >> 32));
                    }
                }
            }
        } else {
            if (rs.src_dead)                               // a dead source (KeyIP's P rows): drop its lines
                for (int i2 = tid; i2 < N2; i2 += NT)
                    discard_line(rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * NN + row0 + (size_t)N1 * i2);
            const u64* T = reinterpret_cast<const u64*>(sD);
            int i1o = i1;                                  // row of tmp this thread's row lands in
            if (rs.galois) {
                // fused automorphism X -> X^g (HROTATE): output index i1o + N1 i2 reads source
                // index pi = g (i1o + N1 i2) + (g-1)/2 mod N = i1 + N1 ((kk + g i2) mod N2), with
                // i1 = (g i1o + (g-1)/2) mod N1 the source row this tile holds and kk = floor(s / N1)
                const unsigned g = rs.galois, cst = (g - 1) / 2;
                const unsigned ginv = rs.galois_inv_n1;
                i1o = (int)((ginv * (unsigned)(i1 + N1 - (int)(cst & (unsigned)(N1 - 1)))) & (unsigned)(N1 - 1));
                const unsigned s0 = (unsigned)(((unsigned long long)g * (unsigned)i1o + cst) & (unsigned long long)(NN - 1));
                const unsigned kk = s0 / (unsigned)N1;
#pragma unroll
                for (int ib = 0; ib < R; ++ib)
                    x[ib] = u2d(T[swz((int)((kk + g * (unsigned)(r + R * ib)) & (unsigned)(N2 - 1)), rho)]);
            } else {
#pragma unroll
                for (int ib = 0; ib < R; ++ib) x[ib] = u2d(T[swz(r + R * ib, rho)]);
            }
            cyc_dif<R>(x, CYC, q);
            __syncthreads();
#pragma unroll
            for (int nb = 0; nb < R; ++nb) S[r + CF::EP * nb] = mulc(x[BitRev<R>::of(nb)], TW2[nb * R + r], q);
            __syncthreads();
#pragma unroll
            for (int ia = 0; ia < R; ++ia) x[ia] = S[ia + CF::EP * r];
            cyc_dif<R>(x, CYC, q);
            double* dd = reinterpret_cast<double*>(dst);
            if (rs.l2hint == 2) {
                const uint64_t pol = l2_keep_policy();
#pragma unroll
                for (int na = 0; na < R; ++na) st_keep(dd + (size_t)i1o * N2 + R * na + r, x[BitRev<R>::of(na)], pol);
            } else {
#pragma unroll
                for (int na = 0; na < R; ++na) dd[(size_t)i1o * N2 + R * na + r] = x[BitRev<R>::of(na)];
            }
        }
        __syncthreads();
        issue(t + STAGES * G, s);
    }
    cp_wait<0>();
}

// ------------------------------------------------------------------ row pass + KeyIP (a5 + a6)
// ntt.h KipArgs.  Work items are (tile, i) with i over the ntr[k] transforms of the tile's
// target (at least one item per tile: with beta = 1 a Q target has only its own-digit term);
// the CTA walks its tiles in order, so the accumulator of item i > 0 is read back by the same
// thread that stored it in item i - 1 (plain loads, not the non-coherent path).
template <int R, int MINB, int U>
__global__ void __launch_bounds__(RowCfg<R>::NT, MINB)
k_ntt_row_kip(NttArgs a, TileMap tm, const __grid_constant__ KipArgs A) {
    using CF = RowCfg<R>;
    constexpr int RR = kC, NT = CF::NT, N2 = CF::N2;
    extern __shared__ __align__(16) unsigned char smem_raw[];
    const int tid = threadIdx.x, rho = tid / R, r = tid % R;
    constexpr int N1 = R * R;                   // compile-time strides
    constexpr long long N = (long long)N1 * N1;
    TWD* sT = reinterpret_cast<TWD*>(smem_raw);
    double* sD = reinterpret_cast<double*>(smem_raw + CF::NS * sizeof(TWD));

    auto issue = [&](int t, int i) {
        if (t < tm.total) {
            int b, k, blk;
            tm.decode(t, b, k, blk);
            if (A.ntr[k] > 0) {
                const TWD* ptab = a.tabd + (size_t)A.limb[k] * a.tab_stride;
                for (int e = tid; e < CF::NS; e += NT) {
                    int dd = e;
                    if (e >= R / 2) {
                        const int f = e - R / 2;
                        dd = R / 2 + (f % R) * R + f / R;
                    }
                    cp16(sT + dd, ptab + a.L.rowf_cyc + e);
                }
                const double* g = A.tmp + b * A.tmp_bstride + (size_t)A.row[k][i] * N + (size_t)blk * RR * N2;
                for (int e = tid; e < RR * N2 / 2; e += NT) cp16(sD + 2 * e, g + 2 * e);
            }
        }
        cp_commit();
    };
    auto next = [&](int t, int i, int& tn, int& in) {
        int b, k, blk;
        tm.decode(t, b, k, blk);
        const int items = A.ntr[k] > 0 ? A.ntr[k] : 1;
        if (i + 1 < items) { tn = t; in = i + 1; } else { tn = t + gridDim.x; in = 0; }
    };

    int t = blockIdx.x, i = 0;
    pdl_wait();
    pdl_trigger();
    issue(t, 0);
    while (t < tm.total) {
        int tn, in;
        next(t, i, tn, in);
        int b, k, blk;
        tm.decode(t, b, k, blk);
        const int row0 = blk * RR, nt = A.ntr[k], lid = A.limb[k];
        // L2 prefetch: this item's key rows (consumed after the transform) and the next item's tile
        const int j = nt > 0 ? A.dig[k][i] : -1;
        const int jo = i == 0 ? A.own[k] : -1;
        if (j >= 0)
            for (int i2 = tid; i2 < N2; i2 += NT)
                for (int c = 0; c < 2; ++c)
                    pf_l2(A.evk_lo + ((size_t)(2 * j + c) * A.evk_limbs + lid) * N + row0 + (size_t)N1 * i2);
        if (tn < tm.total) {
            int b2, k2, blk2;
            tm.decode(tn, b2, k2, blk2);
            if (A.ntr[k2] > 0) {
                const double* g = A.tmp + b2 * A.tmp_bstride + (size_t)A.row[k2][in] * N + (size_t)blk2 * RR * N2;
                for (int e = tid; e < RR * N2 / 16; e += NT) pf_l2(g + 16 * e);
            }
        }
        cp_wait<0>();
        __syncthreads();
        const u64* T = reinterpret_cast<const u64*>(sD);
        if (nt > 0) {
            const TWD* CYC = sT;
            const double q = CYC[0].w, qinv = CYC[0].wq;
            const TWD* TW2 = CYC + R / 2;
            double* S = sD + rho * CF::XP;
            double x[R];
#pragma unroll
            for (int na = 0; na < R; ++na) x[na] = sD[rho * N2 + R * na + r];
            cyc_dif<R>(x, CYC, q);
            __syncthreads();
#pragma unroll
            for (int ia = 0; ia < R; ++ia) S[ia + CF::EP * r] = mulc(x[BitRev<R>::of(ia)], TW2[ia * R + r], q);
            __syncthreads();
#pragma unroll
            for (int nb = 0; nb < R; ++nb) x[nb] = S[r + CF::EP * nb];
            cyc_dif<R>(x, CYC, q);
            __syncthreads();
            u64* Tw = reinterpret_cast<u64*>(sD);
#pragma unroll
            for (int ib = 0; ib < R; ++ib) Tw[swz(r + R * ib, rho)] = d2u(canon(x[BitRev<R>::of(ib)], q, qinv));
            __syncthreads();
        }
        // epilogue: acc_c = (i > 0 || accumulate ? acc_c : 0) + x * evk_{j,c} (+ dhat * evk_{own,c})
        {
            const ModQ m = A.mods[lid];
            const bool prev = i > 0 || A.accumulate;
            const size_t kr = (size_t)A.evk_limbs * N;
            const uint32_t* klo = A.evk_lo + ((size_t)(2 * (j < 0 ? 0 : j)) * A.evk_limbs + lid) * N;
            const uint8_t* khi = A.evk_hi + ((size_t)(2 * (j < 0 ? 0 : j)) * A.evk_limbs + lid) * N;
            const uint32_t* olo = A.evk_lo + ((size_t)(2 * (jo < 0 ? 0 : jo)) * A.evk_limbs + lid) * N;
            const uint8_t* ohi = A.evk_hi + ((size_t)(2 * (jo < 0 ? 0 : jo)) * A.evk_limbs + lid) * N;
            const u64* dsrc = A.d + b * A.d_bstride + (size_t)lid * N;
            u64* acc0 = A.acc + b * A.acc_bstride + (size_t)k * N;
            u64* acc1 = acc0 + A.acc_cstride;
            static_assert((N2 * 8) % (NT * U) == 0, "epilogue rounds");
#pragma unroll 1
            for (int e0 = tid; e0 < N2 * 8; e0 += NT * U) {
                uint2 kl0[U], kl1[U], ol0[U], ol1[U];
                unsigned kh[U], oh[U];
                uint4 p0[U], p1[U], dv[U];
                size_t pos[U];
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int e = e0 + u * NT, i2 = e >> 3, p = e & 7;
                    pos[u] = row0 + (size_t)N1 * i2 + 2 * p;
                    if (j >= 0) {
                        kl0[u] = __ldg(reinterpret_cast<const uint2*>(klo + pos[u]));
                        kl1[u] = __ldg(reinterpret_cast<const uint2*>(klo + kr + pos[u]));
                        kh[u] = (unsigned)__ldg(reinterpret_cast<const unsigned short*>(khi + pos[u])) |
                                ((unsigned)__ldg(reinterpret_cast<const unsigned short*>(khi + kr + pos[u])) << 16);
                    }
                    if (jo >= 0) {
                        ol0[u] = __ldg(reinterpret_cast<const uint2*>(olo + pos[u]));
                        ol1[u] = __ldg(reinterpret_cast<const uint2*>(olo + kr + pos[u]));
                        oh[u] = (unsigned)__ldg(reinterpret_cast<const unsigned short*>(ohi + pos[u])) |
                                ((unsigned)__ldg(reinterpret_cast<const unsigned short*>(ohi + kr + pos[u])) << 16);
                        if (A.galois) {                              // sigma_g(d), gathered
                            const unsigned gg = A.galois, msk = (unsigned)N - 1;
                            const unsigned s0 = (unsigned)(((unsigned long long)gg * pos[u] + (gg - 1) / 2) & msk);
                            const u64 x0 = __ldg(dsrc + s0), x1 = __ldg(dsrc + ((s0 + gg) & msk));
                            dv[u] = make_uint4((unsigned)x0, (unsigned)(x0 >> 32), (unsigned)x1, (unsigned)(x1 >> 32));
                        } else {
                            dv[u] = __ldg(reinterpret_cast<const uint4*>(dsrc + pos[u]));
                        }
                    }
                    if (prev) {
                        p0[u] = __ldcg(reinterpret_cast<const uint4*>(acc0 + pos[u]));   // ld.global.cg: coherent
                        p1[u] = __ldcg(reinterpret_cast<const uint4*>(acc1 + pos[u]));
                    }
                }
#pragma unroll
                for (int u = 0; u < U; ++u) {
                    const int e = e0 + u * NT, i2 = e >> 3, p = e & 7;
                    u64 xv[2] = {0, 0}, dd[2] = {0, 0};
                    if (nt > 0) {
                        const uint4 v = *reinterpret_cast<const uint4*>(T + i2 * 16 + ((p ^ (i2 & 7)) << 1));
                        xv[0] = ((u64)v.y << 32) | v.x;
                        xv[1] = ((u64)v.w << 32) | v.z;
                    }
                    if (jo >= 0) {
                        dd[0] = ((u64)dv[u].y << 32) | dv[u].x;
                        dd[1] = ((u64)dv[u].w << 32) | dv[u].z;
                    }
                    u64 rr[2][2];
#pragma unroll
                    for (int c = 0; c < 2; ++c) {
#pragma unroll
                        for (int h = 0; h < 2; ++h) {
                            u64 hi = 0, lo = 0;
                            if (j >= 0) {
                                const uint2 kl = c ? kl1[u] : kl0[u];
                                const u64 kv = (u64)(h ? kl.y : kl.x) | ((u64)((kh[u] >> (16 * c + 8 * h)) & 0xffu) << 32);
                                mac128(hi, lo, xv[h], kv);
                            }
                            if (jo >= 0) {
                                const uint2 ol = c ? ol1[u] : ol0[u];
                                const u64 ov = (u64)(h ? ol.y : ol.x) | ((u64)((oh[u] >> (16 * c + 8 * h)) & 0xffu) << 32);
                                mac128(hi, lo, dd[h], ov);
                            }
                            if (prev) {
                                const uint4 pv = c ? p1[u] : p0[u];
                                const u64 pw = h ? (((u64)pv.w << 32) | pv.z) : (((u64)pv.y << 32) | pv.x);
                                lo += pw;
                                hi += lo < pw;
                            }
                            rr[c][h] = barrett_reduce(hi, lo, m);
                        }
                    }
                    *reinterpret_cast<uint4*>(acc0 + pos[u]) =
                        make_uint4((unsigned)rr[0][0], (unsigned)(rr[0][0] >> 32), (unsigned)rr[0][1], (unsigned)(rr[0][1] >> 32));
                    *reinterpret_cast<uint4*>(acc1 + pos[u]) =
                        make_uint4((unsigned)rr[1][0], (unsigned)(rr[1][0] >> 32), (unsigned)rr[1][1], (unsigned)(rr[1][1] >> 32));
                }
            }
        }
        __syncthreads();
        issue(tn, in);
        t = tn;
        i = in;
    }
    cp_wait<0>();
}

// ------------------------------------------------------------------ launchers

// Pipeline depth / occupancy variant: 0 = 2 stages x 2 CTAs/SM, 1 = 1 stage x 3,
// 2 = 1 stage x 4 CTAs/SM (default: fastest on B200, bench of 2026-10-17 in DESIGN.md);
// NEO_NTT_CFG overrides for experiments.
static int ntt_cfg() {
    static int v = -1;
    if (v < 0) {
        const char* e = std::getenv("NEO_NTT_CFG");
        v = e ? std::atoi(e) : 2;
        if (v < 0 || v > 2) v = 2;
    }
    return v;
}

template <int R, bool FWD, int STAGES, int MINB>
static cudaError_t launch_cfg(bool col, const RowSet& rs, const NttArgs& a, int batch, cudaStream_t st,
                             const RowEpi* epi) {
    static bool init = false;
    const size_t smc = STAGES * ColCfg<R>::STAGE, smr = STAGES * RowCfg<R>::STAGE;
    if (!init) {
        cudaFuncSetAttribute(k_ntt_col<R, FWD, STAGES, MINB>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smc);
        cudaFuncSetAttribute(k_ntt_row<R, FWD, STAGES, MINB, false>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smr);
        cudaFuncSetAttribute(k_ntt_row<R, FWD, STAGES, MINB, true>, cudaFuncAttributeMaxDynamicSharedMemorySize,
                             (int)smr);
        init = true;
    }
    TileMap tm;
    tm.batch = batch;
    tm.tpr = col ? a.N2 / kC : a.N1 / kC;
    tm.tpr_log = 0;
    while ((1 << tm.tpr_log) < tm.tpr) ++tm.tpr_log;
    tm.bmagic = batch > 1 ? (unsigned)((1ull << 32) / (unsigned)batch + 1) : 0u;
    tm.total = tm.tpr * rs.n * batch;
    int grid = MINB * a.num_sms;
    if (grid > tm.total) grid = tm.total;
    if (col) {
        return launch_k(k_ntt_col<R, FWD, STAGES, MINB>, dim3(grid), dim3(ColCfg<R>::NT), smc, st, rs, a, tm);
    } else if (epi) {
        if (!FWD) return cudaErrorInvalidValue;
        return launch_k(k_ntt_row<R, FWD, STAGES, MINB, true>, dim3(grid), dim3(RowCfg<R>::NT), smr, st, rs, a, tm,
                        *epi);
    } else {
        static const RowEpi none{};
        return launch_k(k_ntt_row<R, FWD, STAGES, MINB, false>, dim3(grid), dim3(RowCfg<R>::NT), smr, st, rs, a, tm,
                        none);
    }
    return cudaGetLastError();
}

template <int R, bool FWD>
static cudaError_t launch_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, cudaStream_t st,
                               const RowEpi* epi) {
    switch (ntt_cfg()) {
        case 1: return launch_cfg<R, FWD, 1, 3>(col, rs, a, batch, st, epi);
        case 0: return launch_cfg<R, FWD, 2, 2>(col, rs, a, batch, st, epi);
        default: return launch_cfg<R, FWD, 1, 4>(col, rs, a, batch, st, epi);
    }
}

cudaError_t ntt_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st,
                     const RowEpi* epi) {
    if (rs.n == 0 || batch == 0) return cudaSuccess;
    switch (a.L.R) {
        case 8: return fwd ? launch_pass<8, true>(col, rs, a, batch, st, epi) : launch_pass<8, false>(col, rs, a, batch, st, epi);
        case 16: return fwd ? launch_pass<16, true>(col, rs, a, batch, st, epi) : launch_pass<16, false>(col, rs, a, batch, st, epi);
        default: return cudaErrorInvalidValue;
    }
}

// fused ModUp row pass + KeyIP: npos target positions x batch, 1 stage x 4 CTAs per SM
cudaError_t ntt_row_kip(const NttArgs& a, const KipArgs& A, int npos, int batch, cudaStream_t st) {
    if (npos == 0 || batch == 0) return cudaSuccess;
    TileMap tm;
    tm.batch = batch;
    tm.tpr = a.N1 / kC;
    tm.tpr_log = 0;
    while ((1 << tm.tpr_log) < tm.tpr) ++tm.tpr_log;
    tm.bmagic = batch > 1 ? (unsigned)((1ull << 32) / (unsigned)batch + 1) : 0u;
    tm.total = tm.tpr * npos * batch;
    auto go = [&](auto kern, int nt, size_t sm, int minb) -> cudaError_t {
        static bool init = false;
        if (!init) {
            cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
            init = true;
        }
        int grid = minb * a.num_sms;
        if (grid > tm.total) grid = tm.total;
        return launch_k(kern, dim3(grid), dim3(nt), sm, st, a, tm, A);
    };
    switch (a.L.R) {
        case 8: return go(k_ntt_row_kip<8, 4, 2>, RowCfg<8>::NT, RowCfg<8>::STAGE, 4);
        case 16: {
            // occupancy x loads-in-flight variant (NEO_KIP_CFG): 0 = 4 CTAs x 1 chunk, 1 = 3 x 2, 2 = 2 x 4
            static int v = -1;
            if (v < 0) {
                const char* e = std::getenv("NEO_KIP_CFG");
                v = e ? std::atoi(e) : 0;
            }
            if (v == 1) return go(k_ntt_row_kip<16, 3, 2>, RowCfg<16>::NT, RowCfg<16>::STAGE, 3);
            if (v == 2) return go(k_ntt_row_kip<16, 2, 4>, RowCfg<16>::NT, RowCfg<16>::STAGE, 2);
            return go(k_ntt_row_kip<16, 4, 1>, RowCfg<16>::NT, RowCfg<16>::STAGE, 4);
        }
        default: return cudaErrorInvalidValue;
    }
}

}  // namespace neo
