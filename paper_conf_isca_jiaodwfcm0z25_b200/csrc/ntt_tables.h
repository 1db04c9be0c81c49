// ntt_tables.h -- layout of the per-prime NTT twiddle block (host builder + device users).
//
// N = N1 * N2 with N1 = N2 = R*R (R = 16 for N = 2^16, R = 8 for N = 2^12).  The forward
// transform a_hat[i] = sum_n a[n] psi^((2i+1)n) (natural order, Z6) is factored as
// (n = N2*n1 + n2, i = i1 + N1*i2):
//   pass 1 (column kernel): negacyclic N1-point NTT over n1 with psi1 = psi^N2, then the
//                           twist T[i1][n2] = psi^((2 i1 + 1) n2)            (tmp[i1][n2])
//   pass 2 (row kernel)   : cyclic N2-point DFT over n2 with omega2 = psi^(2 N1),
//                           written to a_hat[i1 + N1*i2]
// and each N1/N2-point transform is itself R x R in registers with a shared-memory
// exchange.  Every table entry is a TWD {w, fl(w / q)} pair; entry 0 of the four
// neg / cyc tables (the unit twiddle, never multiplied by) holds {q, fl(1 / q)} instead.
#pragma once

struct NttLayout {
    int R, N1, N2;
    // small tables (copied to shared memory per CTA)
    int colf_neg, colf_tw1, colf_cyc;   // R, R*R, R/2
    int coli_neg, coli_tw1, coli_cyc;
    int rowf_cyc, rowf_tw2;             // R/2, R*R
    int rowi_cyc, rowi_tw2;
    int small_end;
    // outer twist, factored: T[r + R*ib][n2] = A[n2][r] * B[n2][ib]
    int outf_a, outf_b, outi_a, outi_b; // N2*R each
    int total;                           // entries per prime
};

inline NttLayout make_ntt_layout(int log_n) {
    NttLayout L;
    L.N1 = 1 << (log_n / 2);
    L.N2 = 1 << (log_n - log_n / 2);
    int r = 1;
    while (r * r < L.N1) r <<= 1;
    L.R = r;
    int R = r, o = 0;
    L.colf_neg = o; o += R;
    L.colf_tw1 = o; o += R * R;
    L.colf_cyc = o; o += R / 2;
    L.coli_neg = o; o += R;
    L.coli_tw1 = o; o += R * R;
    L.coli_cyc = o; o += R / 2;
    L.rowf_cyc = o; o += R / 2;
    L.rowf_tw2 = o; o += R * R;
    L.rowi_cyc = o; o += R / 2;
    L.rowi_tw2 = o; o += R * R;
    o = (o + 7) & ~7;
    L.small_end = o;
    L.outf_a = o; o += L.N2 * R;
    L.outf_b = o; o += L.N2 * R;
    L.outi_a = o; o += L.N2 * R;
    L.outi_b = o; o += L.N2 * R;
    L.total = o;
    return L;
}
