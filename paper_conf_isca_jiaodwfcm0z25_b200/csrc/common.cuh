// common.cuh -- shared device types and 36-bit modular arithmetic for libneo (sm_100a).
//
// Residues live in uint64 words, canonical in [0, q) at every kernel boundary, with
// q < 2^36 (WordSize 36, Table 4).  Two reductions are used:
//  * Shoup multiplication by a constant w (twiddles, BConv factors, P^-1 ...):
//      w' = floor(w * 2^64 / q);  r = a*w - umulhi(a, w')*q  in [0, 2q) for any a < 2^64.
//  * Barrett for a variable product / lazy sum X < 2^98:
//      mu = floor(2^98 / q);  qe = umulhi(X >> 34, mu)  in [X/q - 2, X/q]  => r in [0, 3q).
#pragma once
#include <cstdint>
#include <cuda_runtime.h>

typedef uint64_t u64;
typedef unsigned __int128 u128;

struct TW {   // a constant with its Shoup companion
    u64 w, ws;
};

struct ModQ {  // per-limb modulus constants
    u64 q;
    u64 mu;    // floor(2^98 / q)
};

#define NEO_DEV __device__ __forceinline__

NEO_DEV u64 shoup_lazy(u64 a, u64 w, u64 ws, u64 q) {
    u64 hi = __umul64hi(a, ws);
    return a * w - hi * q;                      // [0, 2q)
}
NEO_DEV u64 shoup(u64 a, TW t, u64 q) {
    u64 r = shoup_lazy(a, t.w, t.ws, q);
    return r >= q ? r - q : r;
}
NEO_DEV u64 add_mod(u64 a, u64 b, u64 q) {
    u64 s = a + b;
    return s >= q ? s - q : s;
}
NEO_DEV u64 sub_mod(u64 a, u64 b, u64 q) { return a >= b ? a - b : a + q - b; }

// X = hi:lo < 2^98  ->  X mod q
NEO_DEV u64 barrett_reduce(u64 hi, u64 lo, ModQ m) {
    u64 x = (hi << 30) | (lo >> 34);            // X >> 34  (< 2^64)
    u64 qe = __umul64hi(x, m.mu);
    u64 r = lo - qe * m.q;                      // true value < 3q < 2^38: low word is exact
    r = r >= m.q ? r - m.q : r;
    return r >= m.q ? r - m.q : r;
}
NEO_DEV u64 mul_mod(u64 a, u64 b, ModQ m) {     // a, b < 2^62 with a*b < 2^98
    return barrett_reduce(__umul64hi(a, b), a * b, m);
}
// 128-bit accumulator helpers
NEO_DEV void mac128(u64& hi, u64& lo, u64 a, u64 b) {
    u64 l = a * b, h = __umul64hi(a, b);
    lo += l;
    hi += h + (lo < l);
}

// ---------------------------------------------------------------------------
// Batched limb-row descriptor: one kernel launch covers `batch x n` polynomial rows;
// row k of batch entry b lives at base + b*bstride + off[k]*N and is reduced mod the
// prime of limb id prime[k].
constexpr int NEO_MAX_ROWS = 160;

struct RowSet {
    const u64* src;
    u64* dst;
    long long src_bstride, dst_bstride;   // elements between batch entries
    int n;                                 // rows per batch entry
    int src_off[NEO_MAX_ROWS];
    int dst_off[NEO_MAX_ROWS];
    short prime[NEO_MAX_ROWS];
};

template <int R>
struct BitRev {
    static constexpr int log = (R == 2) ? 1 : (R == 4) ? 2 : (R == 8) ? 3 : (R == 16) ? 4 : (R == 32) ? 5 : 0;
    static __host__ __device__ constexpr int of(int x) {
        int y = 0;
        for (int b = 0; b < log; ++b) y |= ((x >> b) & 1) << (log - 1 - b);
        return y;
    }
};
