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
#include <utility>
#include <cuda_runtime.h>

typedef uint64_t u64;
typedef unsigned __int128 u128;

struct TW {   // a constant with its Shoup companion
    u64 w, ws;
};

struct ModQ {  // per-limb modulus constants
    u64 q;
    u64 mu;    // floor(2^98 / q)
    double qd, qinv;   // q and fl(1/q)
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
// ---------------------------------------------------------------------------
// FP64 residue arithmetic.  A residue (or a lazy, signed representative of one) is held
// exactly in a double while |x| < 2^50.  Multiplication by a constant w < q uses the pair
// (w, wq = fl(w/q)):  h = fl(a w), l = a w - h (exact, FMA), qf = round(a wq) (magic-number
// rounding), r = (h - qf q) + l.  For integral |a| < 2^45 every step is exact except the
// quotient estimate, |qf - a w / q| <= 0.625, so r == a w (mod q) with |r| <= 0.625 q.
// (DESIGN.md "FP64 residue arithmetic".)  sm_100a issues 63 DFMA/clk/SM vs ~2.2 64-bit
// integer Shoup butterflies/clk/SM (tools/microbench/pipes.cu), hence FP64.
struct TWD {   // constant w < q and fl(w / q)
    double w, wq;
};
constexpr double kMagic = 6755399441055744.0;      // 1.5 * 2^52: fma(x, y, M) - M = round(x y)
constexpr double kTwo52 = 4503599627370496.0;

NEO_DEV double u2d(u64 x) {                         // exact for x < 2^52
    return __dadd_rn(__longlong_as_double((long long)(x | 0x4330000000000000ull)), -kTwo52);
}
NEO_DEV u64 d2u(double r) {                         // 0 <= r < 2^52, integral
    return (u64)__double_as_longlong(__dadd_rn(r, kTwo52)) - 0x4330000000000000ull;
}
NEO_DEV double mulc(double a, TWD t, double q) {    // a * w mod q, |result| <= 0.625 q
    const double h = __dmul_rn(a, t.w);
    const double l = __fma_rn(a, t.w, -h);
    const double qf = __dadd_rn(__fma_rn(a, t.wq, kMagic), -kMagic);
    return __dadd_rn(__fma_rn(-qf, q, h), l);
}
NEO_DEV double mulv(double a, double b, double q, double qinv) {   // a * b mod q, |a|,|b| < 2^37
    const double h = __dmul_rn(a, b);
    const double l = __fma_rn(a, b, -h);
    const double qf = __dadd_rn(__fma_rn(h, qinv, kMagic), -kMagic);
    return __dadd_rn(__fma_rn(-qf, q, h), l);
}
NEO_DEV double canon(double x, double q, double qinv) {   // |x| < 2^50 integral -> [0, q)
    const double qf = __dadd_rn(__fma_rn(x, qinv, kMagic), -kMagic);
    const double r = __fma_rn(-qf, q, x);                   // exact, |r| <= q/2 + 1 < q
    return __dadd_rn(r, r < 0.0 ? q : 0.0);                 // branch-free: selects, one DADD
}

// 128-bit accumulator helpers
NEO_DEV void mac128(u64& hi, u64& lo, u64 a, u64 b) {
    u64 l = a * b, h = __umul64hi(a, b);
    lo += l;
    hi += h + (lo < l);
}

// ---------------------------------------------------------------------------
// Programmatic dependent launch (PDL): kernels are launched with programmatic stream
// serialization so a kernel's launch and constant-table prologue overlap its predecessor's
// tail; pdl_wait() must precede every access to data another kernel writes or reads.
NEO_DEV void pdl_wait() { asm volatile("griddepcontrol.wait;\n" ::: "memory"); }
NEO_DEV void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;\n" ::: "memory"); }

bool neo_pdl_enabled();   // NEO_PDL=1 enables (launch.cu); griddepcontrol.* are no-ops otherwise

bool neo_pdl_bconv();      // NEO_PDL=2: programmatic dependent launch for the BConv launches only (launch.cu)

template <typename... KArgs, typename... Args>
inline cudaError_t launch_k_pdl(bool pdl, void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem,
                                cudaStream_t st, Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = pdl ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
}

template <typename... KArgs, typename... Args>
inline cudaError_t launch_k(void (*kernel)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t st,
                            Args&&... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = st;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = neo_pdl_enabled() ? 1 : 0;
    return cudaLaunchKernelEx(&cfg, kernel, std::forward<Args>(args)...);
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
    int in_lazy;                           // forward column pass: src holds lazy doubles |x| < 2^40
    int has_scale;                         // inverse column pass: multiply row k by scale[k]
    unsigned galois;                       // inverse row pass: read sigma_g(src) (X -> X^g, NTT domain); 0 = none
    unsigned galois_inv_n1;                //   g^-1 mod N1
    int dst_keep = 0;                      // second (row) pass, no epilogue: the output is read again soon
                                           //   (the ModUp rows KeyIP reads next): stored L2 evict_last
    int src_dead = 0;                      // first pass: the source rows are dead once read (a BConv output,
                                           //   KeyIP's P rows): their L2 lines are discarded, no write-back
    int l2hint = 0;                        // the pass's intermediate side (first pass: dst, second: src):
                                           //   stores keep it in L2 (evict_last), the consumer discards its
                                           //   lines after reading them (no write-back of dead data)
    const u64* sub = nullptr;              // forward column pass: x -= sub[b][k][n] (canonical, row k of
    long long sub_bstride = 0;             //   batch entry b at sub + b * sub_bstride + k * N), or nullptr
    const u64* fold = nullptr;             // forward column pass: x += [fold[b][n]] * scale[k] (fused
                                           //   HMULT + Rescale: conv_i + P c_l), canonical mod the row's
                                           //   limb ... or nullptr; fold row b of batch entry b, stride N
    int src_off[NEO_MAX_ROWS];
    int dst_off[NEO_MAX_ROWS];
    short prime[NEO_MAX_ROWS];
    TWD scale[NEO_MAX_ROWS];               // (w, w/q) per row
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
