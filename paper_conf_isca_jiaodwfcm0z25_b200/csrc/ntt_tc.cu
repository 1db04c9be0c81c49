// ntt_tc.cu -- negacyclic NTT / INTT for N = 2^16 with the DFT stages on tcgen05 (sm_100a).
//
// Transform (Z6): a_hat[i] = sum_n a[n] psi^((2i+1)n), natural order in and out.  The 4-step
// split is the one of ntt.cu (n = n1 N2 + n2, i = i1 + N1 i2, N1 = N2 = 256): a column pass
// (negacyclic 256-point NTT over n1 with rho = psi^N2, then the twist psi^((2 i1 + 1) n2)) and
// a row pass (cyclic 256-point DFT over n2 with omega = psi^(2 N1)).  Neo replaces the
// radix-16 butterflies of each pass by matrix products (L438-450, Fig. 9 "Mul & Trans"); here
// every 256-point pass is two radix-16 stages, each ONE int8 GEMM on the tensor cores:
//
//   input p = p_a + 16 p_b, output o = o_a + 16 o_b, the tile's 16 independent transforms x:
//   stage 1 (vectors (p_a, x), K = p_b):  Z[p_a][o_a] = sum_p_b S1[o_a][p_b] x[p_a + 16 p_b]
//   twiddle:                               Z'         = Z * T[p_a][o_a]
//   stage 2 (vectors (o_a, x), K = p_a):  y[o_a + 16 o_b] = sum_p_a S2[o_b][p_a] Z'[p_a][o_a]
//
// with S1, T, S2 per pass (ntt_tc.h).  Each 36-bit operand is split into 5 bytes with the
// constant side pre-shifted, exactly as in bconv_tc.cu:
//   B[(b, o)][(p, a)] = byte_b((2^(8a) S[o][p]) mod q),  D_b = sum_(p,a) x^(a)_p B[(b,o)][(p,a)],
//   sum_b 2^(8b) D_b == sum_p S[o][p] x_p (mod q),
// one tcgen05.mma.kind::i8 of M = 128, N = 80 (5 bytes x 16 outputs), K = 96 (80 + zero pad)
// per 128 vectors.  D_0..3 < 80 * 255^2 < 2^23 and D_4 < 80 * 255 * 15 < 2^19, so
// V = sum_b 2^(8b) D_b < 2^51 is assembled exactly as the bits of the double 2^52 + V (three
// integer MADs) and reduced by ONE FP64 multiply-by-constant (common.cuh mulc), which also applies
// the twiddle: the epilogue never reduces V separately.  Between the stages the residue is stored
// back into the A operand as its low 32 bits and its top byte (values < 2^37 after + q).
//
// Kernel: persistent, 2 CTAs of 256 threads per SM, each CTA walks a contiguous range of tiles
// (16 transforms x 256 points; consecutive tiles share the prime, so the 19 KB of per-prime
// matrices are reloaded only when it changes).  Per tile: cp.async input (issued during the
// previous tile) -> producers (one thread per stage-1 vector) build A -> one thread issues 6
// MMAs (2 M-blocks x 3 K-steps) into TMEM -> epilogue 1 (one thread per TMEM lane: 80 columns,
// 16 outputs) writes A again -> 6 MMAs -> epilogue 2 (reduction, twist, stores).  Intermediates
// between the passes: forward = the 2^52-biased bits of a residue < 2^37 (u64), inverse = the
// double V < 2^51 (the next pass's FP64 multiply reduces it).
#include <cstdlib>
#include <cstring>

#include "common.cuh"
#include "ntt_tc.h"
#include "tc.cuh"

namespace neo {

// ------------------------------------------------------------------ host tables
static inline u64 h_mulm(u64 a, u64 b, u64 m) { return (u64)((u128)a * b % m); }
static u64 h_powm(u64 a, u64 e, u64 m) {
    u64 r = 1 % m;
    a %= m;
    for (; e; e >>= 1, a = h_mulm(a, a, m))
        if (e & 1) r = h_mulm(r, a, m);
    return r;
}

// SWIZZLE_NONE K-major image of an operand row n, K byte kk: core matrices of 8 rows x 16 B,
// LBO = 128 B between K chunks, SBO = 768 B between 8-row groups (6 K chunks per row).
static inline int op_off(int n, int kk) { return (n >> 3) * 768 + (kk >> 4) * 128 + (n & 7) * 16 + (kk & 15); }
// K index of input p's byte a: the low 4 bytes of p at 4p..4p+3, the top byte at 64 + p
static inline int kslot(int p, int a) { return a < 4 ? 4 * p + a : 64 + p; }

static void put_bmat(uint8_t* B, const u64 S[16][16], u64 q) {
    std::memset(B, 0, NTC_BMAT);
    for (int o = 0; o < 16; ++o)
        for (int p = 0; p < 16; ++p)
            for (int a = 0; a < 5; ++a) {
                const u64 c = h_mulm(S[o][p], (1ull << (8 * a)) % q, q);   // 2^(8a) S[o][p] mod q
                for (int b = 0; b < 5; ++b) B[op_off(16 * b + o, kslot(p, a))] = (uint8_t)(c >> (8 * b));
            }
}

bool make_ntt_tc_block(uint8_t* dst, u64 q, u64 psi, int N) {
    if (N != 65536 || (q >> 36) != 0 || (q >> 35) == 0) return false;
    const u64 ipsi = h_powm(psi, q - 2, q);
    const u64 rho = h_powm(psi, 256, q), irho = h_powm(ipsi, 256, q);   // primitive 512th roots
    const u64 om = h_powm(psi, 512, q), iom = h_powm(ipsi, 512, q);     // primitive 256th roots
    for (int pt = 0; pt < 4; ++pt) {
        u64 S1[16][16], S2[16][16], T[16][16];
        for (int o = 0; o < 16; ++o)
            for (int p = 0; p < 16; ++p) {
                switch (pt) {
                    case TC_COL_FWD:   // Y[o] = sum_p x[p] rho^((2o+1)p)
                        S1[o][p] = h_powm(rho, (u64)(16 * (2 * o + 1) * p) % 512, q);
                        T[p][o] = h_powm(rho, (u64)((2 * o + 1) * p) % 512, q);      // [p_a][o_a]
                        S2[o][p] = h_powm(rho, (u64)(32 * o * p) % 512, q);
                        break;
                    case TC_COL_INV:   // a[o] = sum_p Y[p] rho^-((2p+1)o)
                        S1[o][p] = h_powm(irho, (u64)(32 * o * p) % 512, q);
                        T[p][o] = h_powm(irho, (u64)((2 * p + 1) * o) % 512, q);
                        S2[o][p] = h_powm(irho, (u64)(16 * (2 * p + 1) * o) % 512, q);
                        break;
                    default: {         // cyclic DFT with omega (forward) or omega^-1 (inverse)
                        const u64 w = pt == TC_ROW_FWD ? om : iom;
                        S1[o][p] = h_powm(w, (u64)(16 * o * p) % 256, q);
                        T[p][o] = h_powm(w, (u64)(o * p) % 256, q);
                        S2[o][p] = h_powm(w, (u64)(16 * o * p) % 256, q);
                    }
                }
            }
        uint8_t* blk = dst + (size_t)pt * NTC_PASS_BYTES;
        put_bmat(blk, S1, q);
        put_bmat(blk + NTC_BMAT, S2, q);
        TWD* tw = reinterpret_cast<TWD*>(blk + 2 * NTC_BMAT);
        for (int pa = 0; pa < 16; ++pa)
            for (int oa = 0; oa < 16; ++oa) tw[pa * 16 + oa] = TWD{(double)T[pa][oa], (double)T[pa][oa] / (double)q};
    }
    return true;
}

// ------------------------------------------------------------------ device
namespace {

constexpr int kThr = 256;
constexpr int kAB = 256 * 96;                        // A operand: 256 vectors x 96 K bytes
constexpr int kTwB = 2 * 256 * 16;                   // twist A and B blocks of one column tile (TWD)
constexpr int kPitch = 260;                          // u64 per row of a [16][256] input tile
constexpr int kInB = 16 * kPitch * 8;                // >= 256 x 16 x 8
constexpr int kStgPitch = 257;                       // doubles per row of the inverse row pass's staging
// layout: A | twist[2] | S1 S2 T | input tile
constexpr int kOffTw = kAB;
constexpr int kOffTab = kOffTw + 2 * kTwB;
constexpr int kOffIn = kOffTab + NTC_PASS_BYTES;
constexpr size_t kSmem = (size_t)kOffIn + kInB;      // 93696 B: two CTAs per SM
static_assert(16 * kStgPitch * 8 <= kAB + 2 * kTwB, "staging of the inverse row pass fits over A + twist");
static_assert(kOffTab % 16 == 0 && kOffIn % 16 == 0, "16-byte alignment");

NEO_DEV uint32_t s_u32(const void* p) { return static_cast<uint32_t>(__cvta_generic_to_shared(p)); }
NEO_DEV void cp16(void* s, const void* g) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;\n" ::"r"(s_u32(s)), "l"(g) : "memory");
}
NEO_DEV void cp_commit() { asm volatile("cp.async.commit_group;\n" ::: "memory"); }
NEO_DEV void cp_wait_all() { asm volatile("cp.async.wait_group 0;\n" ::: "memory"); }

// [256][16] u64 tile, 16-byte chunks XOR-swizzled by the row's parity (conflict-free producers)
NEO_DEV int swz16(int row, int col) { return row * 16 + ((((col >> 1) ^ ((row & 1) << 2)) << 1) | (col & 1)); }

// V = sum_b 2^(8b) D_b < 2^51 as an exact double (bits of 2^52 + V)
NEO_DEV double vsum(uint32_t d0, uint32_t d1, uint32_t d2, uint32_t d3, uint32_t d4) {
    const u64 w = (u64)(d0 + (d1 << 8)) + (u64)(d2 + (d3 << 8)) * 65536ull;   // < 2^47.1
    return __dadd_rn(__hiloint2double((int)((uint32_t)(w >> 32) + d4 + 0x43300000u), (int)(uint32_t)w), -kTwo52);
}

NEO_DEV u64 dbits(double x) { return (u64)__double_as_longlong(x); }

}  // namespace

template <int PT>
__global__ void __launch_bounds__(kThr, 2)
k_ntt_tc(RowSet rs, NttArgs a, TileMap tm, const __grid_constant__ RowEpi ep, int epi) {
    extern __shared__ __align__(1024) uint8_t smem[];
    uint8_t* sA = smem;
    uint8_t* sTab = smem + kOffTab;
    const TWD* sT = reinterpret_cast<const TWD*>(sTab + 2 * NTC_BMAT);
    u64* sIn = reinterpret_cast<u64*>(smem + kOffIn);
    __shared__ uint64_t mbar;
    __shared__ uint32_t tmem_base;

    const int tid = threadIdx.x, warp = tid >> 5, lane = tid & 31;
    const int N = a.N, N1 = a.N1, N2 = a.N2;
    // stage-1 vector of this thread (= its A row and its TMEM lane): 4 consecutive p_a x 8
    // consecutive x per warp (conflict-free epilogue-1 stores)
    const int pa1 = 4 * (warp >> 1) + (lane & 3), x1 = 8 * (warp & 1) + (lane >> 2);
    // stage-2 vector of this thread: row m2 = 16 o_a + x
    const int oa2 = tid >> 4, x2 = tid & 15;
    const uint32_t taddr_lane = ((uint32_t)((warp & 3) * 32) << 16) + (uint32_t)((warp >> 2) * 128);

    if (warp == 0) tc::tmem_alloc(&tmem_base, 256);
    if (tid == 0) tc::mbar_init(&mbar, 1);
    tc::fence_before();
    __syncthreads();
    tc::fence_after();
    const uint32_t tmem = tmem_base;

    const int G = gridDim.x;
    const int t_beg = (int)((long long)blockIdx.x * tm.total / G);
    const int t_end = (int)((long long)(blockIdx.x + 1) * tm.total / G);

    auto issue_input = [&](int t) {   // input tile + twist blocks of tile t (its i-th of this CTA)
        int b, k, blk;
        tm.decode(t, b, k, blk);
        const int lid = rs.prime[k];
        const u64* src = rs.src + b * rs.src_bstride + (size_t)rs.src_off[k] * N;
        if (PT == TC_COL_FWD || PT == TC_COL_INV) {        // 256 rows x 16 columns
            const u64* g = src + blk * 16;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int e = tid + j * kThr, row = e >> 3, ch = e & 7;
                cp16(sIn + row * 16 + ((ch ^ ((row & 1) << 2)) << 1), g + (size_t)row * N2 + 2 * ch);
            }
            const TWD* ptab = a.tabd + (size_t)lid * a.tab_stride;
            TWD* tw = reinterpret_cast<TWD*>(smem + kOffTw + ((t - t_beg) & 1) * kTwB);
            const int oa = (PT == TC_COL_FWD ? a.L.outf_a : a.L.outi_a) + blk * 16 * 16;
            const int ob = (PT == TC_COL_FWD ? a.L.outf_b : a.L.outi_b) + blk * 16 * 16;
            cp16(tw + tid, ptab + oa + tid);              // [x][o_a or p_a]
            cp16(tw + 256 + tid, ptab + ob + tid);        // [x][o_b or p_b]
        } else if (PT == TC_ROW_FWD) {                     // 16 contiguous rows of 256
            const u64* g = src + (size_t)blk * 16 * N2;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int e = tid + j * kThr, x = e >> 7, ch = e & 127;
                cp16(sIn + x * kPitch + 2 * ch, g + (size_t)x * N2 + 2 * ch);
            }
        } else {                                            // 256 segments a_hat[row0 .. +15 + N1 i2]
            const u64* g = src + blk * 16;
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int e = tid + j * kThr, i2 = e >> 3, ch = e & 7;
                cp16(sIn + i2 * 16 + ((ch ^ ((i2 & 1) << 2)) << 1), g + (size_t)N1 * i2 + 2 * ch);
            }
        }
    };
    auto issue_tables = [&](int lid) {
        const uint8_t* g = a.tct + (size_t)lid * NTC_PRIME_BYTES + (size_t)PT * NTC_PASS_BYTES;
        for (int e = tid; e < NTC_PASS_BYTES / 16; e += kThr) cp16(sTab + 16 * e, g + 16 * e);
    };

    pdl_wait();
    pdl_trigger();
    int cur_lid = -1;
    if (t_beg < t_end) {
        int b, k, blk;
        tm.decode(t_beg, b, k, blk);
        cur_lid = rs.prime[k];
        issue_tables(cur_lid);
        issue_input(t_beg);
    }
    cp_commit();
    uint32_t phase = 0;
    const uint32_t idesc = tc::idesc_u8(128, 80);
    const uint32_t aS = tc::smem_u32(sA), bS1 = tc::smem_u32(sTab), bS2 = tc::smem_u32(sTab + NTC_BMAT);

    for (int t = t_beg; t < t_end; ++t) {
        int b, k, blk;
        tm.decode(t, b, k, blk);
        const int lid = rs.prime[k];
        const ModQ mq = a.mods[lid];
        const double q = mq.qd, qinv = mq.qinv, qp52 = __dadd_rn(q, kTwo52);
        const TWD* tw = reinterpret_cast<const TWD*>(smem + kOffTw + ((t - t_beg) & 1) * kTwB);
        cp_wait_all();
        __syncthreads();

        // ---------------------------------------------------------------- producers
        {
            uint32_t lo[16], hb[4] = {0u, 0u, 0u, 0u};
            TWD ta;
            if (PT == TC_COL_INV) {
                ta = tw[x1 * 16 + pa1];
                if (rs.has_scale) {                        // fold a per-row constant into the untwist
                    double w = mulc(ta.w, rs.scale[k], q);
                    w = w < 0.0 ? __dadd_rn(w, q) : w;
                    ta = TWD{w, __dmul_rn(w, qinv)};
                }
            }
            int kk = 0;
            if (PT == TC_ROW_INV && rs.galois) {           // source i2 of output i2: (kk + g i2) mod N2
                const unsigned g = rs.galois, cst = (g - 1) / 2;
                const int i1 = blk * 16 + x1;
                const unsigned i1o = (rs.galois_inv_n1 * (unsigned)(i1 + N1 - (int)(cst & (unsigned)(N1 - 1)))) &
                                     (unsigned)(N1 - 1);
                const unsigned s0 = (unsigned)(((unsigned long long)g * i1o + cst) & (unsigned long long)(N - 1));
                kk = (int)(s0 / (unsigned)N1);
            }
#pragma unroll
            for (int pb = 0; pb < 16; ++pb) {
                const int p = pa1 + 16 * pb;
                u64 v;
                if (PT == TC_COL_FWD) {
                    v = sIn[swz16(p, x1)];
                    if (rs.in_lazy) v = dbits(__dadd_rn(__longlong_as_double((long long)v), qp52));   // |x| <= q/2 + 1
                } else if (PT == TC_ROW_FWD) {
                    v = sIn[x1 * kPitch + p];
                } else if (PT == TC_ROW_INV) {
                    const int ps = rs.galois ? ((kk + (int)rs.galois * p) & 255) : p;
                    v = sIn[swz16(ps, x1)];
                } else {
                    const double d = __longlong_as_double((long long)sIn[swz16(p, x1)]);
                    v = dbits(__dadd_rn(mulc(mulc(d, ta, q), tw[256 + x1 * 16 + pb], q), qp52));
                }
                lo[pb] = (uint32_t)v;
                hb[pb >> 2] |= ((uint32_t)(v >> 32) & 0xFFu) << (8 * (pb & 3));
            }
            uint8_t* arow = sA + (tid >> 3) * 768 + (tid & 7) * 16;
#pragma unroll
            for (int j = 0; j < 4; ++j)
                *reinterpret_cast<uint4*>(arow + j * 128) = make_uint4(lo[4 * j], lo[4 * j + 1], lo[4 * j + 2], lo[4 * j + 3]);
            *reinterpret_cast<uint4*>(arow + 4 * 128) = make_uint4(hb[0], hb[1], hb[2], hb[3]);
        }
        tc::fence_proxy_async();
        __syncthreads();
        if (t + 1 < t_end) issue_input(t + 1);
        cp_commit();

        // ---------------------------------------------------------------- stage 1
        if (tid == 0) {
            tc::fence_after();
#pragma unroll
            for (int mb = 0; mb < 2; ++mb)
#pragma unroll
                for (int ks = 0; ks < 3; ++ks)
                    tc::mma_u8(tmem + mb * 128, tc::sdesc(aS + mb * 16 * 768 + ks * 256, 128, 768),
                               tc::sdesc(bS1 + ks * 256, 128, 768), idesc, ks > 0);
            tc::commit(&mbar);
        }
        tc::mbar_wait(&mbar, phase);
        phase ^= 1;
        tc::fence_after();

        // ---------------------------------------------------------------- epilogue 1 -> A
#pragma unroll
        for (int h = 0; h < 2; ++h) {
            TWD tw[8];                                         // loaded before the TMEM wait (latency overlap)
#pragma unroll
            for (int j = 0; j < 8; ++j) tw[j] = sT[pa1 * 16 + 8 * h + j];
            uint32_t v[5][8];
#pragma unroll
            for (int bb = 0; bb < 5; ++bb) tc::tmem_ld8(tmem + taddr_lane + (uint32_t)(bb * 16 + 8 * h), v[bb]);
            tc::tmem_wait_ld();
#pragma unroll
            for (int j = 0; j < 8; ++j) {
                const int oa = 8 * h + j;
                const double V = vsum(v[0][j], v[1][j], v[2][j], v[3][j], v[4][j]);
                const u64 z = dbits(__dadd_rn(mulc(V, tw[j], q), qp52));   // < 2^37 after + q
                uint8_t* row = sA + ((16 * oa + x1) >> 3) * 768 + (x1 & 7) * 16;
                *reinterpret_cast<uint32_t*>(row + (pa1 >> 2) * 128 + (pa1 & 3) * 4) = (uint32_t)z;
                row[4 * 128 + pa1] = (uint8_t)(z >> 32);
            }
        }
        tc::fence_proxy_async();
        tc::fence_before();
        __syncthreads();

        // ---------------------------------------------------------------- stage 2
        if (tid == 0) {
            tc::fence_after();
#pragma unroll
            for (int mb = 0; mb < 2; ++mb)
#pragma unroll
                for (int ks = 0; ks < 3; ++ks)
                    tc::mma_u8(tmem + mb * 128, tc::sdesc(aS + mb * 16 * 768 + ks * 256, 128, 768),
                               tc::sdesc(bS2 + ks * 256, 128, 768), idesc, ks > 0);
            tc::commit(&mbar);
        }
        tc::mbar_wait(&mbar, phase);
        phase ^= 1;
        tc::fence_after();
        if (t + 1 < t_end) {                               // S1 / S2 / T are free: next prime's tables
            int b2, k2, blk2;
            tm.decode(t + 1, b2, k2, blk2);
            const int lid2 = rs.prime[k2];
            if (lid2 != cur_lid) {
                issue_tables(lid2);
                cur_lid = lid2;
            }
        }
        cp_commit();

        // ---------------------------------------------------------------- epilogue 2
        if (PT == TC_COL_FWD || PT == TC_COL_INV) {
            u64* dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * N + blk * 16 + x2;
            const TWD tA = tw[x2 * 16 + oa2];
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                TWD tB[8];
                if (PT == TC_COL_FWD) {
#pragma unroll
                    for (int j = 0; j < 8; ++j) tB[j] = tw[256 + x2 * 16 + 8 * h + j];
                }
                uint32_t v[5][8];
#pragma unroll
                for (int bb = 0; bb < 5; ++bb) tc::tmem_ld8(tmem + taddr_lane + (uint32_t)(bb * 16 + 8 * h), v[bb]);
                tc::tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 8; ++j) {
                    const int ob = 8 * h + j;
                    const double V = vsum(v[0][j], v[1][j], v[2][j], v[3][j], v[4][j]);
                    u64 outv;
                    if (PT == TC_COL_FWD)              // twist psi^((2 i1 + 1) n2) = A[n2][o_a] B[n2][o_b]
                        outv = dbits(__dadd_rn(mulc(mulc(V, tA, q), tB[j], q), qp52));
                    else
                        outv = d2u(canon(V, q, qinv));
                    dst[(size_t)(oa2 + 16 * ob) * N2] = outv;
                }
            }
        } else if (PT == TC_ROW_FWD) {
            const int row0 = blk * 16;
            const size_t pos0 = (size_t)row0 + x2 + (size_t)N1 * oa2;   // + N1 * 16 o_b
            if (!epi) {
                u64* dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * N + pos0;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    uint32_t v[5][8];
#pragma unroll
                    for (int bb = 0; bb < 5; ++bb) tc::tmem_ld8(tmem + taddr_lane + (uint32_t)(bb * 16 + 8 * h), v[bb]);
                    tc::tmem_wait_ld();
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        const int ob = 8 * h + j;
                        dst[(size_t)N1 * 16 * ob] = d2u(canon(vsum(v[0][j], v[1][j], v[2][j], v[3][j], v[4][j]), q, qinv));
                    }
                }
            } else {      // fused ModDown tail (a10): out = (acc - conv) P^-1 (+ add) (x post)
                const int bb = b >> 1, cc = b & 1;
                const u64 qq = mq.q;
                const TW pinv = ep.pinv[k];
                const u64* accr = ep.acc ? ep.acc + bb * ep.acc_b + cc * ep.acc_c + (size_t)k * N : nullptr;
                const u64* addr = cc ? ep.add1 : ep.add0;
                if (addr) addr += bb * ep.add_b + (size_t)k * N;
                u64* outr = (cc ? ep.out1 : ep.out0) + bb * ep.out_b + (size_t)k * N;
                const bool gat = cc == 0 && ep.add_galois;
#pragma unroll
                for (int h = 0; h < 2; ++h) {
                    u64 av[8], dv[8];
#pragma unroll
                    for (int j = 0; j < 8; ++j) {             // operand loads first: their latency overlaps the TMEM reads
                        const size_t pos = pos0 + (size_t)N1 * 16 * (8 * h + j);
                        av[j] = accr ? __ldg(accr + pos) : 0ull;
                        dv[j] = 0ull;
                        if (addr) {
                            if (gat) {
                                const unsigned gg = ep.add_galois;
                                dv[j] = __ldg(addr + (size_t)(((unsigned long long)gg * pos + (gg - 1) / 2) & (unsigned long long)(N - 1)));
                            } else {
                                dv[j] = __ldg(addr + pos);
                            }
                        }
                    }
                    uint32_t v[5][8];
#pragma unroll
                    for (int b5 = 0; b5 < 5; ++b5) tc::tmem_ld8(tmem + taddr_lane + (uint32_t)(b5 * 16 + 8 * h), v[b5]);
                    tc::tmem_wait_ld();
#pragma unroll
                    for (int j = 0; j < 8; ++j) {
                        const size_t pos = pos0 + (size_t)N1 * 16 * (8 * h + j);
                        const u64 conv = d2u(canon(vsum(v[0][j], v[1][j], v[2][j], v[3][j], v[4][j]), q, qinv));
                        u64 r = shoup(sub_mod(av[j], conv, qq), pinv, qq);
                        r = add_mod(r, dv[j], qq);
                        if (ep.has_post) r = shoup(r, ep.post[k], qq);
                        outr[pos] = r;
                    }
                }
            }
        } else {   // TC_ROW_INV: V (< 2^51, a double the next pass's multiply reduces) via staging
            tc::fence_before();
            __syncthreads();                                   // every thread is past its A / twist reads
            double* stg = reinterpret_cast<double*>(smem);     // [16][kStgPitch] over A + twist
#pragma unroll
            for (int h = 0; h < 2; ++h) {
                uint32_t v[5][8];
#pragma unroll
                for (int bb = 0; bb < 5; ++bb) tc::tmem_ld8(tmem + taddr_lane + (uint32_t)(bb * 16 + 8 * h), v[bb]);
                tc::tmem_wait_ld();
#pragma unroll
                for (int j = 0; j < 8; ++j) stg[x2 * kStgPitch + oa2 + 16 * (8 * h + j)] = vsum(v[0][j], v[1][j], v[2][j], v[3][j], v[4][j]);
            }
            __syncthreads();
            u64* dst = rs.dst + b * rs.dst_bstride + (size_t)rs.dst_off[k] * N;
            const unsigned g = rs.galois, cst = (g - 1) / 2;
#pragma unroll 4
            for (int e = tid; e < 16 * 256; e += kThr) {
                const int x = e >> 8, n2 = e & 255;
                int i1o = blk * 16 + x;
                if (g) i1o = (int)((rs.galois_inv_n1 * (unsigned)(i1o + N1 - (int)(cst & (unsigned)(N1 - 1)))) & (unsigned)(N1 - 1));
                dst[(size_t)i1o * N2 + n2] = dbits(stg[x * kStgPitch + n2]);
            }
        }
        tc::fence_before();
        __syncthreads();                                       // TMEM drained, A / staging free
    }
    cp_wait_all();
    if (warp == 0) tc::tmem_dealloc(tmem, 256);
}

template <int PT>
static cudaError_t launch_tc(const RowSet& rs, const NttArgs& a, int batch, cudaStream_t st, const RowEpi* epi) {
    static bool init = false;
    if (!init) {
        cudaFuncSetAttribute(k_ntt_tc<PT>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kSmem);
        init = true;
    }
    TileMap tm;
    tm.batch = batch;
    tm.tpr = 16;
    tm.tpr_log = 4;
    tm.bmagic = batch > 1 ? (unsigned)((1ull << 32) / (unsigned)batch + 1) : 0u;
    tm.total = tm.tpr * rs.n * batch;
    static const RowEpi none{};
    int grid = 2 * a.num_sms;
    if (grid > tm.total) grid = tm.total;
    return launch_k(k_ntt_tc<PT>, dim3(grid), dim3(kThr), kSmem, st, rs, a, tm, epi ? *epi : none, epi ? 1 : 0);
}

cudaError_t ntt_pass_tc(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st,
                        const RowEpi* epi) {
    if (rs.n == 0 || batch == 0) return cudaSuccess;
    if (a.N != 65536 || a.N1 != 256 || a.N2 != 256 || !a.tct) return cudaErrorInvalidValue;
    if (epi && !(fwd && !col)) return cudaErrorInvalidValue;
    if (col) return fwd ? launch_tc<TC_COL_FWD>(rs, a, batch, st, nullptr) : launch_tc<TC_COL_INV>(rs, a, batch, st, nullptr);
    return fwd ? launch_tc<TC_ROW_FWD>(rs, a, batch, st, epi) : launch_tc<TC_ROW_INV>(rs, a, batch, st, nullptr);
}

}  // namespace neo
