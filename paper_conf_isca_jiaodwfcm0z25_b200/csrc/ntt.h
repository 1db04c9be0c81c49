// ntt.h -- launch interface of the two NTT passes (see ntt.cu, ntt_tables.h).
#pragma once
#include "common.cuh"
#include "ntt_tables.h"

namespace neo {

// rows (b, k) in limb-major order: consecutive tiles share a prime
struct TileMap {        // rows (b, k) in limb-major order: consecutive tiles share a prime
    int batch, tpr, total;
    int tpr_log;            // tpr = 2^tpr_log
    unsigned bmagic;        // floor(2^32 / batch) + 1 (batch > 1): exact for ri * batch < 2^32
    NEO_DEV void decode(int t, int& b, int& k, int& blk) const {
        const int ri = t >> tpr_log;
        blk = t & (tpr - 1);
        k = (batch == 1) ? ri : (int)__umulhi((unsigned)ri, bmagic);
        b = ri - k * batch;
    }
};

struct NttArgs {
    const TWD* tabd;      // device: [limb id][L.total] twiddle blocks (w, w/q) in FP64
    long long tab_stride; // = L.total
    const ModQ* mods;     // device: per limb id
    int N, N1, N2;
    int num_sms;          // persistent grid = 2 CTAs per SM
    NttLayout L;
    const uint8_t* tct = nullptr;   // device: tensor-core pass tables [limb id][NTC_PRIME_BYTES] (ntt_tc.h), or null
};

// Optional epilogue of the forward row pass for the ModDown NTT (a9 + a10 fused):
// instead of storing conv = NTT(...) the pass stores, for batch index bc = 2b + c and row k,
//   out_c[b][k] = (acc[b][c][k] - conv) * P^-1 mod q  (+ add_c[b][k])
struct RowEpi {
    const u64* acc;
    long long acc_b, acc_c;
    const u64* add0;
    const u64* add1;
    long long add_b;
    u64* out0;
    u64* out1;
    long long out_b;
    unsigned add_galois;  // != 0: the addend of component 0 is sigma_g(add0), gathered on the fly
    int has_post = 0;     // != 0: the result is further multiplied by post[k] (fused HMULT + Rescale)
    TW pinv[64];          // per row k
    TW post[64];          // per row k: q_l^-1 mod q_k
};

// KeyIP fused into the forward row pass of the ModUp NTT (a5 + a6): one tile = 16 rows x N2
// of ONE target limb (position k of PQ_l) of one batch entry; the CTA transforms that tile of
// each digit j whose ModUp output reaches k (ntr[k] of them, column-pass intermediates in tmp)
// and accumulates acc_c[k] = sum_j NTT(up_j[k]) * evk_{j,c}[k] (+ dhat[k] * evk_{own,c}[k] for
// the digit that owns k) in its epilogue, so the ModUp outputs never reach HBM (Alg. 3).
constexpr int KIP_MAX_EXT = 64;
constexpr int KIP_MAX_BETA = 12;
struct KipArgs {
    const double* tmp;          // column-pass output [B][rows][N] (lazy doubles)
    long long tmp_bstride;
    const u64* d;               // KS input [B][l+1][N] in NTT form (the own-digit term)
    long long d_bstride;
    unsigned galois;            // != 0: the own-digit term reads sigma_g(d) (fused HROTATE)
    const uint32_t* evk_lo;     // [dnum][2][evk_limbs][N]
    const uint8_t* evk_hi;
    int evk_limbs;
    u64* acc;                   // [B][2][E][N]
    long long acc_bstride, acc_cstride;
    const ModQ* mods;
    int accumulate;             // acc += (neo_hrot_sum's giant steps)
    int limb[KIP_MAX_EXT];      // position -> limb id
    signed char ntr[KIP_MAX_EXT];                // transformed digits reaching position k
    signed char own[KIP_MAX_EXT];                // digit owning position k, or -1
    unsigned char dig[KIP_MAX_EXT][KIP_MAX_BETA];   // digit of the i-th transform of k
    short row[KIP_MAX_EXT][KIP_MAX_BETA];           // its row in tmp
};
cudaError_t ntt_row_kip(const NttArgs& a, const KipArgs& A, int npos, int batch, cudaStream_t st);

// One pass over batch x rs.n limb rows.  Forward NTT = column pass (src -> tmp) then row
// pass (tmp -> dst); inverse = row pass then column pass.  src and dst of one pass must
// not overlap.
cudaError_t ntt_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st,
                     const RowEpi* epi = nullptr);

}  // namespace neo
