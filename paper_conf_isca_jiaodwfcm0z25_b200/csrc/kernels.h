// kernels.h -- argument blocks and launchers of the streaming kernels (kernels.cu).
#pragma once
#include "context.h"

namespace neo {

constexpr int KS_MAX_EXT = 64;
constexpr int KS_MAX_BETA = 12;

struct KeyIPArgs {
    const u64* d;          // KS input [B][l+1][N] (NTT form)
    const u64* up;         // ModUp outputs after NTT [B][beta][E][N]
    const uint32_t* evk_lo;   // [dnum][2][evk_limbs][N] low 32 bits of each key residue
    const uint8_t* evk_hi;    // [dnum][2][evk_limbs][N] bits 32..39
    u64* acc;              // [B][2][E][N]
    const ModQ* mods;
    long long d_bstride, up_bstride, acc_bstride, acc_cstride;
    int N, beta, evk_limbs;
    unsigned galois;                         // != 0: rows of kind 0 (d) are read as sigma_g(d)
    int accumulate = 0;                      // != 0: acc += (sum over the giant steps, neo_hrot_sum)
    int limb[KS_MAX_EXT];                    // position -> limb id
    unsigned char src_kind[KS_MAX_BETA][KS_MAX_EXT];   // 0: d, 1: up
    int src_off[KS_MAX_BETA][KS_MAX_EXT];    // row (in N units) inside the chosen buffer
};

struct CombineArgs {
    const u64* acc;        // [B][2][E][N]; Q limbs are positions 0..l
    const u64* conv;       // [2B][l+1][N]
    const u64* add0;       // optional [B][..][N] addend of component 0 (nullptr: none)
    const u64* add1;
    u64* out0;
    u64* out1;
    const ModQ* mods;
    long long acc_bstride, acc_cstride, conv_stride, add_bstride, out_bstride;
    int N;
    TW pinv[64];           // per position
    int limb[64];          // position -> limb id (modulus)
};


// Element-wise ciphertext ops (L133-135) on [batch][2][limbs][N] ciphertexts and
// [batch][limbs][N] plaintexts, NTT form.
enum EwOp { EW_PMULT = 0, EW_HADD = 1, EW_PADD = 2, EW_HSUB = 3 };
struct EwArgs {
    const u64* a;          // ct [B][2][limbs][N]
    const u64* b;          // ct (HADD) or plaintext [B][limbs][N]
    u64* out;              // ct [B][2][limbs][N]
    const ModQ* mods;
    int N, limbs, op;
};

// Plaintext inner product: out[b] = sum_k PMULT(ct[k][b], pt[k][b or 0]) (neo_pmult_acc)
constexpr int NEO_MAX_ACC = 32;
struct PmaccArgs {
    const u64* ct[NEO_MAX_ACC];   // each [B][2][limbs][N]
    const u64* pt[NEO_MAX_ACC];   // each [B][limbs][N], or [limbs][N] when pt_shared
    u64* out;                     // [B][2][limbs][N]
    const ModQ* mods;
    int N, limbs, n_terms, pt_shared;
};

// Limb-subset element-wise operations (neo_ew_limbs; the limb-sharded evaluator): row k of
// every polynomial is reduced mod q_{lid[k]}.
enum EwlOp { EWL_HADD = 0, EWL_HSUB = 1, EWL_PMULT = 2, EWL_PADD = 3, EWL_TENSOR = 4, EWL_SUBMUL = 5, EWL_LIFT = 6 };
struct EwlArgs {
    const u64* a;          // ct [B][2][n][N]  (LIFT: coefficient rows [B][2][N] mod q_src)
    const u64* b;          // ct [B][2][n][N] or pt [B][n][N]
    u64* out;              // ct [B][2][n][N] (TENSOR: d [B][3][n][N])
    const ModQ* mods;
    int N, n, op, src;
    short lid[64];
    TW scal[64];           // SUBMUL: per row
};

// Fused HMULT + Rescale (neo_hmult_rescale): with c_l = INTT(HMULT output limb l) =
// (accl - conv_l) P^-1 + dl mod q_l (coefficient form, canonical), rewrite the ModDown BConv
// output rows i < l as z_i = conv_i + P c_l mod q_i, so one NTT of z carries both ModDown's
// and Rescale's corrections.
struct HmrFoldArgs {
    u64* conv;             // [2B][l+1][N]: lazy doubles (lazy != 0) or canonical u64
    const u64* accl;       // [2B][N] INTT(acc_c limb l), canonical mod q_l
    const u64* dl;         // [2B][N] INTT(d_c limb l), canonical mod q_l
    const ModQ* mods;
    TW pinv_l;             // P^-1 mod q_l
    TWD pmod[64];          // (P mod q_i, /q_i), i < l
    int N, l, lazy;
};

// Double Rescale step 2: from the coefficient form of the last two limbs r[bc][2][N]
// (mod q_{l-1}, mod q_l) writes corr[bc][i][N] = [x mod q_{l-1} q_l]_{q_i} for i < l - 1.
struct DsArgs {
    const u64* last2;      // [2B][2][N]
    u64* corr;             // [2B][l-1][N]
    const ModQ* mods;
    int N, l;
    TW qlinv_m;            // q_l^-1 mod q_{l-1}
    TW ql[64];             // q_l mod q_i
};

cudaError_t launch_ew(const EwArgs& A, int batch, cudaStream_t st);
// out = a + b mod q_i for polynomials [batch][limbs][N] (one component; out may alias a)
cudaError_t launch_add_rows(const u64* a, const u64* b, u64* out, const ModQ* mods, int limbs, int N, int batch,
                            cudaStream_t st);
cudaError_t launch_pmult_acc(const PmaccArgs& A, int batch, cudaStream_t st);
cudaError_t launch_hmr_fold(const HmrFoldArgs& A, int bc, cudaStream_t st);
cudaError_t launch_hmr_cl(const HmrFoldArgs& A, int bc, cudaStream_t st);   // c_l only, over accl
cudaError_t launch_ew_limbs(const EwlArgs& A, int batch, cudaStream_t st);
// 36-bit wire format (neo_wire_pack / neo_wire_unpack); n % 8 == 0
cudaError_t launch_wire(bool pack, const void* in, void* out, size_t n, cudaStream_t st);
// ModRaise: coef[bc][N] (coefficient form mod q_0, canonical) -> out[bc][i][N] = centred lift mod q_i
cudaError_t launch_modraise(const u64* coef, u64* out, const ModQ* mods, int limbs, int N, int bc, cudaStream_t st);
// drop limbs: in [B][2][li][N] -> out [B][2][lo][N] (lo <= li), the first lo limbs of each component
cudaError_t launch_drop(const u64* in, u64* out, int li, int lo, int N, int batch, cudaStream_t st);
cudaError_t launch_ds_corr(const DsArgs& A, int bc, cudaStream_t st);
cudaError_t launch_bconv(const BConvTab& T, const BConvIO& io, int N, int batch, cudaStream_t st);
cudaError_t launch_keyip(const KeyIPArgs& A, int limbs, int batch, cudaStream_t st);
cudaError_t launch_combine(const CombineArgs& A, int limbs, int batch, cudaStream_t st);
cudaError_t launch_tensor(const u64* a, const u64* b, u64* d, const ModQ* mods, int limbs, int N, int batch,
                          cudaStream_t st);
cudaError_t launch_automorph(const u64* in, u64* out, unsigned g, int N, int rows, cudaStream_t st, int batch = 1,
                             long long in_bs = 0, long long out_bs = 0);
cudaError_t launch_pack5(const u64* in, uint32_t* lo, uint8_t* hi, size_t n, cudaStream_t st);
cudaError_t launch_pack6(const u64* in, uint32_t* lo, uint16_t* hi, size_t n, cudaStream_t st);

}  // namespace neo
