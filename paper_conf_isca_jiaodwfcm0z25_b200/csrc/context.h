// context.h -- host-side definition of neo_ctx / neo_evk and of the per-launch constant
// blocks (passed by value as kernel parameters, so no hot-path H2D copies are needed).
#pragma once
#include <string>
#include <vector>

#include "common.cuh"
#include "neo.h"
#include "ntt.h"

namespace neo {

constexpr int BC_MAX_IN = 16;
constexpr int BC_MAX_OUT = 64;

// Constants of one basis conversion (Algorithm 1) from n_in to n_out limbs:
//   y_i = [c_i * qhat_i^-1]_{q_i};  out_j = sum_i y_i * (qhat_i mod t_j) mod t_j.
// f is stored as 18-bit halves so the CUDA-core kernel accumulates with 32x32->64 MADs.
struct BConvTab {
    int n_in, n_out;
    u64 qin[BC_MAX_IN];
    TW qhat_inv[BC_MAX_IN];
    ModQ tmod[BC_MAX_OUT];
    unsigned f_lo[BC_MAX_IN][BC_MAX_OUT];   // (qhat_i mod t_j) & (2^18 - 1)
    unsigned f_hi[BC_MAX_IN][BC_MAX_OUT];   // (qhat_i mod t_j) >> 18
};

// Row addressing of a BConv launch: input row i of batch entry b at in + b*in_bstride +
// in_off[i]*N, output row j at out + b*out_bstride + out_off[j]*N.
struct BConvIO {
    const u64* in;
    u64* out;
    long long in_bstride, out_bstride;
    int in_off[BC_MAX_IN];
    int out_off[BC_MAX_OUT];
};

constexpr int BCTC_MAX_IN = 12;     // K = 5 * n_in <= 64
constexpr int BCTC_MAX_OUT = 45;    // targets per conversion (5 parts of 9: one MMA of N = 240)
constexpr int BCTC_PART_J = 9;      // targets per TMEM job (N = 5 J = 45 -> 48 columns)
constexpr int BCTC_PART_ROWS = 48;  // B rows per part (padded to the MMA N)
constexpr int BCTC_MAX_PARTS = (BCTC_MAX_OUT + BCTC_PART_J - 1) / BCTC_PART_J;   // 6

struct BConvTC {
    int n_in, n_out;
    int nparts, J;                  // targets split in nparts jobs of J (last may be shorter)
    int ncols;                      // MMA N per job = round_up(nb J, 16) <= 48
    int nb;                         // bytes per target in B: 5 (targets < 2^40) or 6 (48-bit T primes)
    double qin[BCTC_MAX_IN], qinv_in[BCTC_MAX_IN];
    TWD qhat_inv[BCTC_MAX_IN];      // [qhat_i^-1]_{q_i}
    double t[BCTC_MAX_OUT], tinv[BCTC_MAX_OUT];
};

struct BMatParam {                   // B passed by value (generic neo_bconv, no device tables)
    uint4 d[BCTC_MAX_PARTS * BCTC_PART_ROWS * 64 / 16];   // parts of 48 rows x 64 B
};

// KLSS Recover Limbs (exact centred CRT from T to a limb p of PQ), device table:
//   y_k = [a_k That_k^-1]_{t_k},  u = rint(sum_k y_k / t_k),  out_p = sum_k y_k [That_k]_p - u [T]_p
constexpr int KLSS_MAX_T = 16;
constexpr int KLSS_MAX_EXT = 64;
struct RecTab {
    TW that_inv[KLSS_MAX_T];                 // That_k^-1 mod t_k
    double tinv[KLSS_MAX_T];                 // fl(1 / t_k)
    TW that_p[KLSS_MAX_EXT][KLSS_MAX_T];     // That_k mod p, by limb id p of PQ
    unsigned that_lo[KLSS_MAX_EXT][KLSS_MAX_T], that_hi[KLSS_MAX_EXT][KLSS_MAX_T];   // its 18-bit halves
    TW T_p[KLSS_MAX_EXT];                    // T mod p
};

}  // namespace neo

struct neo_ctx {
    int log_n, N, num_q, num_p, dnum, alpha, word_bits, device;
    unsigned long long uid = 0;           // unique per created context (host-side caches key on it)
    cudaStream_t side = nullptr;          // second stream for chunked batches (fork/join on the caller's)
    std::vector<u64> mod;                 // by limb id
    std::vector<u64> psi;                 // by limb id
    std::vector<ModQ> h_mods;
    NttLayout L;
    TWD* d_tab = nullptr;                 // [limb id][L.total]
    uint8_t* d_ntt_tc = nullptr;          // [limb id][NTC_PRIME_BYTES]: tensor-core NTT tables (N = 2^16), or null
    int ntt_impl = 0;                     // NEO_NTT_FP64 (0) or NEO_NTT_TC (1); neo_ntt_select
    ModQ* d_mods = nullptr;
    neo::NttArgs ntt;
    // per level l (index l = 0..num_q-1)
    std::vector<std::vector<neo::BConvTab>> modup;   // [l][digit j]
    std::vector<std::vector<std::vector<int>>> digits;  // [l][j] -> limb ids
    std::vector<neo::BConvTab> moddown;              // [l]: P limbs -> q_0..q_l
    std::vector<TW> pinv;                            // [i] P^-1 mod q_i (Shoup)
    // tensor-core BConv (bconv_tc.cu): constants and device byte matrices per (l, j) / l
    std::vector<std::vector<neo::BConvTC>> modup_tc;
    std::vector<neo::BConvTC> moddown_tc;
    std::vector<std::vector<size_t>> modup_boff;     // byte offsets into d_bmat
    std::vector<size_t> moddown_boff;
    uint8_t* d_bmat = nullptr;
    int num_sms = 148;
    bool use_tc = true;                              // NEO_BCONV=cuda selects the CUDA-core control kernel
    std::vector<std::vector<TW>> ql_inv;             // [l][i] q_l^-1 mod q_i, i < l
    // Double Rescale at level l >= 2 (i < l - 1): (q_{l-1} q_l)^-1 mod q_i and q_l mod q_i;
    // ds_qlinv_m[l] = q_l^-1 mod q_{l-1}
    std::vector<std::vector<TW>> ds_inv, ds_ql;
    std::vector<TW> ds_qlinv_m;
    // KLSS (alpha_t > 0): T primes are limb ids num_q+num_p .. +num_t-1
    int alpha_t = 0, num_t = 0;
    int word_bits_t = 0;                                   // WordSize_T of the T primes (Table 4; 36 or 48)
    bool klss_rec_tc_ok = true;                            // tensor-core Recover needs T primes < 2^40
    std::vector<std::vector<int>> klss_groups;             // [i] limb ids of PQ_L in group i
    std::vector<std::vector<neo::BConvTab>> klss_up;       // [l][j] digit -> T (CUDA-core control)
    std::vector<std::vector<neo::BConvTC>> klss_up_tc;     // [l][j] digit -> T (tensor cores)
    std::vector<std::vector<size_t>> klss_up_boff;
    neo::RecTab* d_rec = nullptr;
    std::vector<std::vector<neo::BConvTC>> klss_rec_tc;    // [l][i] T -> group i's limbs in PQ_l (centred)
    std::vector<std::vector<size_t>> klss_rec_boff;
    int limbs_total() const { return num_q + num_p + num_t; }

    int beta(int level) const { return (level + 1 + alpha - 1) / alpha; }
    int ext(int level) const { return level + 1 + num_p; }          // limbs of PQ_l
    int ext_id(int level, int pos) const {                           // position -> limb id
        return pos <= level ? pos : num_q + (pos - level - 1);
    }
};

struct neo_evk {
    const neo_ctx* ctx;
    // 36-bit residues stored as 5 bytes (SURVEY §7 planar layout): low 32 bits and the top
    // byte in two planes, each [dnum][2][num_q+num_p][N]; 94 MB instead of 151 MB at Set-B.
    uint32_t* lo = nullptr;
    uint8_t* hi = nullptr;
    uint32_t galois = 0;                  // hoisted rotation keys: the key is stored as sigma_{g^-1}(evk_g)
    int klss = 0;                         // KLSS key: planes are [2][beta~][dnum][alpha'][N] over T
    int hi_bytes = 1;                     // bytes per residue in the hi plane: 1 (5-byte key) or 2 (48-bit T: 6 bytes)
};
