// klss.h -- KLSS key-switching kernels (klss.cu): the inner product over the T basis and
// Recover Limbs; the other KLSS steps reuse the NTT, BConv and ModDown machinery.
#pragma once
#include "context.h"

namespace neo {

constexpr int KLSS_MAX_BETA = 12;     // digits (beta <= dnum)
constexpr int KLSS_MAX_GROUPS = 8;    // beta~ (one warp per group in the IP CTA)
constexpr int KLSS_MAX_OUT_G = 16;    // limbs per group (alpha~)

// IP (Alg. 3 L359-382 / Alg. 4): for every T limb k and coefficient n,
//   acc[b][c][i][k] = sum_{j < beta} up[b][j][k] * e[c][i][j][k]  mod t_k
// for the groups i present at this level (NTT form over T).
struct KlssIpArgs {
    const u64* up;            // [B][beta][alpha'][N]
    const uint32_t* key_lo;   // [2][beta~][dnum][alpha'][N] (5-byte residues: low 32 bits ...)
    const uint8_t* key_hi;    //                              ... and bits 32..39)
    u64* acc;                 // [B][2][beta~][alpha'][N]
    const ModQ* mods;         // by limb id
    int N, beta, dnum, beta_t, alpha_p, t0;   // t0 = limb id of t_0
    int n_groups;
    int group[KLSS_MAX_GROUPS];               // present group indices
};

// Recover Limbs (reading K4): exact centred CRT of acc[b][c][i] (coefficient form over T) to
// the limbs of group i present at this level, written to rec[b][c][pos] (pos = position in
// the PQ_l basis q_0..q_l, p_0..p_K).
struct KlssRecArgs {
    const u64* acc;           // [B][2][beta~][alpha'][N]
    u64* rec;                 // [B][2][E][N]
    const RecTab* tab;
    const ModQ* mods;
    int N, alpha_p, beta_t, t0, E;
    int n_groups;
    int group[KLSS_MAX_GROUPS];               // present group indices
    int first[KLSS_MAX_GROUPS + 1];           // outputs of present group g: first[g] .. first[g+1]-1
    int out_id[KLSS_MAX_EXT];                 // limb id of each output
    int out_pos[KLSS_MAX_EXT];                // its position in PQ_l
};


cudaError_t launch_klss_ip(const KlssIpArgs& A, int batch, cudaStream_t st);
cudaError_t launch_klss_recover(const KlssRecArgs& A, int batch, cudaStream_t st);
// WordSize_T = 48 variants (64-bit products; the key's hi plane holds 16 bits per residue)
cudaError_t launch_klss_ip48(const KlssIpArgs& A, int batch, cudaStream_t st);
cudaError_t launch_klss_recover48(const KlssRecArgs& A, int batch, cudaStream_t st);

}  // namespace neo
