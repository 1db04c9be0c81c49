/*
 * neo.h -- C-ABI of the B200-native CKKS Hybrid key-switching library (libneo.so).
 *
 * The operations follow the problem statement of "Neo: Towards Efficient Fully
 * Homomorphic Encryption Acceleration using Tensor Core" (ISCA'25); citations are
 * /root/reference/PAPER.md lines (L<n>) and the readings Z1-Z23 of SURVEY.md §8(c),
 * restated in DESIGN.md.
 *
 * Conventions (all entry points):
 *  - Residues are uint64 in [0, m) for the limb's modulus m (canonical).  Inputs that
 *    are not canonical give unspecified (but memory-safe) outputs.
 *  - Limb ids index the concatenated basis q_0..q_{num_q-1}, p_0..p_{num_p-1}.
 *  - Polynomials are laid out [batch][limb][N] with the limb contiguous (D1, L280, L355).
 *    Ciphertexts are [batch][2][level+1][N], NTT form, natural order (Z6).
 *  - Tensor arguments are CUDA DEVICE pointers owned by the caller; the library never
 *    frees them.  Host arrays (limb id lists, prime lists) are read before return.
 *    Device buffers must be 16-byte aligned.
 *  - `stream` is a cudaStream_t (NULL = legacy default stream).  Every compute call is
 *    asynchronous on it: no host synchronisation and no device allocation inside the
 *    hot-path calls (ntt, intt, bconv, tensor, automorphism, keyswitch, hmult, hrot,
 *    rescale).  create/destroy calls may synchronise and allocate.
 *  - No aliasing between inputs and outputs except where an entry point says "in place".
 *  - Errors: arguments are validated before any launch; a non-OK status is returned and
 *    a thread-local message is available from neo_last_error().  Launch failures return
 *    NEO_ECUDA.  Nothing aborts or throws across the ABI.
 *  - A context is immutable after creation and may be shared by threads.
 */
#ifndef NEO_H
#define NEO_H

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef struct neo_ctx neo_ctx;   /* parameters + device constant tables */
typedef struct neo_evk neo_evk;   /* a device-resident evaluation (key-switching) key */
typedef struct neo_comm neo_comm; /* limb-sharded key-switching communicator (one per rank) */
typedef void* neo_stream_t;       /* cudaStream_t */

typedef enum {
    NEO_OK = 0,
    NEO_EINVAL = 1,        /* bad argument (null pointer, level out of range, batch <= 0, ...) */
    NEO_EUNSUPPORTED = 2,  /* valid request outside what this build implements (e.g. log_n) */
    NEO_ENOMEM = 3,        /* device/host allocation failed in a create call */
    NEO_ECUDA = 4,         /* a CUDA call or kernel launch failed */
    NEO_ENCCL = 5,         /* NCCL unavailable or failed (limb-sharded key-switch) */
    NEO_ENOPRIME = 6       /* not enough word_bits-bit primes p = 1 mod 2N */
} neo_status;

/* Operation codes for neo_workspace_size. */
enum { NEO_OP_KEYSWITCH = 0, NEO_OP_HMULT = 1, NEO_OP_HROT = 2, NEO_OP_RESCALE = 3, NEO_OP_HROT_HOISTED = 4,
       NEO_OP_DOUBLE_RESCALE = 5, NEO_OP_MODRAISE = 6, NEO_OP_HMULT_RESCALE = 7, NEO_OP_HROT_SUM = 8 };

/* Parameter description (Table 1, Table 4).
 *  log_n      : log2 N; this build supports 12 and 16 (N = 2^12 tiny config, 2^16 Set-B).
 *  num_q      : number of Q limbs (L+1; Set-B: 36, Z2).
 *  num_p      : number of special limbs (K+1; Set-B: 12, Z3).
 *  dnum       : digits; alpha = ceil(num_q/dnum) (L98); ceil(num_q/alpha) must equal dnum.
 *  word_bits  : prime bit width; this build supports 36 (WordSize of Set-B, L510).
 *  device     : CUDA device ordinal the tables live on.
 *  q, p       : optional explicit primes (host arrays of num_q / num_p entries, each
 *               = 1 mod 2N, word_bits wide); NULL selects rule Z4: k*2N+1 for k from
 *               floor((2^W-1)/2N) downward, prime, first num_q are q, next num_p are p.
 * psi is always the minimal primitive 2N-th root of each prime (Z5). */
typedef struct {
    int32_t log_n, num_q, num_p, dnum, word_bits, device;
    const uint64_t* q;
    const uint64_t* p;
    int32_t alpha_t;     /* KLSS key-decomposition group size alpha~ (Table 4); 0 = Hybrid only.
                          * > 0 adds alpha' T primes (alpha' from Eq. 4, reading K3)
                          * and the KLSS tables; requires generated primes (q = p = NULL). */
    int32_t word_bits_t; /* WordSize_T of the T primes (Table 4: 48 for Set-C), used when
                          * alpha_t > 0: 0 or word_bits = the Z4 rule continued after p; 48 = the
                          * Z4 rule at 48 bits (reading K6).  Other values fail with
                          * NEO_EUNSUPPORTED. */
} neo_params_desc;

/* Build the context: primes, psi, NTT twiddle tables, BConv tables for every
 * (level, digit) of ModUp and every level of ModDown, P^-1 and q_l^-1 tables. */
neo_status neo_params_create(const neo_params_desc* desc, neo_ctx** out);
neo_status neo_params_destroy(neo_ctx* ctx);

/* Copy the moduli and psi to host arrays (any may be NULL): q[num_q], p[num_p],
 * psi[num_q+num_p] (psi indexed by limb id). */
neo_status neo_params_query(const neo_ctx* ctx, uint64_t* q, uint64_t* p, uint64_t* psi);

/* KLSS extras of the context: alpha~, alpha' (number of T primes) and the T primes (host array
 * of alpha' entries, may be NULL).  T limb ids are num_q+num_p .. num_q+num_p+alpha'-1. */
neo_status neo_klss_query(const neo_ctx* ctx, int32_t* alpha_t, int32_t* alpha_p, uint64_t* t);

/* Bytes of device workspace `ws` the caller must pass to op (NEO_OP_*) at this level
 * and batch; 0 on invalid arguments. */
size_t neo_workspace_size(const neo_ctx* ctx, int32_t op, int32_t level, int32_t batch);

/* Negacyclic NTT, IN PLACE, per limb (L438-450; definition a_hat[i] = a(psi^(2i+1)),
 * natural order in and out, Z6).  poly is [batch][n_limbs][N]; row k is reduced mod the
 * prime of limb id limb_ids[k] (host array), 1 <= n_limbs <= 160.  ws is a device scratch
 * buffer of at least batch*n_limbs*N*8 bytes (the two passes run out of place). */
neo_status neo_ntt(const neo_ctx* ctx, uint64_t* poly, const int32_t* limb_ids, int32_t n_limbs,
                   int32_t batch, void* ws, size_t ws_bytes, neo_stream_t stream);
/* Inverse of neo_ntt (includes the N^-1 scaling), IN PLACE; same arguments. */
neo_status neo_intt(const neo_ctx* ctx, uint64_t* poly, const int32_t* limb_ids, int32_t n_limbs,
                    int32_t batch, void* ws, size_t ws_bytes, neo_stream_t stream);

/* Select the NTT implementation every transform of this context uses (neo_ntt / neo_intt and
 * every NTT inside the key-switching operations); the result is bit-identical either way.
 *   NEO_NTT_TC   : both radix-16 DFT stages of each 256-point pass as tcgen05 kind::i8 GEMMs
 *                  (Neo's matrix-multiplication NTT, L438-450 / Fig. 9, on the int8 tensor
 *                  cores; N = 2^16 with 36-bit primes only; environment NEO_NTT=tc at
 *                  context creation makes it the context's default);
 *   NEO_NTT_FP64 : radix-2 butterflies in FP64 on the CUDA cores (any supported N) -- the
 *                  default: faster on B200 (profiles/r02_ntt_ab.md).
 * Returns NEO_EUNSUPPORTED (selection unchanged) if NEO_NTT_TC is not available for this
 * context.  Not thread-safe with respect to operations running on the same context. */
enum { NEO_NTT_FP64 = 0, NEO_NTT_TC = 1 };
neo_status neo_ntt_select(neo_ctx* ctx, int32_t impl);
/* The implementation currently selected (NEO_NTT_*), or -1 for a NULL context. */
int32_t neo_ntt_selected(const neo_ctx* ctx);

/* Rescale constants (L137, Z10): out[k] = q_level^-1 mod q_{limb_ids[k]} for n limb ids < level
 * (host arrays), from the context's tables -- for callers that sequence a Rescale themselves
 * (the limb-sharded bootstrapping).  NEO_EINVAL for a limb id outside [0, level). */
neo_status neo_query_ql_inv(const neo_ctx* ctx, int32_t level, const int32_t* limb_ids, int32_t n, uint64_t* out);

/* Basis conversion, Algorithm 1 (L296-319), non-centred (Z7), coefficient form:
 *   out[t] = sum_i [in_i * qhat_i^-1]_{q_i} * (qhat_i mod t) mod t,
 *   qhat_i = prod_{i' != i} q_{i'} over the input limbs.
 * in [batch][n_in][N] with limb ids in_ids (1 <= n_in <= 16, distinct);
 * out [batch][n_out][N] with limb ids out_ids (1 <= n_out <= 64).
 * The first call for a given (context, in_ids, out_ids) builds that conversion's constants on the
 * host and caches them per thread (one host allocation); later calls with the same ids do no
 * host work beyond argument validation.  No device allocation. */
neo_status neo_bconv(const neo_ctx* ctx, const uint64_t* in, const int32_t* in_ids, int32_t n_in,
                     uint64_t* out, const int32_t* out_ids, int32_t n_out, int32_t batch,
                     neo_stream_t stream);

/* HMULT tensor product (L132), NTT form: from ct_a, ct_b [batch][2][level+1][N] writes
 * d [batch][3][level+1][N] with d0 = a0 b0, d1 = a0 b1 + a1 b0, d2 = a1 b1. */
neo_status neo_tensor(const neo_ctx* ctx, const uint64_t* ct_a, const uint64_t* ct_b, int32_t level,
                      uint64_t* d, int32_t batch, neo_stream_t stream);

/* Galois automorphism X -> X^g (AUTO, L268-270) in the NTT domain:
 *   out[i] = in[(g*i + (g-1)/2) mod N]   per limb; in/out [batch][n_limbs][N].
 * galois_elt must be odd and < 2N. */
neo_status neo_automorphism(const neo_ctx* ctx, const uint64_t* in, int32_t n_limbs,
                            uint32_t galois_elt, uint64_t* out, int32_t batch, neo_stream_t stream);

/* Evaluation key (L184; gadget Z8): evk is a DEVICE array [dnum][2][num_q+num_p][N] in NTT
 * form, evk[j][0] = b_j, evk[j][1] = a_j.  The library re-lays it out once into 5 bytes per
 * residue (a 32-bit and an 8-bit plane: 94 MB instead of 151 MB at Set-B), so the caller may
 * free its copy after return.  Synchronises the current device. */
neo_status neo_evk_create(const neo_ctx* ctx, const uint64_t* evk, neo_evk** out);
neo_status neo_evk_destroy(neo_evk* evk);

/* KLSS evaluation key (L155-180, Alg. 3/4; readings K1-K6 in DESIGN.md): ekey is a DEVICE array
 * [2][beta~][dnum][alpha'][N], NTT form over the T primes, ekey[c][i][j] = the Hybrid key
 * component evk_{j,c} reduced modulo the group modulus P~_i (group i = limbs i*alpha~ ..
 * of q_0..q_L, p_0..p_K).  Re-laid out to 5 bytes per residue; the caller may free its copy.
 * neo_keyswitch / neo_hmult / neo_hrot given a KLSS key run the KLSS method:
 *   INTT -> ModUp BConv to T (alpha' limbs) -> NTT over T -> IP (beta x beta~) -> INTT over T
 *   -> Recover Limbs (exact centred CRT from T) -> ModDown -> NTT,
 * whose output equals the Hybrid method's for the key it was derived from (reading K4).
 * Needs a context created with alpha_t > 0. */
neo_status neo_evk_create_klss(const neo_ctx* ctx, const uint64_t* ekey, neo_evk** out);

/* Hybrid key-switch (Table 2, Eq. 2, Fig. 5) at `level`:
 *   INTT -> ModUp BConv (per digit) -> NTT -> KeyIP -> INTT(P part) -> ModDown BConv
 *   -> NTT -> (acc - conv) * P^-1.
 * d [batch][level+1][N] NTT form; out0, out1 [batch][level+1][N] NTT form with
 * out0 + out1 s ~= d s' for the key's (s, s').  All batch entries use the same key (Z21).
 * ws: device workspace of at least neo_workspace_size(ctx, NEO_OP_KEYSWITCH, level, batch). */
neo_status neo_keyswitch(const neo_ctx* ctx, const neo_evk* evk, const uint64_t* d, int32_t level,
                         uint64_t* out0, uint64_t* out1, int32_t batch, void* ws, size_t ws_bytes,
                         neo_stream_t stream);

/* HMULT (L132) = tensor + relinearise (KS of d2 with the relinearisation key) + add to
 * (d0, d1).  No rescale (Z22).  ct_a, ct_b, ct_out: [batch][2][level+1][N]. */
neo_status neo_hmult(const neo_ctx* ctx, const neo_evk* relin, const uint64_t* ct_a,
                     const uint64_t* ct_b, int32_t level, uint64_t* ct_out, int32_t batch, void* ws,
                     size_t ws_bytes, neo_stream_t stream);

/* HMULT followed by Rescale (L132 + L137) as one fused call: ct_out [batch][2][level][N] equals
 * neo_rescale(neo_hmult(ct_a, ct_b)) residue for residue.  Rescale's correction is folded
 * into the key-switch's ModDown: with c_l = INTT of the product's last limb (its coefficient
 * form, from INTT(acc_l), INTT(d_l) and the ModDown BConv output), the BConv output of every
 * q_i (i < l) gets P [c_l]_{q_l} added before the one forward NTT, whose fused tail writes
 * ((acc_i - NTT_i) P^-1 + d_i) q_l^-1 -- so Rescale's own INTT / NTT passes disappear.
 * Hybrid keys only (NEO_EUNSUPPORTED for a KLSS key); 1 <= level <= 64;
 * ws >= neo_workspace_size(ctx, NEO_OP_HMULT_RESCALE, level, batch). */
neo_status neo_hmult_rescale(const neo_ctx* ctx, const neo_evk* relin, const uint64_t* ct_a,
                             const uint64_t* ct_b, int32_t level, uint64_t* ct_out, int32_t batch,
                             void* ws, size_t ws_bytes, neo_stream_t stream);

/* HROTATE (L136): (sigma_g(c0) + k0, k1) with (k0, k1) = KS(sigma_g(c1)) under rotkey
 * = KSGen(s, sigma_g(s)) (L184).  galois_elt = 5^r mod 2N rotates slots left by r (Z11). */
neo_status neo_hrot(const neo_ctx* ctx, const neo_evk* rotkey, uint32_t galois_elt,
                    const uint64_t* ct_in, int32_t level, uint64_t* ct_out, int32_t batch, void* ws,
                    size_t ws_bytes, neo_stream_t stream);

/* Hoisted rotations: n_rot rotations of the same ciphertexts share one
 * ModUp of c1.  For rotation r with Galois element g_r the result is
 *   sigma_{g_r}( c0 + k0', k1' ),   (k0', k1') = KeySwitch(c1) under sigma_{g_r}^{-1}(rotkey_r),
 * which decrypts to the slot rotation like neo_hrot (it is a different, equally valid
 * ciphertext: the automorphism is applied after ModDown instead of before ModUp).
 * keys[r] must come from neo_evk_create_hoisted (which stores sigma_{g^-1}(evk) once).
 * ct_in [batch][2][level+1][N]; ct_out [n_rot][batch][2][level+1][N];
 * ws >= neo_workspace_size(ctx, NEO_OP_HROT_HOISTED, level, batch) (two ModDown areas: the odd
 * rotations run on the context's internal side stream, forked from and joined back into `stream`
 * by events -- asynchronous and graph-capturable; NEO_TWO_STREAM=0 at process start: one stream). */
neo_status neo_evk_create_hoisted(const neo_ctx* ctx, const uint64_t* evk, uint32_t galois_elt,
                                  neo_evk** out);
neo_status neo_hrot_hoisted(const neo_ctx* ctx, const neo_evk* const* keys, int32_t n_rot,
                            const uint64_t* ct_in, int32_t level, uint64_t* ct_out, int32_t batch,
                            void* ws, size_t ws_bytes, neo_stream_t stream);

/* Sum of rotations with one ModDown (the giant steps of a baby-step giant-step linear
 * transform; reading BOOT-G):  ct_out = (sum_k sigma_{g_k}(c0_k) + k0, k1) with
 * (k0, k1) = ModDown( sum_k KeyIP(ModUp(sigma_{g_k}(c1_k)), keys[k]) ), the KeyIP outputs summed
 * in PQ_l (Table 2).  Decrypts to sum_k rot_{g_k}(m_k); saves n - 1 ModDowns against n
 * neo_hrot calls (a different, equally valid ciphertext: ModDown's floor rounding is applied once).
 * keys[k]: neo_evk_create rotation keys (KSGen(s, sigma_{g_k}(s)), L184); galois[k] odd < 2N;
 * cts: host array of n device pointers, each [batch][2][level+1][N]; ct_out likewise, not
 * aliasing any input; 1 <= n <= 64; ws >= neo_workspace_size(ctx, NEO_OP_HROT_SUM, level, batch)
 * (two ModUp areas: the ModUps of odd k run on the context's internal side stream, joined back
 * into `stream`; the KeyIP sums stay on `stream` in order). */
neo_status neo_hrot_sum(const neo_ctx* ctx, const neo_evk* const* keys, const uint32_t* galois, int32_t n,
                        const uint64_t* const* cts, int32_t level, uint64_t* ct_out, int32_t batch, void* ws,
                        size_t ws_bytes, neo_stream_t stream);

/* ------------------------------------------------------------------ limb-sharded key-switch
 * One Hybrid key-switch (Table 2, Fig. 5) split by RNS limb over nranks ranks, one
 * GPU each (the paper has no multi-GPU design, L648 cites HE-Booster).  Limb
 * ownership at level l (round-robin, so a Rescale's dropped top limb rotates over the ranks):
 * rank r owns the Q limbs q_i with i = r (mod nranks), i <= l, and the P limbs p_k with
 * k = r (mod nranks).  NTT, KeyIP and the ModDown tail are limb-local; BConv needs every limb,
 * so the library runs two all-gathers of coefficient-form limbs inside the call: one per ModUp
 * digit (overlapped with the previous digit's BConv + NTT on a communication stream) and one of
 * the P limbs before ModDown.  The result equals neo_keyswitch restricted to the rank's limbs,
 * bit for bit.
 *
 * neo_comm_unique_id : a 128-byte NCCL unique id (ncclGetUniqueId); rank 0 creates it and the
 *                      caller distributes it (e.g. a torch.distributed broadcast).
 * neo_comm_create    : collective over the nranks processes (same uid); NCCL over NVLink for
 *                      nranks > 1 (libnccl.so.2 is loaded with dlopen; NEO_ENCCL if absent or if
 *                      ncclCommInitRank fails, e.g. two ranks on one GPU); nranks = 1 needs no NCCL.
 *                      Builds this rank's BConv tables for every level (synchronises the device).
 * neo_comm_create_local : nranks communicators sharing the context's GPU inside ONE process (one
 *                      host thread per rank must call each sharded operation concurrently; the
 *                      exchanges are device-to-device copies after a host barrier; not capturable
 *                      in a CUDA graph).  For tests and single-GPU runs of the sharded path.
 * neo_comm_limbs     : this rank's Q limb ids (return value = their count) and P limb ids
 *                      (count in *n_p) at `level`; arrays may be NULL; -1 on invalid arguments.
 * neo_keyswitch_sharded : d_local [batch][nq][N] = the rank's Q limbs of the KS input, rising
 *                      limb order, NTT form; out0/out1 [batch][nq][N] the rank's rows of (k0, k1).
 *                      A rank with nq = 0 (nranks > level + 1) passes NULL buffers and still
 *                      takes part in both exchanges.  evk: the full Hybrid key (neo_evk_create)
 *                      on every rank.  1 <= batch <= 32.  ws: neo_workspace_size_sharded bytes.
 *                      Asynchronous on `stream` (NCCL transport: graph-capturable). */
neo_status neo_comm_unique_id(uint8_t uid[128]);
neo_status neo_comm_create(const neo_ctx* ctx, const uint8_t uid[128], int32_t nranks, int32_t rank,
                           neo_comm** out);
neo_status neo_comm_create_local(const neo_ctx* ctx, int32_t nranks, neo_comm** comms);
neo_status neo_comm_destroy(neo_comm* comm);
int32_t neo_comm_limbs(const neo_comm* comm, int32_t level, int32_t* q_ids, int32_t* p_ids, int32_t* n_p);
size_t neo_workspace_size_sharded(const neo_comm* comm, int32_t level, int32_t batch);
neo_status neo_keyswitch_sharded(const neo_ctx* ctx, const neo_comm* comm, const neo_evk* evk,
                                 const uint64_t* d_local, int32_t level, uint64_t* out0, uint64_t* out1,
                                 int32_t batch, void* ws, size_t ws_bytes, neo_stream_t stream);

/* Building blocks of the limb-sharded key-switch (each rank owns a subset of
 * the limbs of PQ_l and calls these on its own limbs between NCCL all-gathers):
 *
 * KeyIP (Alg. 3) on an arbitrary limb subset:
 *   acc[b][c][t] = sum_{j<beta} dhat[b][j][t] * evk_{j,c}[limb_ids[t]]  mod q_{limb_ids[t]}
 * dhat [batch][beta][n][N] NTT form, acc [batch][2][n][N]; 1 <= n <= 64, 1 <= beta <= dnum. */
neo_status neo_keyip(const neo_ctx* ctx, const neo_evk* evk, const uint64_t* dhat, const int32_t* limb_ids,
                     int32_t n_limbs, int32_t beta, uint64_t* acc, int32_t batch, neo_stream_t stream);

/* ModDown tail (Table 2, Z9) on Q limbs q_ids[0..n):
 *   out[b][c][i] = (acc[b][c][i] - conv[b][c][i]) * P^-1  mod q_{q_ids[i]}
 * acc, conv, out [batch][2][n][N] NTT form. */
neo_status neo_moddown_combine(const neo_ctx* ctx, const uint64_t* acc, const uint64_t* conv,
                               const int32_t* q_ids, int32_t n, uint64_t* out, int32_t batch,
                               neo_stream_t stream);

/* Rescale (L137), floor reading (Z10): ct_in [batch][2][level+1][N] -> ct_out
 * [batch][2][level][N], c'_i = (c_i - NTT_i([INTT_l(c_l)] mod q_i)) * q_l^-1 mod q_i.
 * level >= 1. */
neo_status neo_rescale(const neo_ctx* ctx, const uint64_t* ct_in, int32_t level, uint64_t* ct_out,
                       int32_t batch, void* ws, size_t ws_bytes, neo_stream_t stream);

/* Double Rescale (DS, L138 and L151: "requires the last two levels of limbs to generate noise
 * reduction limbs ... consumes two ciphertext levels").  Reading: floor
 * division by q_{l-1} q_l, i.e. bit-identical to two successive neo_rescale calls:
 *   r = x mod q_{l-1} q_l  (exact, Garner on the last two limbs),
 *   c'_i = (c_i - [r]_{q_i}) * (q_{l-1} q_l)^-1 mod q_i,  i < l - 1.
 * ct_in [batch][2][level+1][N] -> ct_out [batch][2][level-1][N]; level >= 2;
 * ws >= neo_workspace_size(ctx, NEO_OP_DOUBLE_RESCALE, level, batch). */
neo_status neo_double_rescale(const neo_ctx* ctx, const uint64_t* ct_in, int32_t level, uint64_t* ct_out,
                              int32_t batch, void* ws, size_t ws_bytes, neo_stream_t stream);

/* Element-wise ciphertext operations without key-switching (L133-135), NTT form, one launch
 * each, no workspace.  ct_* are [batch][2][level+1][N]; pt is a plaintext polynomial
 * [batch][level+1][N] (one per ciphertext).  ct_out may alias ct_in / ct_a (same position).
 *   PMULT: (c0 * m, c1 * m);   HADD: (a0 + b0, a1 + b1);   PADD: (c0 + m, c1)  (Z1 sign). */
neo_status neo_pmult(const neo_ctx* ctx, const uint64_t* ct_in, const uint64_t* pt, int32_t level,
                     uint64_t* ct_out, int32_t batch, neo_stream_t stream);
neo_status neo_hadd(const neo_ctx* ctx, const uint64_t* ct_a, const uint64_t* ct_b, int32_t level,
                    uint64_t* ct_out, int32_t batch, neo_stream_t stream);
neo_status neo_padd(const neo_ctx* ctx, const uint64_t* ct_in, const uint64_t* pt, int32_t level,
                    uint64_t* ct_out, int32_t batch, neo_stream_t stream);

/* HSUB: (a0 - b0, a1 - b1), same conventions as neo_hadd. */
neo_status neo_hsub(const neo_ctx* ctx, const uint64_t* ct_a, const uint64_t* ct_b, int32_t level,
                    uint64_t* ct_out, int32_t batch, neo_stream_t stream);

/* Limb-subset element-wise operations for the limb-sharded evaluator (SURVEY §8(e)/(f) row 2:
 * each rank holds the rows limb_ids[0..n) of its ciphertexts, in that order; row k is reduced
 * mod q_{limb_ids[k]}, ids index the concatenated basis q_0..q_L, p_0..p_K).  NTT form unless
 * stated; ct_* [batch][2][n][N], pt [batch][n][N]; 1 <= n <= 64.
 *   NEO_EWL_HADD / _HSUB / _PMULT / _PADD (0-3): as neo_hadd / neo_hsub / neo_pmult / neo_padd (L133-135)
 *   NEO_EWL_TENSOR (4): out d [batch][3][n][N] = (a0 b0, a0 b1 + a1 b0, a1 b1) (L132)
 *   NEO_EWL_SUBMUL (5): out = (a - b) * scal[k]; scal a HOST array of n residues (Rescale's
 *                       (c_i - r_i) q_l^-1 on a rank's limbs, L137)
 *   NEO_EWL_LIFT (6):   a = coefficient rows [batch][2][N], canonical mod q_{src_limb}; out
 *                       [batch][2][n][N] = each value's centred representative reduced mod
 *                       q_{limb_ids[k]} (coefficient form; ModRaise on a rank's limbs, L529)
 * b is ignored for LIFT; scal only read for SUBMUL; out may alias a (same positions). */
enum { NEO_EWL_HADD = 0, NEO_EWL_HSUB = 1, NEO_EWL_PMULT = 2, NEO_EWL_PADD = 3, NEO_EWL_TENSOR = 4,
       NEO_EWL_SUBMUL = 5, NEO_EWL_LIFT = 6 };
neo_status neo_ew_limbs(const neo_ctx* ctx, int32_t op, const uint64_t* a, const uint64_t* b,
                        const int32_t* limb_ids, int32_t n, const uint64_t* scal, int32_t src_limb,
                        uint64_t* out, int32_t batch, neo_stream_t stream);

/* 36-bit wire format for host<->device transfers of residues (serialization, no arithmetic):
 * n canonical residues < 2^36 take neo_wire_bytes(n) = 4.5 n bytes instead of 8 n:
 *   bytes [0, 4n):      the low 32 bits of residue i at 4 i (little endian),
 *   bytes [4n, 4.5n):   byte k = (residue 2k >> 32) | (residue 2k+1 >> 32) << 4.
 * neo_wire_pack: device u64 residues -> device wire buffer; neo_wire_unpack: the inverse.
 * n must be a positive multiple of 8; the wire buffer 16-byte aligned; word_bits <= 36
 * (NEO_EUNSUPPORTED otherwise).  A ciphertext [batch][2][l+1][N] is n = batch 2 (l+1) N.
 * Residues >= 2^36 lose their high bits (the caller's inputs must be canonical). */
size_t     neo_wire_bytes(size_t n);
neo_status neo_wire_pack(const neo_ctx* ctx, const uint64_t* in, void* wire, size_t n, neo_stream_t stream);
neo_status neo_wire_unpack(const neo_ctx* ctx, const void* wire, uint64_t* out, size_t n, neo_stream_t stream);

/* Plaintext inner product (the diagonal method's inner loop of CoeffToSlot / SlotToCoeff and of
 * a packed convolution: PMULT L133 followed by HADD L134, fused):
 *   ct_out[b] = sum_{k < n_terms} ( c0_k[b] * m_k, c1_k[b] * m_k )   mod q_i, NTT form.
 * cts: host array of n_terms device pointers, each ciphertexts [batch][2][level+1][N];
 * pts: host array of n_terms device pointers, each plaintexts [batch][level+1][N], or one
 * plaintext [level+1][N] applied to every batch entry when pt_shared != 0.
 * 1 <= n_terms <= 32; ct_out [batch][2][level+1][N] must not alias any cts[k] (NEO_EINVAL).
 * Equal, residue for residue, to n_terms neo_pmult calls summed by neo_hadd; one launch. */
neo_status neo_pmult_acc(const neo_ctx* ctx, const uint64_t* const* cts, const uint64_t* const* pts,
                         int32_t n_terms, int32_t pt_shared, int32_t level, uint64_t* ct_out, int32_t batch,
                         neo_stream_t stream);

/* Bootstrapping's ModRaise (the first step of PackBootstrap, L529):
 * ct_in [batch][2][1][N] mod q_0 (NTT form) -> ct_out [batch][2][level+1][N]: each coefficient's
 * centred representative in (-q_0/2, q_0/2] reduced mod q_0..q_level, NTT form, so that
 * decryption gives m + q_0 I for a small integer polynomial I.
 * ws >= neo_workspace_size(ctx, NEO_OP_MODRAISE, level, batch). */
neo_status neo_modraise(const neo_ctx* ctx, const uint64_t* ct_in, int32_t level, uint64_t* ct_out,
                        int32_t batch, void* ws, size_t ws_bytes, neo_stream_t stream);

/* Level drop (modulus switch down without scaling): the first level_out+1 limbs of each
 * component, ct_in [batch][2][level_in+1][N] -> ct_out [batch][2][level_out+1][N]. */
neo_status neo_drop_levels(const neo_ctx* ctx, const uint64_t* ct_in, int32_t level_in, uint64_t* ct_out,
                           int32_t level_out, int32_t batch, neo_stream_t stream);

/* Thread-local message describing the last non-OK status returned on this thread. */
const char* neo_last_error(void);

/* Number of kernels the last hot-path call on this thread launched (for bench.py's
 * gpu_launches accounting). */
int32_t neo_last_launch_count(void);

/* Diagnostics: when enabled (on != 0), every kernel launched by this thread is bracketed
 * by a pair of CUDA events on its stream; enabling or disabling clears the records.
 * neo_profile_read synchronises on the recorded events and returns the summed device
 * time (ms) and launch count of one kernel kind:
 *   0 NTT column pass, 1 NTT row pass, 2 BConv, 3 KeyIP, 4 combine (ModDown tail),
 *   5 tensor, 6 automorphism, 7 mod-switch (Double Rescale's noise-reduction limbs),
 *   8 rescale combine, 9 element-wise (PMULT / HADD / PADD). */
enum { NEO_PK_NTT_COL = 0, NEO_PK_NTT_ROW, NEO_PK_BCONV, NEO_PK_KEYIP, NEO_PK_COMBINE,
       NEO_PK_TENSOR, NEO_PK_AUTO, NEO_PK_MODSW, NEO_PK_RESCALE, NEO_PK_EW, NEO_PK_COUNT };
neo_status neo_profile_enable(int32_t on);
neo_status neo_profile_read(int32_t kind, double* total_ms, int32_t* launches);
/* Diagnostics: the recorded launches in issue order (at most max): kind and start / end time
 * in ms relative to the first recorded launch's start event (events of every stream). */
int32_t neo_profile_timeline(int32_t max, int32_t* kinds, float* start_ms, float* end_ms);

/* Diagnostics: when NEO_BCONV_DBG=1 is set in the environment before the first key-switch,
 * the tensor-core BConv records per-role clock64 stamps of CTA 0 (tiles 0..61: producer
 * start / A ready, MMA start / committed, epilogue start / end) and globaltimer stamps of the
 * setup phase (row 63) of the last ModUp and ModDown launch.  neo_debug_bconv_trace
 * synchronises the device and copies the 2 x 64 x 8 uint64 stamps (ModUp, then ModDown) to
 * `host` (caller-owned, 8 KB).  Returns 1 if tracing is on, 0 if it is off (host untouched). */
int32_t neo_debug_bconv_trace(unsigned long long* host);


#ifdef __cplusplus
}
#endif
#endif /* NEO_H */
