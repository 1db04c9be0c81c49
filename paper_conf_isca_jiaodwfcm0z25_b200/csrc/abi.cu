// abi.cpp -- the extern "C" entry points of libneo.so (include/neo.h) and the key-switch
// orchestrator (Fig. 5: INTT -> ModUp -> NTT -> KeyIP -> INTT -> ModDown -> NTT).
#include <algorithm>
#include <atomic>
#include <map>
#include <memory>
#include <cstdlib>
#include <cstring>
#include <new>
#include <string>

#include "bconv_tc.h"
#include "context.h"
#include "kernels.h"
#include "klss.h"
#include "ntt.h"
#include "ntt_tc.h"

namespace neo {
neo_status build_context(neo_ctx* c, const neo_params_desc* d, std::string& err);
}
using namespace neo;

static thread_local std::string g_err;
static thread_local int g_launches = 0;
// batch chunk of the key-switching ops (see CHUNKED below)
static int batch_chunk() {
    static int v = -1;
    if (v < 0) {
        const char* e = std::getenv("NEO_BATCH_CHUNK");
        v = e ? std::atoi(e) : 32;
        if (v < 1) v = 1 << 30;
    }
    return v;
}

#define FAIL(code, msg)      \
    do {                     \
        g_err = (msg);       \
        return (code);       \
    } while (0)
#define CK(x)                                                               \
    do {                                                                    \
        cudaError_t e_ = (x);                                               \
        if (e_ != cudaSuccess) {                                            \
            g_err = std::string("CUDA error: ") + cudaGetErrorString(e_);   \
            return NEO_ECUDA;                                               \
        }                                                                   \
    } while (0)

constexpr int NEO_HOST_ROWS = 1024;   // host row lists (split into launches of <= NEO_MAX_ROWS)
static inline cudaStream_t S(neo_stream_t s) { return reinterpret_cast<cudaStream_t>(s); }

// BConv pipeline trace (debug only, NEO_BCONV_DBG=1): CTA 0's clock64 stamps of the last launch
static unsigned long long* bconv_dbg() {
    static unsigned long long* p = nullptr;
    static bool tried = false;
    if (!tried) {
        tried = true;
        const char* e = std::getenv("NEO_BCONV_DBG");
        if (e && e[0] == '1') cudaMalloc(&p, 2 * 64 * 8 * sizeof(unsigned long long));
    }
    return p;
}

// ------------------------------------------------------------------ launch profiling
// Optional CUDA-event pairs around every launch (neo_profile_enable), read back per
// kernel kind by neo_profile_read; used by bench.py to time kernels inside its timed region.
enum { PK_NTT_COL = 0, PK_NTT_ROW, PK_BCONV, PK_KEYIP, PK_COMBINE, PK_TENSOR, PK_AUTO, PK_MODSW,
       PK_RESCALE, PK_EW, PK_COUNT };
struct ProfRec { int kind; cudaEvent_t a, b; };
static thread_local bool g_prof = false;
static thread_local std::vector<ProfRec> g_recs;
static thread_local std::vector<cudaEvent_t> g_pool;
static thread_local size_t g_pool_used = 0;

static cudaEvent_t prof_event() {
    if (g_pool_used == g_pool.size()) {
        cudaEvent_t e;
        cudaEventCreate(&e);
        g_pool.push_back(e);
    }
    return g_pool[g_pool_used++];
}
struct ProfScope {
    int kind; cudaStream_t st; cudaEvent_t a = nullptr;
    ProfScope(int k, cudaStream_t s) : kind(k), st(s) {
        if (g_prof) { a = prof_event(); cudaEventRecord(a, st); }
    }
    ~ProfScope() {
        if (a) { cudaEvent_t b = prof_event(); cudaEventRecord(b, st); g_recs.push_back({kind, a, b}); }
        ++g_launches;
    }
};
#define LAUNCH(kind, st, expr)          \
    do {                                \
        ProfScope ps_((kind), (st));    \
        CK(expr);                       \
    } while (0)

// ------------------------------------------------------------------ NTT over a row set
// rows k < n of batch entry b: src + b*src_bs + src_off[k]*N  ->  dst + b*dst_bs + dst_off[k]*N
// in_lazy: (forward) src holds lazy doubles from the tensor-core BConv; scale: (inverse) per-row
// constant folded into the column pass (Algorithm 2 line 1's [c qhat^-1] fused into the INTT).
static neo_status ntt_rows(const neo_ctx* c, bool fwd, const u64* src, long long src_bs, const int* src_off,
                           u64* dst, long long dst_bs, const int* dst_off, const int* prime, int n, u64* tmp,
                           int batch, cudaStream_t st, const RowEpi* epi = nullptr, bool in_lazy = false,
                           const TWD* scale = nullptr, unsigned galois = 0, const u64* fold = nullptr,
                           const TWD* fold_w = nullptr, const u64* sub = nullptr, long long sub_bs = 0,
                           bool src_dead = false, bool dst_keep = false) {
    if (n <= 0) return NEO_OK;
    if (n > NEO_MAX_ROWS) {               // more rows than one launch's descriptor holds: chunks
        if (epi || fold || sub) FAIL(NEO_EUNSUPPORTED, "too many limb rows for a fused-epilogue transform");
        for (int k0 = 0; k0 < n; k0 += NEO_MAX_ROWS) {
            const int m = std::min(NEO_MAX_ROWS, n - k0);
            neo_status s = ntt_rows(c, fwd, src, src_bs, src_off + k0, dst, dst_bs, dst_off + k0, prime + k0, m, tmp,
                                    batch, st, nullptr, in_lazy, scale ? scale + k0 : nullptr, galois, nullptr,
                                    nullptr, nullptr, 0, src_dead);
            if (s) return s;
        }
        return NEO_OK;
    }
    RowSet a, b;
    const long long N = c->N;
    a.n = b.n = n;
    a.in_lazy = fwd && in_lazy;
    a.has_scale = 0;
    b.in_lazy = 0;
    b.has_scale = (!fwd && scale) ? 1 : 0;
    // inverse transform of sigma_g(src): the automorphism is folded into the first (row) pass
    a.galois = b.galois = 0;
    a.galois_inv_n1 = b.galois_inv_n1 = 0;
    if (galois && !fwd) {
        a.galois = galois;
        unsigned gi = galois;                 // g^-1 mod 2^32 by Newton: g g = 1 mod 8 and every
        for (int it = 0; it < 4; ++it) gi *= 2u - galois * gi;   // x <- x (2 - g x) doubles the bits
        a.galois_inv_n1 = gi & (unsigned)(c->ntt.N1 - 1);
    }
    if (b.has_scale)
        for (int k = 0; k < n; ++k) b.scale[k] = scale[k];
    if (fwd && sub) {                     // forward column pass: x -= sub row k of entry b
        a.sub = sub;
        a.sub_bstride = sub_bs;
    }
    if (fwd && fold) {                    // forward column pass: x += fold[b] * fold_w[k]
        a.fold = fold;
        for (int k = 0; k < n; ++k) a.scale[k] = fold_w[k];
    }
    // first pass: src -> tmp ; second pass: tmp -> dst (tmp kept in L2, discarded once read: NEO_L2HINT=0 off)
    static const int l2h = [] { const char* e = std::getenv("NEO_L2HINT"); return (e && e[0] == '0') ? 0 : 1; }();
    // evict_last only while the intermediate fits comfortably in L2 (large batched launches would
    // pin more than the L2 holds: discard only)
    a.l2hint = b.l2hint = l2h ? (((size_t)n * batch * N * 8 <= ((size_t)48 << 20)) ? 2 : 1) : 0;
    a.src_dead = (src_dead && l2h) ? 1 : 0;
    static const bool keep = [] { const char* e = std::getenv("NEO_UPKEEP"); return !(e && e[0] == '0'); }();
    b.dst_keep = (keep && dst_keep && fwd && !epi && l2h && (size_t)n * batch * N * 8 <= ((size_t)64 << 20)) ? 1 : 0;
    a.src = src; a.src_bstride = src_bs;
    a.dst = tmp; a.dst_bstride = (long long)n * N;
    b.src = tmp; b.src_bstride = (long long)n * N;
    b.dst = dst; b.dst_bstride = dst_bs;
    for (int k = 0; k < n; ++k) {
        a.src_off[k] = src_off[k]; a.dst_off[k] = k; a.prime[k] = (short)prime[k];
        b.src_off[k] = k; b.dst_off[k] = dst_off[k]; b.prime[k] = (short)prime[k];
    }
    // forward: column pass then row pass; inverse: row pass then column pass
    if (c->ntt_impl == NEO_NTT_TC && c->ntt.tct) {     // both DFT stages of each pass on tcgen05
        LAUNCH(fwd ? PK_NTT_COL : PK_NTT_ROW, st, ntt_pass_tc(fwd, a, c->ntt, batch, fwd, st));
        LAUNCH(fwd ? PK_NTT_ROW : PK_NTT_COL, st, ntt_pass_tc(!fwd, b, c->ntt, batch, fwd, st, epi));
    } else {                                           // FP64 butterflies on the CUDA cores
        LAUNCH(fwd ? PK_NTT_COL : PK_NTT_ROW, st, ntt_pass(fwd, a, c->ntt, batch, fwd, st));
        LAUNCH(fwd ? PK_NTT_ROW : PK_NTT_COL, st, ntt_pass(!fwd, b, c->ntt, batch, fwd, st, epi));
    }
    return NEO_OK;
}

// ------------------------------------------------------------------ workspace layout
struct KsLayout {
    size_t y, up, acc, conv, pc, tmp, extra, total;   // u64 offsets
    // second scratch area for the two-stream forms (neo_hrot_hoisted: acc, conv, pc, tmp, extra;
    // neo_hrot_sum: y, up, tmp), 0 when the op has none
    size_t y2 = 0, up2 = 0, acc2 = 0, conv2 = 0, pc2 = 0, tmp2 = 0, extra2 = 0;
    KsLayout area2() const {               // the same layout with the second area's buffers
        KsLayout L = *this;
        if (acc2) { L.acc = acc2; L.conv = conv2; L.pc = pc2; L.tmp = tmp2; L.extra = extra2; }
        if (up2) { L.y = y2; L.up = up2; L.tmp = tmp2; }
        return L;
    }
};

static KsLayout ks_layout(const neo_ctx* c, int l, int B, int op) {
    const size_t N = c->N, Lq = l + 1, E = c->ext(l), beta = c->beta(l), P = c->num_p;
    KsLayout L;
    size_t o = 0;
    L.y = o; o += B * Lq * N;
    L.up = o; o += B * beta * E * N;
    L.acc = o; o += B * 2 * E * N;
    L.conv = o; o += B * 2 * Lq * N;
    L.pc = o; o += B * 2 * P * N;
    size_t tmp_rows = std::max(std::max(beta * E, 2 * Lq), 2 * P);
    if (op == NEO_OP_HMULT_RESCALE) tmp_rows = std::max(tmp_rows, 2 * P + 4);   // merged P-part + last-limb INTT
    L.tmp = o; o += B * tmp_rows * N;
    L.extra = o;
    if (op == NEO_OP_HMULT) o += B * 3 * Lq * N;
    if (op == NEO_OP_HMULT_RESCALE) o += B * 3 * Lq * N + 4 * B * N;   // d, then c_l scratch
    if (op == NEO_OP_HROT) o += B * Lq * N;                       // sigma_g(c0)
    if (op == NEO_OP_HROT_HOISTED) {
        o += B * 2 * Lq * N;                                       // pre (before the automorphism)
        L.acc2 = o; o += B * 2 * E * N;                            // second ModDown area (side stream)
        L.conv2 = o; o += B * 2 * Lq * N;
        L.pc2 = o; o += B * 2 * P * N;
        L.tmp2 = o; o += B * tmp_rows * N;
        L.extra2 = o; o += B * 2 * Lq * N;
    }
    if (op == NEO_OP_HROT_SUM) {
        o += B * 2 * Lq * N;                                       // sum of sigma_g(c0), one sigma_g(c0)
        L.y2 = o; o += B * Lq * N;                                 // second ModUp area (side stream)
        L.up2 = o; o += B * beta * E * N;
        L.tmp2 = o; o += B * tmp_rows * N;
    }
    L.total = o;
    return L;
}

// Two-stream forms of neo_hrot_hoisted / neo_hrot_sum at batch <= one chunk (NEO_TWO_STREAM=0 disables)
static bool two_stream_ok(const neo_ctx* c) {
    static const bool off = [] { const char* e = std::getenv("NEO_TWO_STREAM"); return e && e[0] == '0'; }();
    return c->side && !off;
}

static size_t klss_total(const neo_ctx* c, int l, int B, int op);
// offset (u64 words) of the op's extra buffers (tensor output d, sigma_g(c0)) in the workspace
static size_t extra_offset(const neo_ctx* c, const neo_evk* k, int l, int B, int op);

static size_t rescale_ws(const neo_ctx* c, int l, int B) {
    const size_t N = c->N;
    return (size_t)2 * B * N + (size_t)2 * B * std::max(l, 1) * N;
}

// Double Rescale: last2 [2B][2][N], corr [2B][l-1][N], NTT intermediate [2B][max(l-1, 2)][N]
static size_t ds_ws(const neo_ctx* c, int l, int B) {
    const size_t N = c->N;
    return (size_t)4 * B * N + (size_t)2 * B * (l - 1) * N + (size_t)2 * B * std::max(l - 1, 2) * N;
}

// ------------------------------------------------------------------ key-switch core
// a3-a5: ModUp of d (INTT, BConv of every digit onto PQ_l, NTT) into the workspace.
// The ModUp NTT's row pass can be fused with KeyIP (ntt.h KipArgs): ks_modup(..., fused) then
// stops after the column pass and ks_finish(..., fused) runs the fused pass instead of KeyIP.
// FP64 NTT only; the ModUp rows must fit one launch descriptor.
static bool kip_ok(const neo_ctx* c, int l) {
    if (c->ntt_impl == NEO_NTT_TC && c->ntt.tct) return false;
    const int E = c->ext(l), beta = c->beta(l);
    if (E > KIP_MAX_EXT || beta > KIP_MAX_BETA) return false;
    int n = 0;
    for (int j = 0; j < beta; ++j) n += E - (int)c->digits[l][j].size();
    static int on = -1;                  // measured slower than the separate KeyIP: opt-in
    if (on < 0) {
        const char* e = std::getenv("NEO_KIP");
        on = (e && e[0] == '1') ? 1 : 0;
    }
    return on && n <= NEO_MAX_ROWS;
}

static neo_status ks_modup(const neo_ctx* c, const u64* d, long long d_bs, int l, int B, u64* ws, const KsLayout& Ly,
                           cudaStream_t st, unsigned galois = 0, bool fused = false) {
    const int N = c->N, Lq = l + 1, E = c->ext(l), beta = c->beta(l);
    u64 *y = ws + Ly.y, *up = ws + Ly.up, *tmp = ws + Ly.tmp;
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    neo_status s;

    // a3: INTT of d (l+1 limbs) -> y (coefficient form); on the tensor-core path the ModUp
    // scaling y_i = [c_i qhat_i^-1]_{q_i} (Algorithm 2 line 1) is folded into the INTT
    for (int i = 0; i < Lq; ++i) { so[i] = i; dof[i] = i; pr[i] = i; }
    {
        TWD sc[NEO_MAX_ROWS];
        if (c->use_tc)
            for (int j = 0; j < beta; ++j)
                for (size_t u = 0; u < c->digits[l][j].size(); ++u) sc[c->digits[l][j][u]] = c->modup_tc[l][j].qhat_inv[u];
        if ((s = ntt_rows(c, false, d, d_bs, so, y, (long long)Lq * N, dof, pr, Lq, tmp, B, st, nullptr, false,
                          c->use_tc ? sc : nullptr, galois)))
            return s;
    }

    // a4: ModUp BConv of all beta digits: y[D_j] -> up[j][targets]  (one launch on tensor cores)
    {
        BConvMulti M;
        M.centred = 0;
        M.dbg = bconv_dbg();
        M.njobs = 0;
        M.pre_scaled = 1;
        M.lazy_out = 1;
        for (int j = 0; j < beta; ++j) {
            const BConvTab& T = c->modup[l][j];
            const std::vector<int>& dj = c->digits[l][j];
            BConvIO io;
            io.in = y; io.out = up;
            io.in_bstride = (long long)Lq * N;
            io.out_bstride = (long long)beta * E * N;
            for (int i = 0; i < T.n_in; ++i) io.in_off[i] = dj[i];
            int o = 0;
            for (int pos = 0; pos < E; ++pos) {
                int id = c->ext_id(l, pos);
                if (std::find(dj.begin(), dj.end(), id) != dj.end()) continue;
                io.out_off[o++] = j * E + pos;
            }
            if (c->use_tc) {
                if (M.njobs && !bconv_multi_fits(M, c->modup_tc[l][j])) {   // job / part limits of one launch
                    LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, B, c->num_sms, st));
                    M.njobs = 0;
                }
                M.P[M.njobs] = c->modup_tc[l][j];
                M.io[M.njobs] = io;
                M.bmat[M.njobs] = c->d_bmat + c->modup_boff[l][j];
                ++M.njobs;
            } else {
                LAUNCH(PK_BCONV, st, launch_bconv(T, io, N, B, st));
            }
        }
        if (M.njobs) LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, B, c->num_sms, st));
    }

    // a5: NTT of every ModUp output row
    int n = 0;
    for (int j = 0; j < beta; ++j) {
        const std::vector<int>& dj = c->digits[l][j];
        for (int pos = 0; pos < E; ++pos) {
            int id = c->ext_id(l, pos);
            if (std::find(dj.begin(), dj.end(), id) != dj.end()) continue;
            so[n] = dof[n] = j * E + pos;
            pr[n] = id;
            ++n;
        }
    }
    if (fused) {            // column pass only: the row pass runs fused with KeyIP in ks_finish
        RowSet a;
        a.n = n;
        a.in_lazy = c->use_tc ? 1 : 0;
        a.has_scale = 0;
        a.galois = 0;
        a.galois_inv_n1 = 0;
        a.src = up; a.src_bstride = (long long)beta * E * N;
        a.dst = tmp; a.dst_bstride = (long long)n * N;
        for (int k = 0; k < n; ++k) { a.src_off[k] = so[k]; a.dst_off[k] = k; a.prime[k] = (short)pr[k]; }
        LAUNCH(PK_NTT_COL, st, ntt_pass(true, a, c->ntt, B, true, st));
        return NEO_OK;
    }
    if ((s = ntt_rows(c, true, up, (long long)beta * E * N, so, up, (long long)beta * E * N, dof, pr, n, tmp, B, st,
                      nullptr, c->use_tc, nullptr, 0, nullptr, nullptr, nullptr, 0, true,    // BConv output: dead
                      true)))                                                               // KeyIP reads up next
        return s;

    return NEO_OK;
}

// a6-a10: KeyIP of the ModUp outputs (and d's own digit limbs) with key k, ModDown, combine.
static neo_status ks_finish(const neo_ctx* c, const neo_evk* k, const u64* d, long long d_bs, int l, int B,
                            u64* ws, const KsLayout& Ly, u64* out0, u64* out1, long long out_bs,
                            const u64* add0, const u64* add1, long long add_bs, cudaStream_t st,
                            unsigned galois = 0, bool add_galois = true, u64* hmr_last = nullptr,
                            int phase = 0, bool fused = false) {
    // phase 0: KeyIP then ModDown; 1: KeyIP only (acc overwritten); 2: KeyIP only, accumulated
    // into acc; 3: ModDown only (of the acc already in the workspace) -- neo_hrot_sum
    // hmr_last != nullptr: fused HMULT + Rescale (neo_hmult_rescale).  add0/add1 are then d0/d1
    // (stride add_bs), out0/out1 receive the rescaled ciphertext at level l - 1, and hmr_last
    // is scratch [2][2B][N] for the coefficient form of acc_c and d_c at limb l.
    const int N = c->N, Lq = l + 1, E = c->ext(l), beta = c->beta(l), P = c->num_p;
    u64 *up = ws + Ly.up, *acc = ws + Ly.acc, *conv = ws + Ly.conv, *pc = ws + Ly.pc, *tmp = ws + Ly.tmp;
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    neo_status s;

    // a5 row pass + a6 fused: acc straight from the column-pass intermediates (ntt.h KipArgs)
    if (phase != 3 && fused) {
        KipArgs A;
        A.tmp = reinterpret_cast<const double*>(ws + Ly.tmp);
        int n = 0;
        for (int pos = 0; pos < E; ++pos) { A.ntr[pos] = 0; A.own[pos] = -1; }
        for (int j = 0; j < beta; ++j) {                 // the row order of ks_modup's column pass
            const std::vector<int>& dj = c->digits[l][j];
            for (int pos = 0; pos < E; ++pos) {
                const int id = c->ext_id(l, pos);
                if (std::find(dj.begin(), dj.end(), id) != dj.end()) { A.own[pos] = (signed char)j; continue; }
                A.dig[pos][A.ntr[pos]] = (unsigned char)j;
                A.row[pos][A.ntr[pos]++] = (short)n++;
            }
        }
        for (int pos = 0; pos < E; ++pos) A.limb[pos] = c->ext_id(l, pos);
        A.tmp_bstride = (long long)n * N;
        A.d = d; A.d_bstride = d_bs; A.galois = galois;
        A.evk_lo = k->lo; A.evk_hi = k->hi; A.evk_limbs = c->num_q + c->num_p;
        A.acc = acc;
        A.acc_bstride = (long long)2 * E * N;
        A.acc_cstride = (long long)E * N;
        A.mods = c->d_mods;
        A.accumulate = phase == 2;
        LAUNCH(PK_NTT_ROW, st, ntt_row_kip(c->ntt, A, E, B, st));
    } else if (phase != 3) {   // a6: KeyIP over all E limbs of PQ_l
        KeyIPArgs A;
        A.d = d; A.up = up; A.evk_lo = k->lo; A.evk_hi = k->hi; A.acc = acc; A.mods = c->d_mods;
        A.d_bstride = d_bs;
        A.up_bstride = (long long)beta * E * N;
        A.acc_bstride = (long long)2 * E * N;
        A.acc_cstride = (long long)E * N;
        A.N = N; A.beta = beta; A.evk_limbs = c->num_q + c->num_p;
        A.galois = galois;                     // d's own digit limbs are read as sigma_g(d)
        A.accumulate = phase == 2;
        for (int pos = 0; pos < E; ++pos) {
            int id = c->ext_id(l, pos);
            A.limb[pos] = id;
            for (int j = 0; j < beta; ++j) {
                const std::vector<int>& dj = c->digits[l][j];
                bool own = std::find(dj.begin(), dj.end(), id) != dj.end();
                A.src_kind[j][pos] = own ? 0 : 1;
                A.src_off[j][pos] = own ? id : j * E + pos;
            }
        }
        LAUNCH(PK_KEYIP, st, launch_keyip(A, E, B, st));
    }
    if (phase == 1 || phase == 2) return NEO_OK;

    // a7: INTT of the P part of acc_0, acc_1 -> pc [2B][P][N], with ModDown's [a_k Phat_k^-1] folded in.
    // Fused HMULT + Rescale at small batch: the 4B last-limb rows (acc_c,l and d_c,l, needed in
    // coefficient form below) join the same launch as extra rows (scale 1), one INTT instead of two.
    const bool hmr_merged = hmr_last && (2 * P + 4) * B <= NEO_MAX_ROWS;
    if (hmr_merged) {
        const u64* base = std::min<const u64*>(acc, add0);
        const long long oa = (acc - base) / N, od = (add0 - base) / N, d1 = (add1 - add0) / N;
        const long long oh = (hmr_last - pc) / N;            // hmr_last lies after pc in the workspace
        TWD sc[NEO_MAX_ROWS];
        const TWD one{1.0, 1.0 / (double)c->mod[l]};
        int n = 0;
        for (int b = 0; b < B; ++b)
            for (int cc = 0; cc < 2; ++cc)
                for (int k2 = 0; k2 < P; ++k2) {
                    so[n] = (int)(oa + (long long)b * 2 * E + (long long)cc * E + Lq + k2);
                    dof[n] = (2 * b + cc) * P + k2;
                    pr[n] = c->num_q + k2;
                    sc[n++] = c->use_tc ? c->moddown_tc[l].qhat_inv[k2] : TWD{1.0, 1.0 / (double)c->mod[c->num_q + k2]};
                }
        for (int b = 0; b < B; ++b)
            for (int cc = 0; cc < 2; ++cc) {
                so[n] = (int)(oa + (long long)b * 2 * E + (long long)cc * E + l);
                dof[n] = (int)(oh + 2 * b + cc);
                pr[n] = l;
                sc[n++] = one;
                so[n] = (int)(od + (long long)b * (add_bs / N) + cc * d1 + l);
                dof[n] = (int)(oh + 2 * B + 2 * b + cc);
                pr[n] = l;
                sc[n++] = one;
            }
        if ((s = ntt_rows(c, false, base, 0, so, pc, 0, dof, pr, n, tmp, 1, st, nullptr, false, sc, 0, nullptr, nullptr,
                          nullptr, 0, true)))        // acc's P and last rows, d's last rows: read only here
            return s;
    } else {
        for (int k2 = 0; k2 < P; ++k2) { so[k2] = Lq + k2; dof[k2] = k2; pr[k2] = c->num_q + k2; }
        if ((s = ntt_rows(c, false, acc, (long long)E * N, so, pc, (long long)P * N, dof, pr, P, tmp, 2 * B, st, nullptr,
                          false, c->use_tc ? c->moddown_tc[l].qhat_inv : nullptr, 0, nullptr, nullptr, nullptr, 0,
                          true)))                    // acc's P rows: read only here
            return s;
    }

    // a8: ModDown BConv P -> q_0..q_l, batch 2B
    {
        const BConvTab& T = c->moddown[l];
        BConvIO io;
        io.in = pc; io.out = conv;
        io.in_bstride = (long long)P * N;
        io.out_bstride = (long long)Lq * N;
        for (int i = 0; i < P; ++i) io.in_off[i] = i;
        for (int i = 0; i < Lq; ++i) io.out_off[i] = i;
        if (c->use_tc) {
            BConvMulti M;
            M.centred = 0;
        M.centred = 0;
            M.dbg = bconv_dbg() ? bconv_dbg() + 512 : nullptr;
            M.njobs = 1;
            M.pre_scaled = 1;
            M.lazy_out = 1;
            M.P[0] = c->moddown_tc[l];
            M.io[0] = io;
            M.bmat[0] = c->d_bmat + c->moddown_boff[l];
            LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, 2 * B, c->num_sms, st));
        } else
            LAUNCH(PK_BCONV, st, launch_bconv(T, io, N, 2 * B, st));
    }

    if (hmr_last) {
        // Rescale folded into ModDown: c_l = INTT(acc_l - NTT(conv_l)) P^-1 + INTT(d_l) is the
        // coefficient form of the HMULT output's last limb; conv_i += P c_l for i < l, and the
        // tail below becomes ((acc_i - NTT(conv_i)) P^-1 + d_i) q_l^-1 = Rescale(HMULT) exactly.
        u64* accl = hmr_last;
        u64* dl = hmr_last + (size_t)2 * B * N;
        // the 4 rows acc_0,l acc_1,l d_0,l d_1,l of every batch entry in ONE inverse transform
        // (rows addressed from the lower of the two workspace buffers; batch entries as rows),
        // unless they already went with the P part above
        if (!hmr_merged) {
            const u64* base = std::min<const u64*>(acc, add0);
            const long long oa = (acc - base) / N, od = (add0 - base) / N, d1 = (add1 - add0) / N;
            int n = 0;
            for (int b = 0; b < B; ++b)
                for (int cc = 0; cc < 2; ++cc) {
                    so[n] = (int)(oa + (long long)b * 2 * E + (long long)cc * E + l);
                    dof[n] = 2 * b + cc;
                    pr[n++] = l;
                    so[n] = (int)(od + (long long)b * (add_bs / N) + cc * d1 + l);
                    dof[n] = 2 * B + 2 * b + cc;
                    pr[n++] = l;
                }
            if ((s = ntt_rows(c, false, base, 0, so, hmr_last, 0, dof, pr, n, tmp, 1, st))) return s;
        }
        HmrFoldArgs F;
        F.conv = conv; F.accl = accl; F.dl = dl; F.mods = c->d_mods;
        F.pinv_l = c->pinv[l];
        for (int i = 0; i < l; ++i) {
            const u64 qi = c->mod[i];
            u64 pm = 1;
            for (int k2 = 0; k2 < P; ++k2) pm = (u64)((u128)pm * (c->mod[c->num_q + k2] % qi) % qi);
            F.pmod[i].w = (double)pm;
            F.pmod[i].wq = (double)pm / (double)qi;
        }
        F.N = N; F.l = l; F.lazy = c->use_tc ? 1 : 0;
        // FP64 NTT: c_l alone here, conv_i += P c_l inside the next column pass (RowSet::fold)
        const bool fold_fused = !(c->ntt_impl == NEO_NTT_TC && c->ntt.tct);
        if (fold_fused) LAUNCH(PK_EW, st, launch_hmr_cl(F, 2 * B, st));
        else LAUNCH(PK_EW, st, launch_hmr_fold(F, 2 * B, st));
        for (int i = 0; i < l; ++i) { so[i] = dof[i] = i; pr[i] = i; }
        RowEpi ep;
        ep.acc = acc;
        ep.acc_b = (long long)2 * E * N;
        ep.acc_c = (long long)E * N;
        ep.add0 = add0; ep.add1 = add1; ep.add_b = add_bs;
        ep.out0 = out0; ep.out1 = out1; ep.out_b = out_bs;
        ep.add_galois = 0;
        ep.has_post = 1;
        for (int i = 0; i < l; ++i) { ep.pinv[i] = c->pinv[i]; ep.post[i] = c->ql_inv[l][i]; }
        return ntt_rows(c, true, conv, (long long)Lq * N, so, conv, (long long)Lq * N, dof, pr, l, tmp, 2 * B, st,
                        &ep, c->use_tc, nullptr, 0, fold_fused ? accl : nullptr, F.pmod, nullptr, 0, true);
    }

    // a9 + a10: NTT of conv, with the ModDown tail (acc - conv) * P^-1 (+ add) fused into the
    // epilogue of the row pass (conv is never written back)
    for (int i = 0; i < Lq; ++i) { so[i] = dof[i] = i; pr[i] = i; }
    {
        RowEpi ep;
        ep.acc = acc;
        ep.acc_b = (long long)2 * E * N;
        ep.acc_c = (long long)E * N;
        ep.add0 = add0; ep.add1 = add1; ep.add_b = add_bs;
        ep.out0 = out0; ep.out1 = out1; ep.out_b = out_bs;
        ep.add_galois = add_galois ? galois : 0;   // add0 gathered through sigma_g
        for (int i = 0; i < Lq; ++i) ep.pinv[i] = c->pinv[i];
        if ((s = ntt_rows(c, true, conv, (long long)Lq * N, so, conv, (long long)Lq * N, dof, pr, Lq, tmp, 2 * B, st,
                          &ep, c->use_tc, nullptr, 0, nullptr, nullptr, nullptr, 0, true)))   // conv: dead after
            return s;
    }
    return NEO_OK;
}

// ------------------------------------------------------------------ KLSS key-switch
// Workspace: y [B][Lq], up [B][beta][alpha'] (T basis), accT [B][2][beta~][alpha'],
// rec [B][2][E] (PQ_l, coefficient form), conv [2B][Lq], NTT intermediate.
struct KlssLayout {
    size_t y, up, acc, rec, conv, tmp, extra, total;
};

static KlssLayout klss_layout(const neo_ctx* c, int l, int B, int op) {
    const size_t N = c->N, Lq = l + 1, E = c->ext(l), beta = c->beta(l), ap = c->num_t,
                 bt = c->klss_groups.size();
    KlssLayout L;
    size_t o = 0;
    L.y = o; o += B * Lq * N;
    L.up = o; o += B * beta * ap * N;
    L.acc = o; o += B * 2 * bt * ap * N;
    L.rec = o; o += B * 2 * E * N;
    L.conv = o; o += B * 2 * Lq * N;
    L.tmp = o; o += B * std::max(std::max(beta * ap, 2 * bt * ap), 2 * Lq) * N;
    L.extra = o;
    if (op == NEO_OP_HMULT) o += B * 3 * Lq * N;
    if (op == NEO_OP_HMULT_RESCALE) o += B * 3 * Lq * N + 4 * B * N;   // d, then c_l scratch
    if (op == NEO_OP_HROT) o += B * Lq * N;
    L.total = o;
    return L;
}

static size_t klss_total(const neo_ctx* c, int l, int B, int op) { return klss_layout(c, l, B, op).total; }
static size_t extra_offset(const neo_ctx* c, const neo_evk* k, int l, int B, int op) {
    return k->klss ? klss_layout(c, l, B, op).extra : ks_layout(c, l, B, op).extra;
}

// KLSS (L155-180, Fig. 5): INTT -> ModUp (Eq. 3) -> NTT over T -> IP (Alg. 3/4) -> INTT over T
// -> Recover Limbs -> ModDown (Table 2) -> NTT; readings K1-K6.
static neo_status klss_core(const neo_ctx* c, const neo_evk* k, const u64* d, long long d_bs, int l, int B,
                            u64* ws, const KlssLayout& Ly, u64* out0, u64* out1, long long out_bs,
                            const u64* add0, const u64* add1, long long add_bs, cudaStream_t st, unsigned galois) {
    const int N = c->N, Lq = l + 1, E = c->ext(l), beta = c->beta(l), P = c->num_p, ap = c->num_t;
    const int bt = (int)c->klss_groups.size(), nl = c->num_q + c->num_p;
    if (beta > KLSS_MAX_BETA || bt > KLSS_MAX_GROUPS || c->alpha_t > KLSS_MAX_OUT_G)
        FAIL(NEO_EUNSUPPORTED, "KLSS: too many digits, groups (<= 8) or limbs per group (<= 16)");
    const bool wide = c->word_bits_t > 40;     // 48-bit T words: 6-byte BConv constants, 64-bit IP / Recover
    if (wide && !c->use_tc) FAIL(NEO_EUNSUPPORTED, "KLSS with WordSize_T > 40 needs the tensor-core BConv");
    if ((k->hi_bytes == 2) != wide) FAIL(NEO_EINVAL, "KLSS key packed for another WordSize_T");
    u64 *y = ws + Ly.y, *up = ws + Ly.up, *acc = ws + Ly.acc, *rec = ws + Ly.rec, *conv = ws + Ly.conv,
        *tmp = ws + Ly.tmp;
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    neo_status s;
    // 1. INTT of d; Algorithm 2's [c_i qhat_i^-1]_{q_i} folded in (the digits are Hybrid's)
    for (int i = 0; i < Lq; ++i) { so[i] = i; dof[i] = i; pr[i] = i; }
    {
        TWD sc[NEO_MAX_ROWS];
        if (c->use_tc)
            for (int j = 0; j < beta; ++j)
                for (size_t u = 0; u < c->digits[l][j].size(); ++u) sc[c->digits[l][j][u]] = c->klss_up_tc[l][j].qhat_inv[u];
        if ((s = ntt_rows(c, false, d, d_bs, so, y, (long long)Lq * N, dof, pr, Lq, tmp, B, st, nullptr, false,
                          c->use_tc ? sc : nullptr, galois)))
            return s;
    }
    // 2. ModUp: every digit -> the alpha' T limbs (Eq. 3, Algorithm 1)
    {
        BConvMulti M;
        M.centred = 0;
        M.dbg = nullptr;
        M.njobs = 0;
        M.pre_scaled = 1;
        M.lazy_out = 1;
        for (int j = 0; j < beta; ++j) {
            const std::vector<int>& dj = c->digits[l][j];
            BConvIO io;
            io.in = y; io.out = up;
            io.in_bstride = (long long)Lq * N;
            io.out_bstride = (long long)beta * ap * N;
            for (size_t i = 0; i < dj.size(); ++i) io.in_off[i] = dj[i];
            for (int t = 0; t < ap; ++t) io.out_off[t] = j * ap + t;
            if (c->use_tc) {
                if (M.njobs && !bconv_multi_fits(M, c->klss_up_tc[l][j])) {
                    LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, B, c->num_sms, st));
                    M.njobs = 0;
                }
                M.P[M.njobs] = c->klss_up_tc[l][j];
                M.io[M.njobs] = io;
                M.bmat[M.njobs] = c->d_bmat + c->klss_up_boff[l][j];
                ++M.njobs;
            } else {
                LAUNCH(PK_BCONV, st, launch_bconv(c->klss_up[l][j], io, N, B, st));
            }
        }
        if (M.njobs) LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, B, c->num_sms, st));
    }
    // 3. NTT over T of the beta * alpha' rows
    for (int j = 0; j < beta; ++j)
        for (int t = 0; t < ap; ++t) { so[j * ap + t] = dof[j * ap + t] = j * ap + t; pr[j * ap + t] = nl + t; }
    if ((s = ntt_rows(c, true, up, (long long)beta * ap * N, so, up, (long long)beta * ap * N, dof, pr, beta * ap, tmp,
                      B, st, nullptr, c->use_tc)))
        return s;
    // 4. IP over T for the groups present at level l
    KlssIpArgs I;
    I.up = up; I.key_lo = k->lo; I.key_hi = k->hi; I.acc = acc; I.mods = c->d_mods;
    I.N = N; I.beta = beta; I.dnum = c->dnum; I.beta_t = bt; I.alpha_p = ap; I.t0 = nl;
    KlssRecArgs R;
    R.acc = acc; R.rec = rec; R.tab = c->d_rec; R.mods = c->d_mods;
    R.N = N; R.alpha_p = ap; R.beta_t = bt; R.t0 = nl; R.E = E;
    int ng = 0, no = 0;
    for (int i = 0; i < bt; ++i) {
        int first = no;
        for (int id : c->klss_groups[i]) {
            const bool present = id <= l || id >= c->num_q;
            if (!present) continue;
            R.out_id[no] = id;
            R.out_pos[no] = id <= l ? id : Lq + (id - c->num_q);
            ++no;
        }
        if (no > first) {
            I.group[ng] = R.group[ng] = i;
            R.first[ng] = first;
            ++ng;
        }
    }
    R.first[ng] = no;
    I.n_groups = R.n_groups = ng;
    LAUNCH(PK_KEYIP, st, wide ? launch_klss_ip48(I, B, st) : launch_klss_ip(I, B, st));
    // 5. INTT over T of the 2 * (present groups) * alpha' rows (in place, coefficient form)
    int nr = 0;
    for (int cc = 0; cc < 2; ++cc)
        for (int g = 0; g < ng; ++g)
            for (int t = 0; t < ap; ++t) {
                so[nr] = dof[nr] = (cc * bt + I.group[g]) * ap + t;
                pr[nr] = nl + t;
                ++nr;
            }
    if (nr > NEO_MAX_ROWS) FAIL(NEO_EUNSUPPORTED, "KLSS: too many T rows for one transform");
    // Recover Limbs engine: CUDA cores by default (16 small conversions: the tensor-core kernel's
    // per-tile pipeline cost dominates, measured 0.136 vs 0.102 ms per KS at Set-C); NEO_KLSS_REC=tc
    // selects the tensor-core conversion with the centred-correction column
    static const bool rec_tc = [] { const char* e = std::getenv("NEO_KLSS_REC"); return e && std::string(e) == "tc"; }();
    const bool use_rec_tc = c->use_tc && rec_tc && c->klss_rec_tc_ok;
    TWD tsc[NEO_HOST_ROWS];                // tensor-core Recover: [That_k^-1]_{t_k} folded into the INTT
    if (use_rec_tc)
        for (int r = 0; r < nr; ++r) tsc[r] = c->klss_rec_tc[l][I.group[0]].qhat_inv[r % ap];
    if ((s = ntt_rows(c, false, acc, (long long)2 * bt * ap * N, so, acc, (long long)2 * bt * ap * N, dof, pr, nr,
                      tmp, B, st, nullptr, false, use_rec_tc ? tsc : nullptr)))
        return s;
    // 6. Recover Limbs: exact centred CRT from T to the PQ_l limbs (K4): on tensor cores, one
    //    conversion per (group, component) with the centred-correction column; else CUDA cores
    if (use_rec_tc) {
        BConvMulti M;
        M.dbg = nullptr;
        M.njobs = 0;
        M.pre_scaled = 1;
        M.lazy_out = 0;
        M.centred = 1;
        for (int cc = 0; cc < 2; ++cc)
            for (int g = 0; g < ng; ++g) {
                const int i = I.group[g];
                BConvIO io;
                io.in = acc + (size_t)(cc * bt + i) * ap * N;
                io.out = rec + (size_t)cc * E * N;
                io.in_bstride = (long long)2 * bt * ap * N;
                io.out_bstride = (long long)2 * E * N;
                for (int t = 0; t < ap; ++t) io.in_off[t] = t;
                for (int o = R.first[g]; o < R.first[g + 1]; ++o) io.out_off[o - R.first[g]] = R.out_pos[o];
                if (M.njobs && !bconv_multi_fits(M, c->klss_rec_tc[l][i])) {
                    LAUNCH(PK_COMBINE, st, launch_bconv_tc(M, N, B, c->num_sms, st));
                    M.njobs = 0;
                }
                M.P[M.njobs] = c->klss_rec_tc[l][i];
                M.io[M.njobs] = io;
                M.bmat[M.njobs] = c->d_bmat + c->klss_rec_boff[l][i];
                ++M.njobs;
            }
        if (M.njobs) LAUNCH(PK_COMBINE, st, launch_bconv_tc(M, N, B, c->num_sms, st));
    } else {
        LAUNCH(PK_COMBINE, st, wide ? launch_klss_recover48(R, B, st) : launch_klss_recover(R, B, st));
    }
    // 7. ModDown BConv P -> Q_l on the recovered (coefficient-form) P limbs, batch 2B
    {
        BConvIO io;
        io.in = rec; io.out = conv;
        io.in_bstride = (long long)E * N;
        io.out_bstride = (long long)Lq * N;
        for (int i = 0; i < P; ++i) io.in_off[i] = Lq + i;
        for (int i = 0; i < Lq; ++i) io.out_off[i] = i;
        if (c->use_tc) {                        // canonical u64 out (the next column pass reads it)
            BConvMulti M;
            M.centred = 0;
        M.centred = 0;
            M.dbg = nullptr;
            M.njobs = 1;
            M.pre_scaled = 0;
            M.lazy_out = 0;
            M.P[0] = c->moddown_tc[l];
            M.io[0] = io;
            M.bmat[0] = c->d_bmat + c->moddown_boff[l];
            LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, 2 * B, c->num_sms, st));
        } else {
            LAUNCH(PK_BCONV, st, launch_bconv(c->moddown[l], io, N, 2 * B, st));
        }
    }
    // 8. (conv - acc_Q) in coefficient form, subtracted inside the column pass of 9. its NTT with
    //    the tail out_c = (0 - NTT(conv - acc_Q)) P^-1 (+ add_c) = NTT((acc_Q - conv) P^-1) (+ add_c)   (K5)
    for (int i = 0; i < Lq; ++i) { so[i] = dof[i] = i; pr[i] = i; }
    RowEpi ep;
    ep.acc = nullptr;
    ep.acc_b = ep.acc_c = 0;
    ep.add0 = add0; ep.add1 = add1; ep.add_b = add_bs;
    ep.out0 = out0; ep.out1 = out1; ep.out_b = out_bs;
    ep.add_galois = 0;
    for (int i = 0; i < Lq; ++i) ep.pinv[i] = c->pinv[i];
    return ntt_rows(c, true, conv, (long long)Lq * N, so, conv, (long long)Lq * N, dof, pr, Lq, tmp, 2 * B, st, &ep,
                    false, nullptr, 0, nullptr, nullptr, rec, (long long)E * N, true);
}

static neo_status ks_core(const neo_ctx* c, const neo_evk* k, const u64* d, long long d_bs, int l, int B,
                          u64* ws, const KsLayout& Ly, u64* out0, u64* out1, long long out_bs,
                          const u64* add0, const u64* add1, long long add_bs, cudaStream_t st,
                          unsigned galois = 0, bool add_galois = true) {
    if (k->klss)           // the key decides the method; c0's automorphism was applied by the caller
        return klss_core(c, k, d, d_bs, l, B, ws, klss_layout(c, l, B, NEO_OP_KEYSWITCH), out0, out1, out_bs, add0,
                         add1, add_bs, st, galois);
    const bool fused = kip_ok(c, l);
    neo_status s = ks_modup(c, d, d_bs, l, B, ws, Ly, st, galois, fused);
    if (s) return s;
    return ks_finish(c, k, d, d_bs, l, B, ws, Ly, out0, out1, out_bs, add0, add1, add_bs, st, galois, add_galois,
                     nullptr, 0, fused);
}

// ------------------------------------------------------------------ validation helpers
static neo_status check_ctx(const neo_ctx* c) {
    if (!c) FAIL(NEO_EINVAL, "null context");
    return NEO_OK;
}
static neo_status check_level(const neo_ctx* c, int level, int batch) {
    if (level < 0 || level >= c->num_q) FAIL(NEO_EINVAL, "level out of range");
    if (batch <= 0) FAIL(NEO_EINVAL, "batch must be positive");
    return NEO_OK;
}
static neo_status check_ws(const neo_ctx* c, int op, int level, int batch, const void* ws, size_t bytes) {
    size_t need = neo_workspace_size(c, op, level, batch);
    if (!ws || bytes < need) FAIL(NEO_EINVAL, "workspace missing or too small (see neo_workspace_size)");
    if (reinterpret_cast<uintptr_t>(ws) % 16) FAIL(NEO_EINVAL, "workspace must be 16-byte aligned");
    return NEO_OK;
}
static neo_status check_ptr(const void* p, const char* what) {
    if (!p) FAIL(NEO_EINVAL, std::string("null pointer: ") + what);
    if (reinterpret_cast<uintptr_t>(p) % 16) FAIL(NEO_EINVAL, std::string("pointer not 16-byte aligned: ") + what);
    return NEO_OK;
}
#define TRY(x)                      \
    do {                            \
        neo_status s_ = (x);        \
        if (s_ != NEO_OK) return s_; \
    } while (0)

// ------------------------------------------------------------------ C ABI
// Chunks alternate between the caller's stream and the context's side stream (fork / join
// through events, so the call stays asynchronous and ordered on the caller's stream, and is
// capturable in a CUDA graph): chunk k+1's FP64-bound NTTs overlap chunk k's HBM-bound KeyIP /
// BConv.  Each stream gets its own half of the workspace (neo_workspace_size reserves two
// chunks' worth for batches above the chunk).
template <class F>
static neo_status run_chunked(const neo_ctx* c, int batch, void* ws, size_t ws_bytes, size_t chunk_ws,
                              cudaStream_t st, F&& f) {
    static thread_local cudaEvent_t ev_fork = nullptr, ev_join = nullptr;
    if (!ev_fork) {
        cudaEventCreateWithFlags(&ev_fork, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&ev_join, cudaEventDisableTiming);
    }
    const int ch = batch_chunk();
    const bool two = c->side && ws_bytes >= 2 * chunk_ws;
    if (two) {
        CK(cudaEventRecord(ev_fork, st));
        CK(cudaStreamWaitEvent(c->side, ev_fork, 0));
    }
    int launches = 0, k = 0;
    for (int b0 = 0; b0 < batch; b0 += ch, ++k) {
        const int nb = std::min(ch, batch - b0);
        const bool alt = two && (k & 1);
        void* wk = alt ? static_cast<void*>(static_cast<char*>(ws) + chunk_ws) : ws;
        neo_status s = f(b0, nb, wk, alt ? chunk_ws : (two ? chunk_ws : ws_bytes), alt ? c->side : st);
        launches += g_launches;
        if (s != NEO_OK) {
            if (two) {                     // still join the side stream (keeps a graph capture valid)
                const std::string msg = g_err;
                cudaEventRecord(ev_join, c->side);
                cudaStreamWaitEvent(st, ev_join, 0);
                g_err = msg;
            }
            return s;
        }
    }
    if (two) {
        CK(cudaEventRecord(ev_join, c->side));
        CK(cudaStreamWaitEvent(st, ev_join, 0));
    }
    g_launches = launches;
    return NEO_OK;
}

extern "C" {

const char* neo_last_error(void) { return g_err.c_str(); }

// Debug: copy the BConv pipeline traces (ModUp, ModDown: 2 x 64 x 8 stamps) to host; 0 if tracing is off.
int32_t neo_debug_bconv_trace(unsigned long long* host) {
    unsigned long long* p = bconv_dbg();
    if (!p || !host) return 0;
    cudaDeviceSynchronize();
    cudaMemcpy(host, p, 2 * 64 * 8 * sizeof(unsigned long long), cudaMemcpyDeviceToHost);
    return 1;
}

neo_status neo_profile_enable(int32_t on) {
    g_recs.clear();
    g_pool_used = 0;
    g_prof = on != 0;
    return NEO_OK;
}

int32_t neo_profile_timeline(int32_t max, int32_t* kinds, float* start_ms, float* end_ms) {
    if (g_recs.empty()) return 0;
    cudaEventSynchronize(g_recs.back().b);
    int n = 0;
    for (const ProfRec& r : g_recs) {
        if (n >= max) break;
        float a = 0, b = 0;
        cudaEventSynchronize(r.b);
        cudaEventElapsedTime(&a, g_recs[0].a, r.a);
        cudaEventElapsedTime(&b, g_recs[0].a, r.b);
        if (kinds) kinds[n] = r.kind;
        if (start_ms) start_ms[n] = a;
        if (end_ms) end_ms[n] = b;
        ++n;
    }
    return n;
}

neo_status neo_profile_read(int32_t kind, double* total_ms, int32_t* launches) {
    if (kind < 0 || kind >= PK_COUNT || !total_ms || !launches) FAIL(NEO_EINVAL, "bad profile kind or null output");
    double t = 0;
    int n = 0;
    for (const ProfRec& r : g_recs) {
        if (r.kind != kind) continue;
        CK(cudaEventSynchronize(r.b));
        float ms = 0;
        CK(cudaEventElapsedTime(&ms, r.a, r.b));
        t += ms;
        ++n;
    }
    *total_ms = t;
    *launches = n;
    return NEO_OK;
}
int32_t neo_last_launch_count(void) { return g_launches; }

neo_status neo_params_create(const neo_params_desc* desc, neo_ctx** out) {
    if (!desc || !out) FAIL(NEO_EINVAL, "null argument");
    *out = nullptr;
    if (desc->log_n != 12 && desc->log_n != 16) FAIL(NEO_EUNSUPPORTED, "log_n must be 12 or 16 in this build");
    if (desc->word_bits != 36) FAIL(NEO_EUNSUPPORTED, "word_bits must be 36 in this build");
    if (desc->num_q < 1 || desc->num_p < 1 || desc->dnum < 1 || desc->dnum > desc->num_q)
        FAIL(NEO_EINVAL, "need num_q >= 1, num_p >= 1, 1 <= dnum <= num_q");
    if (desc->num_q + desc->num_p > KS_MAX_EXT) FAIL(NEO_EUNSUPPORTED, "num_q + num_p must be <= 64");
    if (desc->num_p > BC_MAX_IN) FAIL(NEO_EUNSUPPORTED, "num_p must be <= 16");
    int alpha = (desc->num_q + desc->dnum - 1) / desc->dnum;
    if ((desc->num_q + alpha - 1) / alpha != desc->dnum) FAIL(NEO_EINVAL, "every digit must be non-empty");
    if (alpha > BC_MAX_IN) FAIL(NEO_EUNSUPPORTED, "alpha must be <= 16");
    if (desc->dnum > KS_MAX_BETA) FAIL(NEO_EUNSUPPORTED, "dnum must be <= 12");
    if ((desc->q == nullptr) != (desc->p == nullptr)) FAIL(NEO_EINVAL, "give both q and p or neither");
    if (desc->alpha_t > 0 && desc->word_bits_t != 0 && desc->word_bits_t != desc->word_bits && desc->word_bits_t != 48)
        FAIL(NEO_EUNSUPPORTED, "word_bits_t must be 0, word_bits or 48");
    neo_ctx* c = new (std::nothrow) neo_ctx();
    if (!c) FAIL(NEO_ENOMEM, "host allocation failed");
    static std::atomic<unsigned long long> next_uid{0};
    c->uid = ++next_uid;
    std::string err;
    neo_status s;
    try {
        s = build_context(c, desc, err);
    } catch (...) {
        s = NEO_ENOMEM;
        err = "exception while building the context";
    }
    if (s != NEO_OK) {
        neo_params_destroy(c);
        FAIL(s, err);
    }
    if (cudaStreamCreateWithFlags(&c->side, cudaStreamNonBlocking) != cudaSuccess) c->side = nullptr;
    *out = c;
    return NEO_OK;
}

neo_status neo_params_destroy(neo_ctx* c) {
    if (!c) return NEO_OK;
    if (c->side) cudaStreamDestroy(c->side);
    if (c->d_tab) cudaFree(c->d_tab);
    if (c->d_ntt_tc) cudaFree(c->d_ntt_tc);
    if (c->d_mods) cudaFree(c->d_mods);
    if (c->d_bmat) cudaFree(c->d_bmat);
    if (c->d_rec) cudaFree(c->d_rec);
    delete c;
    return NEO_OK;
}

neo_status neo_ntt_select(neo_ctx* c, int32_t impl) {
    if (!c) FAIL(NEO_EINVAL, "null context");
    if (impl != NEO_NTT_FP64 && impl != NEO_NTT_TC) FAIL(NEO_EINVAL, "unknown NTT implementation");
    if (impl == NEO_NTT_TC && !c->ntt.tct) FAIL(NEO_EUNSUPPORTED, "tensor-core NTT needs N = 2^16 and 36-bit primes");
    c->ntt_impl = impl;
    return NEO_OK;
}

int32_t neo_ntt_selected(const neo_ctx* c) { return c ? c->ntt_impl : -1; }

neo_status neo_params_query(const neo_ctx* c, uint64_t* q, uint64_t* p, uint64_t* psi) {
    TRY(check_ctx(c));
    if (q) std::copy(c->mod.begin(), c->mod.begin() + c->num_q, q);
    if (p) std::copy(c->mod.begin() + c->num_q, c->mod.begin() + c->num_q + c->num_p, p);
    if (psi) std::copy(c->psi.begin(), c->psi.begin() + c->num_q + c->num_p, psi);
    return NEO_OK;
}

size_t neo_workspace_size(const neo_ctx* c, int32_t op, int32_t level, int32_t batch) {
    if (!c || batch <= 0 || level < 0 || level >= c->num_q) return 0;
    if ((op == NEO_OP_KEYSWITCH || op == NEO_OP_HMULT || op == NEO_OP_HROT || op == NEO_OP_HMULT_RESCALE) &&
        batch > batch_chunk())                           // these ops run large batches in chunks, two in flight
        return 2 * neo_workspace_size(c, op, level, batch_chunk());
    switch (op) {
        case NEO_OP_KEYSWITCH:
        case NEO_OP_HMULT:
        case NEO_OP_HROT:
        case NEO_OP_HROT_HOISTED:
        case NEO_OP_HROT_SUM:
        case NEO_OP_HMULT_RESCALE: {
            if (op == NEO_OP_HMULT_RESCALE && level < 1) return 0;
            size_t w = ks_layout(c, level, batch, op).total;
            if (c->num_t && op != NEO_OP_HROT_HOISTED && op != NEO_OP_HMULT_RESCALE && op != NEO_OP_HROT_SUM) w = std::max(w, klss_total(c, level, batch, op));
            return w * sizeof(u64);
        }
        case NEO_OP_RESCALE: return level >= 1 ? rescale_ws(c, level, batch) * sizeof(u64) : 0;
        case NEO_OP_DOUBLE_RESCALE: return level >= 2 ? ds_ws(c, level, batch) * sizeof(u64) : 0;
        case NEO_OP_MODRAISE: return (size_t)2 * batch * c->N * (2 + level) * sizeof(u64);
        default: return 0;
    }
}

static neo_status ntt_api(const neo_ctx* c, bool fwd, uint64_t* poly, const int32_t* ids, int32_t n, int32_t batch,
                          void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_ptr(poly, "poly"));
    if (!ids || n <= 0 || n > NEO_MAX_ROWS) FAIL(NEO_EINVAL, "need 1 <= n_limbs <= 160 limb ids");
    if (batch <= 0) FAIL(NEO_EINVAL, "batch must be positive");
    if ((long long)n * batch * batch >= (1ll << 32))      // the tile decode's 32-bit magic division
        FAIL(NEO_EUNSUPPORTED, "neo_ntt / neo_intt: n_limbs * batch^2 must be < 2^32");
    for (int k = 0; k < n; ++k)
        if (ids[k] < 0 || ids[k] >= c->limbs_total()) FAIL(NEO_EINVAL, "unknown limb id");
    size_t need = (size_t)batch * n * c->N * sizeof(u64);
    if (!ws || ws_bytes < need) FAIL(NEO_EINVAL, "ntt workspace must hold batch*n_limbs*N words");
    int off[NEO_MAX_ROWS];
    for (int k = 0; k < n; ++k) off[k] = k;
    long long bs = (long long)n * c->N;
    return ntt_rows(c, fwd, poly, bs, off, poly, bs, off, ids, n, static_cast<u64*>(ws), batch, S(st));
}

neo_status neo_ntt(const neo_ctx* c, uint64_t* poly, const int32_t* ids, int32_t n, int32_t batch, void* ws,
                      size_t ws_bytes, neo_stream_t st) {
    return ntt_api(c, true, poly, ids, n, batch, ws, ws_bytes, st);
}
neo_status neo_intt(const neo_ctx* c, uint64_t* poly, const int32_t* ids, int32_t n, int32_t batch, void* ws,
                       size_t ws_bytes, neo_stream_t st) {
    return ntt_api(c, false, poly, ids, n, batch, ws, ws_bytes, st);
}

neo_status neo_query_ql_inv(const neo_ctx* c, int32_t level, const int32_t* limb_ids, int32_t n, uint64_t* out) {
    TRY(check_ctx(c));
    if (level < 1 || level >= c->num_q) FAIL(NEO_EINVAL, "level out of range");
    if (n < 0 || (n > 0 && (!limb_ids || !out))) FAIL(NEO_EINVAL, "null argument");
    for (int k = 0; k < n; ++k) {
        if (limb_ids[k] < 0 || limb_ids[k] >= level) FAIL(NEO_EINVAL, "limb id outside [0, level)");
        out[k] = c->ql_inv[level][limb_ids[k]].w;
    }
    return NEO_OK;
}

neo_status neo_bconv(const neo_ctx* c, const uint64_t* in, const int32_t* in_ids, int32_t n_in, uint64_t* out,
                     const int32_t* out_ids, int32_t n_out, int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_ptr(in, "in"));
    TRY(check_ptr(out, "out"));
    if (!in_ids || !out_ids || n_in < 1 || n_in > BC_MAX_IN || n_out < 1 || n_out > BC_MAX_OUT)
        FAIL(NEO_EINVAL, "need 1 <= n_in <= 16 and 1 <= n_out <= 64");
    if (batch <= 0) FAIL(NEO_EINVAL, "batch must be positive");
    if (batch >= 4096) FAIL(NEO_EUNSUPPORTED, "neo_bconv: batch must be < 4096 (12-bit tile schedule field)");
    const int nl = c->num_q + c->num_p;
    for (int i = 0; i < n_in; ++i) {
        if (in_ids[i] < 0 || in_ids[i] >= nl) FAIL(NEO_EINVAL, "unknown input limb id");
        for (int k = 0; k < i; ++k)
            if (in_ids[k] == in_ids[i]) FAIL(NEO_EINVAL, "input limb ids must be distinct");
    }
    for (int j = 0; j < n_out; ++j)
        if (out_ids[j] < 0 || out_ids[j] >= nl) FAIL(NEO_EINVAL, "unknown output limb id");
    // constants of Algorithm 1 for this (in, out) pair, passed by value (no allocation); built
    // once per (context, in_ids, out_ids) and cached per thread (the limb-sharded path calls
    // this with the same id lists at every key-switch)
    struct BcEntry { BConvTab T; BConvTC P; BMatParam bp; };
    static thread_local std::map<std::vector<long long>, std::unique_ptr<BcEntry>> cache;
    std::vector<long long> key{(long long)c->uid, n_in, n_out};
    key.insert(key.end(), in_ids, in_ids + n_in);
    key.insert(key.end(), out_ids, out_ids + n_out);
    auto hit = cache.find(key);
    if (hit == cache.end()) {
        if (cache.size() > 512) cache.clear();
        std::unique_ptr<BcEntry> e(new BcEntry);
        BConvTab& T = e->T;
        std::memset(&T, 0, sizeof(T));
        T.n_in = n_in;
        T.n_out = n_out;
        auto mulm = [](u64 a, u64 b, u64 m) { return (u64)((u128)a * b % m); };
        auto powm = [&](u64 a, u64 x, u64 m) {
            u64 r = 1;
            for (a %= m; x; x >>= 1, a = mulm(a, a, m))
                if (x & 1) r = mulm(r, a, m);
            return r;
        };
        for (int i = 0; i < n_in; ++i) {
            u64 qi = c->mod[in_ids[i]], qh = 1;
            for (int k = 0; k < n_in; ++k)
                if (k != i) qh = mulm(qh, c->mod[in_ids[k]] % qi, qi);
            u64 inv = powm(qh, qi - 2, qi);
            T.qin[i] = qi;
            T.qhat_inv[i] = TW{inv, (u64)(((u128)inv << 64) / qi)};
        }
        for (int j = 0; j < n_out; ++j) {
            u64 t = c->mod[out_ids[j]];
            T.tmod[j] = ModQ{t, (u64)(((u128)1 << 98) / t), (double)t, 1.0 / (double)t};
            for (int i = 0; i < n_in; ++i) {
                u64 f = 1;
                for (int k = 0; k < n_in; ++k)
                    if (k != i) f = mulm(f, c->mod[in_ids[k]] % t, t);
                T.f_lo[i][j] = (unsigned)(f & 0x3FFFF);
                T.f_hi[i][j] = (unsigned)(f >> 18);
            }
        }

        if (c->use_tc && n_in <= BCTC_MAX_IN && n_out <= BCTC_MAX_OUT) {
            std::vector<u64> sm, tm;
            for (int i = 0; i < n_in; ++i) sm.push_back(c->mod[in_ids[i]]);
            for (int j = 0; j < n_out; ++j) tm.push_back(c->mod[out_ids[j]]);
            std::vector<uint8_t> bm;
            make_bconv_tc(sm, tm, e->P, bm);
            std::memset(&e->bp, 0, sizeof(e->bp));
            std::memcpy(&e->bp, bm.data(), bm.size());
        }
        hit = cache.emplace(key, std::move(e)).first;
    }
    const BcEntry& E = *hit->second;
    BConvIO io;
    io.in = in; io.out = out;
    io.in_bstride = (long long)n_in * c->N;
    io.out_bstride = (long long)n_out * c->N;
    for (int i = 0; i < n_in; ++i) io.in_off[i] = i;
    for (int j = 0; j < n_out; ++j) io.out_off[j] = j;
    if (c->use_tc && n_in <= BCTC_MAX_IN && n_out <= BCTC_MAX_OUT) {
        LAUNCH(PK_BCONV, S(st), launch_bconv_tc_param(E.P, io, E.bp, c->N, batch, c->num_sms, S(st)));
    } else {
        LAUNCH(PK_BCONV, S(st), launch_bconv(E.T, io, c->N, batch, S(st)));
    }
    return NEO_OK;
}

neo_status neo_tensor(const neo_ctx* c, const uint64_t* a, const uint64_t* b, int32_t level, uint64_t* d,
                      int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    TRY(check_ptr(a, "ct_a"));
    TRY(check_ptr(b, "ct_b"));
    TRY(check_ptr(d, "d"));
    LAUNCH(PK_TENSOR, S(st), launch_tensor(a, b, d, c->d_mods, level + 1, c->N, batch, S(st)));
    return NEO_OK;
}

neo_status neo_automorphism(const neo_ctx* c, const uint64_t* in, int32_t n_limbs, uint32_t g, uint64_t* out,
                            int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_ptr(in, "in"));
    TRY(check_ptr(out, "out"));
    if (n_limbs <= 0 || batch <= 0) FAIL(NEO_EINVAL, "n_limbs and batch must be positive");
    if ((g & 1) == 0 || g >= 2u * (unsigned)c->N) FAIL(NEO_EINVAL, "galois element must be odd and < 2N");
    LAUNCH(PK_AUTO, S(st), launch_automorph(in, out, g, c->N, n_limbs * batch, S(st)));
    return NEO_OK;
}

static neo_status evk_create(const neo_ctx* c, const uint64_t* evk, uint32_t galois, neo_evk** out) {
    TRY(check_ctx(c));
    if (!evk || !out) FAIL(NEO_EINVAL, "null argument");
    *out = nullptr;
    neo_evk* k = new (std::nothrow) neo_evk();
    if (!k) FAIL(NEO_ENOMEM, "host allocation failed");
    k->ctx = c;
    k->galois = galois;
    const size_t n = (size_t)c->dnum * 2 * (c->num_q + c->num_p) * c->N;
    if (cudaMalloc(&k->lo, n * sizeof(uint32_t)) != cudaSuccess || cudaMalloc(&k->hi, n) != cudaSuccess) {
        neo_evk_destroy(k);
        FAIL(NEO_ENOMEM, "cudaMalloc of the evaluation key failed");
    }
    // the key may have been written on any of the caller's streams (e.g. a non-blocking torch
    // stream, which the legacy stream does not wait for): finish all device work first
    cudaError_t e = cudaDeviceSynchronize();
    const u64* src = evk;
    u64* perm = nullptr;
    if (e == cudaSuccess && galois) {                          // sigma_{g^-1} of every key polynomial (NTT-domain gather)
        const u64 two_n = 2ull * c->N;
        u64 ginv = 1, b = galois, ex = c->N - 1;            // g^-1 = g^(N-1) mod 2N (odd g)
        for (; ex; ex >>= 1, b = b * b % two_n)
            if (ex & 1) ginv = ginv * b % two_n;
        e = cudaMalloc(&perm, n * sizeof(u64));
        if (e == cudaSuccess) e = launch_automorph(evk, perm, (unsigned)ginv, c->N, (int)(n / c->N), nullptr);
        src = perm;
    }
    if (e == cudaSuccess) e = launch_pack5(src, k->lo, k->hi, n, nullptr);   // 5 bytes per residue
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (perm) cudaFree(perm);
    if (e != cudaSuccess) {
        neo_evk_destroy(k);
        FAIL(NEO_ECUDA, std::string("evk re-layout failed: ") + cudaGetErrorString(e));
    }
    *out = k;
    return NEO_OK;
}

neo_status neo_evk_create(const neo_ctx* c, const uint64_t* evk, neo_evk** out) { return evk_create(c, evk, 0, out); }

neo_status neo_evk_create_klss(const neo_ctx* c, const uint64_t* ekey, neo_evk** out) {
    TRY(check_ctx(c));
    if (!c->num_t) FAIL(NEO_EINVAL, "context has no KLSS T primes (create it with alpha_t > 0)");
    if (!ekey || !out) FAIL(NEO_EINVAL, "null argument");
    *out = nullptr;
    neo_evk* k = new (std::nothrow) neo_evk();
    if (!k) FAIL(NEO_ENOMEM, "host allocation failed");
    k->ctx = c;
    k->klss = 1;
    const size_t n = (size_t)2 * c->klss_groups.size() * c->dnum * c->num_t * c->N;
    k->hi_bytes = c->word_bits_t > 40 ? 2 : 1;             // 48-bit T residues: 6 bytes per key word
    if (cudaMalloc(&k->lo, n * sizeof(uint32_t)) != cudaSuccess || cudaMalloc(&k->hi, n * k->hi_bytes) != cudaSuccess) {
        neo_evk_destroy(k);
        FAIL(NEO_ENOMEM, "cudaMalloc of the KLSS key failed");
    }
    // the key may have been written on any of the caller's streams (e.g. a non-blocking torch
    // stream, which the legacy stream does not wait for): finish all device work first
    cudaError_t e = cudaDeviceSynchronize();
    if (e == cudaSuccess)
        e = k->hi_bytes == 2 ? launch_pack6(ekey, k->lo, reinterpret_cast<uint16_t*>(k->hi), n, nullptr)
                             : launch_pack5(ekey, k->lo, k->hi, n, nullptr);
    if (e == cudaSuccess) e = cudaDeviceSynchronize();
    if (e != cudaSuccess) {
        neo_evk_destroy(k);
        FAIL(NEO_ECUDA, std::string("KLSS key re-layout failed: ") + cudaGetErrorString(e));
    }
    *out = k;
    return NEO_OK;
}

neo_status neo_klss_query(const neo_ctx* c, int32_t* alpha_t, int32_t* alpha_p, uint64_t* t) {
    TRY(check_ctx(c));
    if (alpha_t) *alpha_t = c->alpha_t;
    if (alpha_p) *alpha_p = c->num_t;
    if (t) std::copy(c->mod.begin() + c->num_q + c->num_p, c->mod.end(), t);
    return NEO_OK;
}

neo_status neo_evk_create_hoisted(const neo_ctx* c, const uint64_t* evk, uint32_t galois_elt, neo_evk** out) {
    TRY(check_ctx(c));
    if ((galois_elt & 1) == 0 || galois_elt >= 2u * (unsigned)c->N) FAIL(NEO_EINVAL, "galois element must be odd and < 2N");
    return evk_create(c, evk, galois_elt, out);
}

neo_status neo_evk_destroy(neo_evk* k) {
    if (!k) return NEO_OK;
    if (k->lo) cudaFree(k->lo);
    if (k->hi) cudaFree(k->hi);
    delete k;
    return NEO_OK;
}

// Large batches run as chunks of <= NEO_BATCH_CHUNK ciphertexts (default 32): the per-KS NTT
// intermediates of a chunk stay L2-resident (B200's 126 MB L2), which measured faster than one
// launch set over the whole batch (HROTATE at Set-B: 5250/s at B = 32 vs 4920/s at B = 256),
// and the workspace shrinks to the chunk's.  The key is re-read once per chunk (0.5 % more bytes).
static inline neo_stream_t NS(cudaStream_t s) { return reinterpret_cast<neo_stream_t>(s); }
#define CHUNKED(op, call_with_b0_nb_wk_bk_sk)                                                     \
    do {                                                                                         \
        if (batch > batch_chunk()) {                                                             \
            const size_t cw_ = neo_workspace_size(c, op, level, batch_chunk());                   \
            return run_chunked(c, batch, ws, ws_bytes, cw_, S(st),                               \
                               [&](int b0, int nb, void* wk, size_t bk, cudaStream_t sk) {       \
                                   return call_with_b0_nb_wk_bk_sk;                              \
                               });                                                               \
        }                                                                                        \
    } while (0)

neo_status neo_keyswitch(const neo_ctx* c, const neo_evk* k, const uint64_t* d, int32_t level, uint64_t* out0,
                         uint64_t* out1, int32_t batch, void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (!k || k->ctx != c) FAIL(NEO_EINVAL, "evaluation key missing or from another context");
    TRY(check_level(c, level, batch));
    TRY(check_ptr(d, "d"));
    TRY(check_ptr(out0, "out0"));
    TRY(check_ptr(out1, "out1"));
    TRY(check_ws(c, NEO_OP_KEYSWITCH, level, batch, ws, ws_bytes));
    {
        const size_t ls_ = (size_t)(level + 1) * c->N;
        CHUNKED(NEO_OP_KEYSWITCH,
                neo_keyswitch(c, k, d + b0 * ls_, level, out0 + b0 * ls_, out1 + b0 * ls_, nb, wk, bk, NS(sk)));
    }
    if (k->klss && !c->num_t) FAIL(NEO_EINVAL, "KLSS key on a context without T primes");
    KsLayout Ly = ks_layout(c, level, batch, NEO_OP_KEYSWITCH);
    const long long ls = (long long)(level + 1) * c->N;
    return ks_core(c, k, d, ls, level, batch, static_cast<u64*>(ws), Ly, out0, out1, ls, nullptr, nullptr, 0, S(st));
}

neo_status neo_hmult(const neo_ctx* c, const neo_evk* relin, const uint64_t* ct_a, const uint64_t* ct_b, int32_t level,
                     uint64_t* ct_out, int32_t batch, void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (!relin || relin->ctx != c) FAIL(NEO_EINVAL, "relinearisation key missing or from another context");
    TRY(check_level(c, level, batch));
    TRY(check_ptr(ct_a, "ct_a"));
    TRY(check_ptr(ct_b, "ct_b"));
    TRY(check_ptr(ct_out, "ct_out"));
    TRY(check_ws(c, NEO_OP_HMULT, level, batch, ws, ws_bytes));
    if (relin->klss && !c->num_t) FAIL(NEO_EINVAL, "KLSS key on a context without T primes");
    {
        const size_t cs_ = (size_t)2 * (level + 1) * c->N;
        CHUNKED(NEO_OP_HMULT,
                neo_hmult(c, relin, ct_a + b0 * cs_, ct_b + b0 * cs_, level, ct_out + b0 * cs_, nb, wk, bk, NS(sk)));
    }
    KsLayout Ly = ks_layout(c, level, batch, NEO_OP_HMULT);
    u64* w = static_cast<u64*>(ws);
    u64* dd = w + extra_offset(c, relin, level, batch, NEO_OP_HMULT);
    const long long ls = (long long)(level + 1) * c->N;
    cudaStream_t s = S(st);
    LAUNCH(PK_TENSOR, s, launch_tensor(ct_a, ct_b, dd, c->d_mods, level + 1, c->N, batch, s));
    return ks_core(c, relin, dd + 2 * ls, 3 * ls, level, batch, w, Ly, ct_out, ct_out + ls, 2 * ls, dd, dd + ls,
                   3 * ls, s);
}

neo_status neo_hmult_rescale(const neo_ctx* c, const neo_evk* relin, const uint64_t* ct_a, const uint64_t* ct_b,
                             int32_t level, uint64_t* ct_out, int32_t batch, void* ws, size_t ws_bytes,
                             neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (!relin || relin->ctx != c) FAIL(NEO_EINVAL, "relinearisation key missing or from another context");
    if (relin->klss) FAIL(NEO_EUNSUPPORTED, "neo_hmult_rescale takes a Hybrid key (use neo_hmult + neo_rescale)");
    TRY(check_level(c, level, batch));
    if (level < 1) FAIL(NEO_EINVAL, "rescale needs level >= 1");
    if (level > 64) FAIL(NEO_EUNSUPPORTED, "level > 64");
    TRY(check_ptr(ct_a, "ct_a"));
    TRY(check_ptr(ct_b, "ct_b"));
    TRY(check_ptr(ct_out, "ct_out"));
    TRY(check_ws(c, NEO_OP_HMULT_RESCALE, level, batch, ws, ws_bytes));
    {
        const size_t cs_ = (size_t)2 * (level + 1) * c->N, co_ = (size_t)2 * level * c->N;
        CHUNKED(NEO_OP_HMULT_RESCALE, neo_hmult_rescale(c, relin, ct_a + b0 * cs_, ct_b + b0 * cs_, level,
                                                        ct_out + b0 * co_, nb, wk, bk, NS(sk)));
    }
    KsLayout Ly = ks_layout(c, level, batch, NEO_OP_HMULT_RESCALE);
    u64* w = static_cast<u64*>(ws);
    u64* dd = w + Ly.extra;
    u64* last = dd + (size_t)3 * batch * (level + 1) * c->N;
    const long long ls = (long long)(level + 1) * c->N, lo = (long long)level * c->N;
    cudaStream_t s = S(st);
    LAUNCH(PK_TENSOR, s, launch_tensor(ct_a, ct_b, dd, c->d_mods, level + 1, c->N, batch, s));
    const bool fused = kip_ok(c, level);
    TRY(ks_modup(c, dd + 2 * ls, 3 * ls, level, batch, w, Ly, s, 0, fused));
    return ks_finish(c, relin, dd + 2 * ls, 3 * ls, level, batch, w, Ly, ct_out, ct_out + lo, 2 * lo, dd, dd + ls,
                     3 * ls, s, 0, true, last, 0, fused);
}

neo_status neo_hrot(const neo_ctx* c, const neo_evk* rk, uint32_t g, const uint64_t* ct_in, int32_t level,
                    uint64_t* ct_out, int32_t batch, void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (!rk || rk->ctx != c) FAIL(NEO_EINVAL, "rotation key missing or from another context");
    TRY(check_level(c, level, batch));
    TRY(check_ptr(ct_in, "ct_in"));
    TRY(check_ptr(ct_out, "ct_out"));
    if ((g & 1) == 0 || g >= 2u * (unsigned)c->N) FAIL(NEO_EINVAL, "galois element must be odd and < 2N");
    TRY(check_ws(c, NEO_OP_HROT, level, batch, ws, ws_bytes));
    if (rk->klss && !c->num_t) FAIL(NEO_EINVAL, "KLSS key on a context without T primes");
    {
        const size_t cs_ = (size_t)2 * (level + 1) * c->N;
        CHUNKED(NEO_OP_HROT, neo_hrot(c, rk, g, ct_in + b0 * cs_, level, ct_out + b0 * cs_, nb, wk, bk, NS(sk)));
    }
    KsLayout Ly = ks_layout(c, level, batch, NEO_OP_HROT);
    u64* w = static_cast<u64*>(ws);
    u64* sc0 = w + extra_offset(c, rk, level, batch, NEO_OP_HROT);   // [B][l+1][N]: sigma_g(c0)
    const long long ls = (long long)(level + 1) * c->N;
    cudaStream_t s = S(st);
    // AUTO on c1 is fused into its consumers: the INTT's row pass and KeyIP
    // read sigma_g(c1) through the index map.  sigma_g(c0) is permuted by its own (streaming)
    // launch up front: the ModDown tail then reads it with 16-byte loads instead of 8-byte
    // gathers, which measured faster when HROTATE overlaps another key-switch
    LAUNCH(PK_AUTO, s, launch_automorph(ct_in, sc0, g, c->N, level + 1, s, batch, 2 * ls, ls));
    return ks_core(c, rk, ct_in + ls, 2 * ls, level, batch, w, Ly, ct_out, ct_out + ls, 2 * ls, sc0, nullptr,
                   ls, s, g, /*add_galois=*/false);
}

neo_status neo_hrot_sum(const neo_ctx* c, const neo_evk* const* keys, const uint32_t* galois, int32_t n,
                        const uint64_t* const* cts, int32_t level, uint64_t* ct_out, int32_t batch, void* ws,
                        size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    TRY(check_ptr(ct_out, "ct_out"));
    if (!keys || !galois || !cts || n < 1 || n > 64) FAIL(NEO_EINVAL, "need 1 <= n <= 64 keys, Galois elements, ciphertexts");
    for (int k = 0; k < n; ++k) {
        if (!keys[k] || keys[k]->ctx != c || keys[k]->klss || keys[k]->galois)
            FAIL(NEO_EINVAL, "keys must be Hybrid rotation keys from neo_evk_create on this context");
        if ((galois[k] & 1) == 0 || galois[k] >= 2u * (unsigned)c->N) FAIL(NEO_EINVAL, "galois element must be odd and < 2N");
        TRY(check_ptr(cts[k], "cts[k]"));
        if (cts[k] == ct_out) FAIL(NEO_EINVAL, "ct_out must not alias an input");
    }
    TRY(check_ws(c, NEO_OP_HROT_SUM, level, batch, ws, ws_bytes));
    KsLayout Ly = ks_layout(c, level, batch, NEO_OP_HROT_SUM);
    u64* w = static_cast<u64*>(ws);
    const long long ls = (long long)(level + 1) * c->N;
    u64* c0sum = w + Ly.extra;                                 // [B][l+1][N]: sum_k sigma_g(c0_k)
    u64* c0k = c0sum + (size_t)batch * ls;                     // [B][l+1][N]: sigma_g(c0_k)
    cudaStream_t s = S(st);
    int launches = 0;
    // two streams: the ModUps of odd k run on the context's side stream into a second ModUp area,
    // overlapping the main stream's KeyIP of k - 1 and ModUp of k + 1; the KeyIPs accumulate in
    // order on the main stream (each after its ModUp's event)
    static thread_local cudaEvent_t ev_f = nullptr, ev_mu = nullptr, ev_kd = nullptr, ev_j = nullptr;
    if (!ev_f) {
        for (cudaEvent_t* e : {&ev_f, &ev_mu, &ev_kd, &ev_j}) cudaEventCreateWithFlags(e, cudaEventDisableTiming);
    }
    const bool fused = kip_ok(c, level);
    const bool two = n > 1 && !fused && two_stream_ok(c);
    const KsLayout Ly2 = Ly.area2();
    if (two) {
        CK(cudaEventRecord(ev_f, s));
        CK(cudaStreamWaitEvent(c->side, ev_f, 0));
    }
    auto join = [&]() {
        if (two) {
            const std::string msg = g_err;
            cudaEventRecord(ev_j, c->side);
            cudaStreamWaitEvent(s, ev_j, 0);
            g_err = msg;
        }
    };
    for (int k = 0; k < n; ++k) {
        // KeyIP(ModUp(sigma_g(c1_k))) accumulated in PQ_l; sigma_g(c1) read through the index map
        const bool alt = two && (k & 1);
        const KsLayout& Lk = alt ? Ly2 : Ly;
        if (alt) {
            if (k >= 2 && cudaStreamWaitEvent(c->side, ev_kd, 0) != cudaSuccess) { join(); FAIL(NEO_ECUDA, "event wait"); }
            neo_status r = ks_modup(c, cts[k] + ls, 2 * ls, level, batch, w, Lk, c->side, galois[k], fused);
            if (r == NEO_OK && (cudaEventRecord(ev_mu, c->side) != cudaSuccess || cudaStreamWaitEvent(s, ev_mu, 0) != cudaSuccess))
                r = NEO_ECUDA;
            if (r != NEO_OK) { join(); return r; }
        } else {
            const neo_status r = ks_modup(c, cts[k] + ls, 2 * ls, level, batch, w, Lk, s, galois[k], fused);
            if (r != NEO_OK) { join(); return r; }
        }
        launches += g_launches;
        {
            const neo_status r = ks_finish(c, keys[k], cts[k] + ls, 2 * ls, level, batch, w, Lk, nullptr, nullptr, 0,
                                           nullptr, nullptr, 0, s, galois[k], false, nullptr, k == 0 ? 1 : 2, fused);
            if (r != NEO_OK) { join(); return r; }
        }
        if (alt && cudaEventRecord(ev_kd, s) != cudaSuccess) { join(); FAIL(NEO_ECUDA, "event record"); }
        launches += g_launches;
        g_launches = 0;
        LAUNCH(PK_AUTO, s, launch_automorph(cts[k], k == 0 ? c0sum : c0k, galois[k], c->N, level + 1, s, batch,
                                           2 * ls, ls));
        if (k > 0) LAUNCH(PK_EW, s, launch_add_rows(c0sum, c0k, c0sum, c->d_mods, level + 1, c->N, batch, s));
        launches += g_launches;
        g_launches = 0;
    }
    join();
    // one ModDown of the summed acc, with the summed sigma_g(c0) added to component 0
    TRY(ks_finish(c, keys[0], nullptr, 0, level, batch, w, Ly, ct_out, ct_out + ls, 2 * ls, c0sum, nullptr, ls, s,
                  0, false, nullptr, 3));
    g_launches += launches;
    return NEO_OK;
}

neo_status neo_hrot_hoisted(const neo_ctx* c, const neo_evk* const* keys, int32_t n_rot, const uint64_t* ct_in,
                            int32_t level, uint64_t* ct_out, int32_t batch, void* ws, size_t ws_bytes,
                            neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    TRY(check_ptr(ct_in, "ct_in"));
    TRY(check_ptr(ct_out, "ct_out"));
    if (!keys || n_rot < 1) FAIL(NEO_EINVAL, "need n_rot >= 1 hoisted rotation keys");
    for (int r = 0; r < n_rot; ++r)
        if (!keys[r] || keys[r]->ctx != c || keys[r]->galois == 0 || keys[r]->klss)
            FAIL(NEO_EINVAL, "keys must come from neo_evk_create_hoisted on this context");
    TRY(check_ws(c, NEO_OP_HROT_HOISTED, level, batch, ws, ws_bytes));
    KsLayout Ly = ks_layout(c, level, batch, NEO_OP_HROT_HOISTED);
    u64* w = static_cast<u64*>(ws);
    u64* pre = w + Ly.extra;                                  // [B][2][l+1][N] before the automorphism
    const long long ls = (long long)(level + 1) * c->N;
    cudaStream_t s = S(st);
    // one ModUp of c1 for all rotations (hoisting): sigma_g(KS'(c1)) with KS' under sigma_g^-1(key)
    TRY(ks_modup(c, ct_in + ls, 2 * ls, level, batch, w, Ly, s));
    // the rotations' KeyIP + ModDown are independent: odd ones on the context's side stream with
    // their own ModDown area (latency-bound small launches at B = 1 overlap); fork / join by events
    static thread_local cudaEvent_t ev_f = nullptr, ev_j = nullptr;
    if (!ev_f) {
        cudaEventCreateWithFlags(&ev_f, cudaEventDisableTiming);
        cudaEventCreateWithFlags(&ev_j, cudaEventDisableTiming);
    }
    const bool two = n_rot > 1 && two_stream_ok(c);
    const KsLayout Ly2 = Ly.area2();
    u64* pre2 = w + Ly.extra2;
    if (two) {
        CK(cudaEventRecord(ev_f, s));
        CK(cudaStreamWaitEvent(c->side, ev_f, 0));
    }
    int launches = g_launches;
    neo_status res = NEO_OK;
    for (int r = 0; r < n_rot && res == NEO_OK; ++r) {
        const bool alt = two && (r & 1);
        cudaStream_t sr = alt ? c->side : s;
        u64* pr = alt ? pre2 : pre;
        g_launches = 0;
        res = ks_finish(c, keys[r], ct_in + ls, 2 * ls, level, batch, w, alt ? Ly2 : Ly, pr, pr + ls, 2 * ls, ct_in,
                        nullptr, 2 * ls, sr);
        launches += g_launches;
        if (res != NEO_OK) break;
        u64* dst = ct_out + (size_t)r * batch * 2 * ls;
        g_launches = 0;
        res = [&]() -> neo_status {
            LAUNCH(PK_AUTO, sr, launch_automorph(pr, dst, keys[r]->galois, c->N, 2 * (level + 1) * batch, sr));
            return NEO_OK;
        }();
        launches += g_launches;
    }
    if (two) {                                 // join (also on error: keeps a graph capture valid)
        const std::string msg = g_err;
        cudaEventRecord(ev_j, c->side);
        cudaStreamWaitEvent(s, ev_j, 0);
        g_err = msg;
    }
    g_launches = launches;
    return res;
}

neo_status neo_keyip(const neo_ctx* c, const neo_evk* k, const uint64_t* dhat, const int32_t* limb_ids, int32_t n,
                     int32_t beta, uint64_t* acc, int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (!k || k->ctx != c || k->klss) FAIL(NEO_EINVAL, "Hybrid evaluation key missing or from another context");
    TRY(check_ptr(dhat, "dhat"));
    TRY(check_ptr(acc, "acc"));
    if (!limb_ids || n < 1 || n > KS_MAX_EXT) FAIL(NEO_EINVAL, "need 1 <= n_limbs <= 64 limb ids");
    if (beta < 1 || beta > c->dnum) FAIL(NEO_EINVAL, "beta must be in [1, dnum]");
    if (batch <= 0) FAIL(NEO_EINVAL, "batch must be positive");
    KeyIPArgs A;
    A.galois = 0;
    A.d = dhat; A.up = dhat; A.evk_lo = k->lo; A.evk_hi = k->hi; A.acc = acc; A.mods = c->d_mods;
    A.d_bstride = A.up_bstride = (long long)beta * n * c->N;
    A.acc_bstride = (long long)2 * n * c->N;
    A.acc_cstride = (long long)n * c->N;
    A.N = c->N; A.beta = beta; A.evk_limbs = c->num_q + c->num_p;
    for (int t = 0; t < n; ++t) {
        if (limb_ids[t] < 0 || limb_ids[t] >= c->num_q + c->num_p) FAIL(NEO_EINVAL, "unknown limb id");
        A.limb[t] = limb_ids[t];
        for (int j = 0; j < beta; ++j) { A.src_kind[j][t] = 1; A.src_off[j][t] = j * n + t; }
    }
    LAUNCH(PK_KEYIP, S(st), launch_keyip(A, n, batch, S(st)));
    return NEO_OK;
}

neo_status neo_moddown_combine(const neo_ctx* c, const uint64_t* acc, const uint64_t* conv, const int32_t* q_ids,
                               int32_t n, uint64_t* out, int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_ptr(acc, "acc"));
    TRY(check_ptr(conv, "conv"));
    TRY(check_ptr(out, "out"));
    if (!q_ids || n < 1 || n > 64) FAIL(NEO_EINVAL, "need 1 <= n <= 64 Q limb ids");
    if (batch <= 0) FAIL(NEO_EINVAL, "batch must be positive");
    CombineArgs A;
    A.acc = acc; A.conv = conv; A.add0 = nullptr; A.add1 = nullptr; A.out0 = out; A.out1 = out + (size_t)n * c->N;
    A.mods = c->d_mods;
    A.acc_bstride = (long long)2 * n * c->N;
    A.acc_cstride = (long long)n * c->N;
    A.conv_stride = (long long)n * c->N;
    A.add_bstride = 0;
    A.out_bstride = (long long)2 * n * c->N;
    A.N = c->N;
    for (int i = 0; i < n; ++i) {
        if (q_ids[i] < 0 || q_ids[i] >= c->num_q) FAIL(NEO_EINVAL, "q_ids must be Q limbs");
        A.pinv[i] = c->pinv[q_ids[i]];
        A.limb[i] = q_ids[i];
    }
    LAUNCH(PK_COMBINE, S(st), launch_combine(A, n, batch, S(st)));
    return NEO_OK;
}

neo_status neo_rescale(const neo_ctx* c, const uint64_t* ct_in, int32_t level, uint64_t* ct_out, int32_t batch,
                       void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    if (level < 1) FAIL(NEO_EINVAL, "rescale needs level >= 1");
    TRY(check_ptr(ct_in, "ct_in"));
    TRY(check_ptr(ct_out, "ct_out"));
    TRY(check_ws(c, NEO_OP_RESCALE, level, batch, ws, ws_bytes));
    const int N = c->N, l = level, B2 = 2 * batch;
    u64* w = static_cast<u64*>(ws);
    u64* last = w;                          // [2B][N]: INTT of c_l, canonical mod q_l
    u64* tmp = last + (size_t)B2 * N;       // NTT intermediate
    cudaStream_t s = S(st);
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    // 1. coefficient form of the last limb of both components
    so[0] = l; dof[0] = 0; pr[0] = l;
    TRY(ntt_rows(c, false, ct_in, (long long)(l + 1) * N, so, last, N, dof, pr, 1, tmp, B2, s));
    // 2. NTT_i of ([c_l]_{q_l} mod q_i) for every i < l: every row reads the same coefficients
    //    (< q_l < 2^36, a valid lazy representative mod q_i, so no mod-switch pass is needed),
    //    and the row pass's epilogue writes (c_i - that) * q_l^-1 mod q_i directly (L137, Z10)
    for (int i = 0; i < l; ++i) { so[i] = 0; dof[i] = i; pr[i] = i; }
    RowEpi ep;
    ep.acc = ct_in;
    ep.acc_b = (long long)2 * (l + 1) * N;
    ep.acc_c = (long long)(l + 1) * N;
    ep.add0 = ep.add1 = nullptr;
    ep.add_b = 0;
    ep.add_galois = 0;
    ep.out0 = ct_out;
    ep.out1 = ct_out + (size_t)l * N;
    ep.out_b = (long long)2 * l * N;
    for (int i = 0; i < l; ++i) ep.pinv[i] = c->ql_inv[l][i];
    TRY(ntt_rows(c, true, last, N, so, ct_out, (long long)l * N, dof, pr, l, tmp, B2, s, &ep));
    return NEO_OK;
}

static neo_status ew_api(const neo_ctx* c, int op, const uint64_t* a, const uint64_t* b, int32_t level, uint64_t* out,
                         int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    TRY(check_ptr(a, "ct_in"));
    TRY(check_ptr(b, op == EW_HADD ? "ct_b" : "pt"));
    TRY(check_ptr(out, "ct_out"));
    EwArgs A;
    A.a = a; A.b = b; A.out = out; A.mods = c->d_mods;
    A.N = c->N; A.limbs = level + 1; A.op = op;
    LAUNCH(PK_EW, S(st), launch_ew(A, batch, S(st)));
    return NEO_OK;
}

neo_status neo_pmult(const neo_ctx* c, const uint64_t* ct_in, const uint64_t* pt, int32_t level, uint64_t* ct_out,
                     int32_t batch, neo_stream_t st) {
    return ew_api(c, EW_PMULT, ct_in, pt, level, ct_out, batch, st);
}
neo_status neo_hadd(const neo_ctx* c, const uint64_t* ct_a, const uint64_t* ct_b, int32_t level, uint64_t* ct_out,
                    int32_t batch, neo_stream_t st) {
    return ew_api(c, EW_HADD, ct_a, ct_b, level, ct_out, batch, st);
}
neo_status neo_padd(const neo_ctx* c, const uint64_t* ct_in, const uint64_t* pt, int32_t level, uint64_t* ct_out,
                    int32_t batch, neo_stream_t st) {
    return ew_api(c, EW_PADD, ct_in, pt, level, ct_out, batch, st);
}

neo_status neo_hsub(const neo_ctx* c, const uint64_t* ct_a, const uint64_t* ct_b, int32_t level, uint64_t* ct_out,
                    int32_t batch, neo_stream_t st) {
    return ew_api(c, EW_HSUB, ct_a, ct_b, level, ct_out, batch, st);
}

neo_status neo_ew_limbs(const neo_ctx* c, int32_t op, const uint64_t* a, const uint64_t* b, const int32_t* limb_ids,
                        int32_t n, const uint64_t* scal, int32_t src_limb, uint64_t* out, int32_t batch,
                        neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (op < EWL_HADD || op > EWL_LIFT) FAIL(NEO_EINVAL, "unknown neo_ew_limbs op");
    if (batch <= 0) FAIL(NEO_EINVAL, "batch must be positive");
    if (n < 1 || n > 64 || !limb_ids) FAIL(NEO_EINVAL, "need 1 <= n <= 64 limb ids");
    TRY(check_ptr(a, "a"));
    TRY(check_ptr(out, "out"));
    if (op != EWL_LIFT) TRY(check_ptr(b, "b"));
    const int tot = c->num_q + c->num_p;
    EwlArgs A;
    for (int k = 0; k < n; ++k) {
        if (limb_ids[k] < 0 || limb_ids[k] >= tot) FAIL(NEO_EINVAL, "unknown limb id");
        A.lid[k] = (short)limb_ids[k];
    }
    if (op == EWL_SUBMUL) {
        if (!scal) FAIL(NEO_EINVAL, "SUBMUL needs the host array scal[n]");
        for (int k = 0; k < n; ++k) {
            const u64 q = c->mod[limb_ids[k]];
            if (scal[k] >= q) FAIL(NEO_EINVAL, "scal[k] must be a residue mod q_{limb_ids[k]}");
            A.scal[k] = TW{scal[k], (u64)(((u128)scal[k] << 64) / q)};
        }
    }
    if (op == EWL_LIFT && (src_limb < 0 || src_limb >= tot)) FAIL(NEO_EINVAL, "bad src_limb");
    A.a = a; A.b = b; A.out = out; A.mods = c->d_mods;
    A.N = c->N; A.n = n; A.op = op; A.src = src_limb;
    LAUNCH(PK_EW, S(st), launch_ew_limbs(A, batch, S(st)));
    return NEO_OK;
}

size_t neo_wire_bytes(size_t n) { return 4 * n + n / 2; }

static neo_status wire_api(const neo_ctx* c, bool pack, const void* in, void* out, size_t n, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_ptr(in, "in"));
    TRY(check_ptr(out, "out"));
    if (c->word_bits > 36) FAIL(NEO_EUNSUPPORTED, "the 36-bit wire format needs word_bits <= 36");
    if (n == 0 || n % 8) FAIL(NEO_EINVAL, "n must be a positive multiple of 8");
    if (reinterpret_cast<uintptr_t>(pack ? out : in) % 16) FAIL(NEO_EINVAL, "wire buffer must be 16-byte aligned");
    LAUNCH(PK_EW, S(st), launch_wire(pack, in, out, n, S(st)));
    return NEO_OK;
}
neo_status neo_wire_pack(const neo_ctx* c, const uint64_t* in, void* wire, size_t n, neo_stream_t st) {
    return wire_api(c, true, in, wire, n, st);
}
neo_status neo_wire_unpack(const neo_ctx* c, const void* wire, uint64_t* out, size_t n, neo_stream_t st) {
    return wire_api(c, false, wire, out, n, st);
}

neo_status neo_pmult_acc(const neo_ctx* c, const uint64_t* const* cts, const uint64_t* const* pts, int32_t n_terms,
                        int32_t pt_shared, int32_t level, uint64_t* ct_out, int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    TRY(check_ptr(ct_out, "ct_out"));
    if (!cts || !pts) FAIL(NEO_EINVAL, "cts / pts arrays are null");
    if (n_terms < 1 || n_terms > NEO_MAX_ACC) FAIL(NEO_EINVAL, "n_terms must be in [1, 32]");
    PmaccArgs A;
    for (int k = 0; k < n_terms; ++k) {
        TRY(check_ptr(cts[k], "cts[k]"));
        TRY(check_ptr(pts[k], "pts[k]"));
        if (cts[k] == ct_out) FAIL(NEO_EINVAL, "ct_out must not alias an input ciphertext");
        A.ct[k] = cts[k];
        A.pt[k] = pts[k];
    }
    A.out = ct_out; A.mods = c->d_mods;
    A.N = c->N; A.limbs = level + 1; A.n_terms = n_terms; A.pt_shared = pt_shared != 0;
    LAUNCH(PK_EW, S(st), launch_pmult_acc(A, batch, S(st)));
    return NEO_OK;
}

neo_status neo_modraise(const neo_ctx* c, const uint64_t* ct_in, int32_t level, uint64_t* ct_out, int32_t batch,
                        void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    TRY(check_ptr(ct_in, "ct_in"));
    TRY(check_ptr(ct_out, "ct_out"));
    TRY(check_ws(c, NEO_OP_MODRAISE, level, batch, ws, ws_bytes));
    const int N = c->N, B2 = 2 * batch, Lq = level + 1;
    u64* w = static_cast<u64*>(ws);
    u64* coef = w;                                   // [2B][N]
    u64* tmp = coef + (size_t)B2 * N;                // NTT intermediate [2B][Lq][N]
    cudaStream_t s = S(st);
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    so[0] = 0; dof[0] = 0; pr[0] = 0;
    TRY(ntt_rows(c, false, ct_in, (long long)N, so, coef, (long long)N, dof, pr, 1, tmp, B2, s));
    LAUNCH(PK_MODSW, s, launch_modraise(coef, ct_out, c->d_mods, Lq, N, B2, s));
    for (int i = 0; i < Lq; ++i) { so[i] = dof[i] = pr[i] = i; }
    return ntt_rows(c, true, ct_out, (long long)Lq * N, so, ct_out, (long long)Lq * N, dof, pr, Lq, tmp, B2, s);
}

neo_status neo_drop_levels(const neo_ctx* c, const uint64_t* ct_in, int32_t level_in, uint64_t* ct_out,
                           int32_t level_out, int32_t batch, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level_in, batch));
    if (level_out < 0 || level_out > level_in) FAIL(NEO_EINVAL, "need 0 <= level_out <= level_in");
    TRY(check_ptr(ct_in, "ct_in"));
    TRY(check_ptr(ct_out, "ct_out"));
    LAUNCH(PK_EW, S(st), launch_drop(ct_in, ct_out, level_in + 1, level_out + 1, c->N, batch, S(st)));
    return NEO_OK;
}

neo_status neo_double_rescale(const neo_ctx* c, const uint64_t* ct_in, int32_t level, uint64_t* ct_out,
                              int32_t batch, void* ws, size_t ws_bytes, neo_stream_t st) {
    g_launches = 0;
    TRY(check_ctx(c));
    TRY(check_level(c, level, batch));
    if (level < 2) FAIL(NEO_EINVAL, "double rescale needs level >= 2");
    TRY(check_ptr(ct_in, "ct_in"));
    TRY(check_ptr(ct_out, "ct_out"));
    TRY(check_ws(c, NEO_OP_DOUBLE_RESCALE, level, batch, ws, ws_bytes));
    const int N = c->N, l = level, B2 = 2 * batch;
    u64* w = static_cast<u64*>(ws);
    u64* last2 = w;                                   // [2B][2][N] coefficient form of c_{l-1}, c_l
    u64* corr = last2 + (size_t)B2 * 2 * N;           // [2B][l-1][N]
    u64* tmp = corr + (size_t)B2 * (l - 1) * N;       // NTT intermediate
    cudaStream_t s = S(st);
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    // 1. coefficient form of the last two limbs of both components
    for (int k = 0; k < 2; ++k) { so[k] = l - 1 + k; dof[k] = k; pr[k] = l - 1 + k; }
    TRY(ntt_rows(c, false, ct_in, (long long)(l + 1) * N, so, last2, 2LL * N, dof, pr, 2, tmp, B2, s));
    // 2. the noise-reduction limbs [x mod q_{l-1} q_l]_{q_i}, i < l - 1 (Garner, exact)
    DsArgs D;
    D.last2 = last2; D.corr = corr; D.mods = c->d_mods; D.N = N; D.l = l;
    D.qlinv_m = c->ds_qlinv_m[l];
    for (int i = 0; i + 1 < l; ++i) D.ql[i] = c->ds_ql[l][i];
    LAUNCH(PK_MODSW, s, launch_ds_corr(D, B2, s));
    // 3. NTT of them; the row pass's epilogue writes (c_i - corr_i) (q_{l-1} q_l)^-1 mod q_i
    for (int i = 0; i + 1 < l; ++i) { so[i] = dof[i] = pr[i] = i; }
    RowEpi ep;
    ep.acc = ct_in;
    ep.acc_b = (long long)2 * (l + 1) * N;
    ep.acc_c = (long long)(l + 1) * N;
    ep.add0 = ep.add1 = nullptr;
    ep.add_b = 0;
    ep.add_galois = 0;
    ep.out0 = ct_out;
    ep.out1 = ct_out + (size_t)(l - 1) * N;
    ep.out_b = (long long)2 * (l - 1) * N;
    for (int i = 0; i + 1 < l; ++i) ep.pinv[i] = c->ds_inv[l][i];
    TRY(ntt_rows(c, true, corr, (long long)(l - 1) * N, so, ct_out, (long long)(l - 1) * N, dof, pr, l - 1, tmp, B2,
                 s, &ep));
    return NEO_OK;
}

}  // extern "C"

// ==================================================================== limb-sharded key-switch
// one key-switch split by RNS limb over `nranks` ranks, NCCL inside the
// library.  Ownership (round-robin, so every Rescale's dropped top limb rotates over the ranks):
// rank r owns the Q limbs i = r (mod nranks) of q_0..q_l and the P limbs p_k, k = r (mod nranks).
// Only BConv needs other ranks' limbs, so the path has two exchange steps, both all-gathers of
// coefficient-form limbs (Table 2, Fig. 5):
//   INTT(own Q, q^_i^-1 folded) -> ALL-GATHER per digit j -> ModUp BConv of digit j onto own
//   targets -> NTT  (digit j+1's gather runs on the communication stream meanwhile)
//   -> KeyIP (own limbs) -> INTT(own P, P^_k^-1 folded) -> ALL-GATHER P -> ModDown BConv onto own
//   Q -> NTT with the fused tail (acc - conv) P^-1.
// Gathers land directly in the BConv input layout ([digit][rank][B][rows][N]; BConv addresses a
// limb by its owner and local index), so nothing is padded, concatenated or copied around them.
// Transports: NCCL (ncclAllGather; libnccl.so.2 resolved with dlopen when the communicator is
// created, so the library has no link-time NCCL dependency), or an in-process group of ranks on
// one GPU (one host thread per rank; device-to-device copies after a host barrier) for tests.
#include <dlfcn.h>
#include <nccl.h>

#include <chrono>
#include <condition_variable>
#include <mutex>

namespace {
struct NcclApi {
    ncclResult_t (*GetUniqueId)(ncclUniqueId*) = nullptr;
    ncclResult_t (*CommInitRank)(ncclComm_t*, int, ncclUniqueId, int) = nullptr;
    ncclResult_t (*AllGather)(const void*, void*, size_t, ncclDataType_t, ncclComm_t, cudaStream_t) = nullptr;
    ncclResult_t (*CommDestroy)(ncclComm_t) = nullptr;
    const char* (*GetErrorString)(ncclResult_t) = nullptr;
    bool ok = false;
};
const NcclApi& nccl_api() {
    static NcclApi A = [] {
        NcclApi a;
        void* h = dlopen("libnccl.so.2", RTLD_NOW | RTLD_GLOBAL);
        if (!h) h = dlopen("libnccl.so", RTLD_NOW | RTLD_GLOBAL);
        if (!h) return a;
        a.GetUniqueId = reinterpret_cast<decltype(a.GetUniqueId)>(dlsym(h, "ncclGetUniqueId"));
        a.CommInitRank = reinterpret_cast<decltype(a.CommInitRank)>(dlsym(h, "ncclCommInitRank"));
        a.AllGather = reinterpret_cast<decltype(a.AllGather)>(dlsym(h, "ncclAllGather"));
        a.CommDestroy = reinterpret_cast<decltype(a.CommDestroy)>(dlsym(h, "ncclCommDestroy"));
        a.GetErrorString = reinterpret_cast<decltype(a.GetErrorString)>(dlsym(h, "ncclGetErrorString"));
        a.ok = a.GetUniqueId && a.CommInitRank && a.AllGather && a.CommDestroy && a.GetErrorString;
        return a;
    }();
    return A;
}

// in-process group: all-gather = publish (pointer + ready event), barrier, copy every peer's
// block on the rank's communication stream, barrier, wait for every peer's copies to finish
// reading this rank's block (so it may be overwritten by later work on its stream)
struct LocalGroup {
    int n;
    std::mutex m;
    std::condition_variable cv;
    int arrived = 0;
    long long gen = 0;
    std::vector<const void*> send;
    std::vector<cudaEvent_t> ready, done;
    int refs = 0;
    bool barrier() {                                   // false: a rank did not arrive within 120 s
        std::unique_lock<std::mutex> lk(m);
        const long long g = gen;
        if (++arrived == n) {
            arrived = 0;
            ++gen;
            cv.notify_all();
            return true;
        }
        return cv.wait_for(lk, std::chrono::seconds(120), [&] { return gen != g; });
    }
};
}  // namespace

struct neo_comm {
    const neo_ctx* ctx;
    int nranks, rank;
    ncclComm_t nccl = nullptr;
    LocalGroup* local = nullptr;
    cudaStream_t cs = nullptr;                         // communication stream
    cudaEvent_t ev_prod = nullptr, ev_p = nullptr;
    std::vector<cudaEvent_t> ev_gath;                // one per digit
    // per level l: BConv tables for this rank's targets
    std::vector<std::vector<neo::BConvTC>> up_tc;      // [l][j]: digit j -> mine \ D_j
    std::vector<std::vector<size_t>> up_off;
    std::vector<neo::BConvTC> down_tc;                 // [l]: P -> my Q limbs (empty if none)
    std::vector<size_t> down_off;
    uint8_t* d_bmat = nullptr;
};

namespace {
struct ShardGeo {                                      // this rank's limbs at level l
    int W, r, Lq, beta, alpha, P, maxd, maxp;
    std::vector<int> my_q, my_p, mine;                 // limb ids (mine = my_q then my_p)
    std::vector<std::vector<int>> dig_own;             // [j] my limbs of digit j
};
ShardGeo shard_geo(const neo_ctx* c, int W, int r, int l) {
    ShardGeo g;
    g.W = W; g.r = r; g.Lq = l + 1; g.beta = c->beta(l); g.alpha = c->alpha; g.P = c->num_p;
    g.maxd = (c->alpha + W - 1) / W;
    g.maxp = (c->num_p + W - 1) / W;
    for (int i = r; i < g.Lq; i += W) g.my_q.push_back(i);
    for (int k = r; k < g.P; k += W) g.my_p.push_back(c->num_q + k);
    g.mine = g.my_q;
    g.mine.insert(g.mine.end(), g.my_p.begin(), g.my_p.end());
    g.dig_own.resize(g.beta);
    for (int j = 0; j < g.beta; ++j)
        for (int i : c->digits[l][j])
            if (i % W == r) g.dig_own[j].push_back(i);
    return g;
}
struct ShardLayout {
    size_t ysend, yall, up, acc, psend, pall, conv, tmp, total;   // u64 offsets
};
ShardLayout shard_layout(const neo_ctx* c, const ShardGeo& g, int B) {
    const size_t N = c->N, nm = g.mine.size(), nq = g.my_q.size();
    ShardLayout L;
    size_t o = 0;
    L.ysend = o; o += (size_t)g.beta * B * g.maxd * N;
    L.yall = o; o += (size_t)g.beta * g.W * B * g.maxd * N;
    L.up = o; o += (size_t)B * g.beta * nm * N;
    L.acc = o; o += (size_t)B * 2 * nm * N;
    L.psend = o; o += (size_t)B * 2 * g.maxp * N;
    L.pall = o; o += (size_t)g.W * B * 2 * g.maxp * N;
    L.conv = o; o += (size_t)B * 2 * std::max<size_t>(nq, 1) * N;
    L.tmp = o; o += (size_t)B * std::max<size_t>(std::max<size_t>((size_t)g.beta * nm, 2 * nq), 2 * g.my_p.size() + 1) * N;
    L.total = o;
    return L;
}
}  // namespace

// all-gather of `bytes` per rank from send (this rank's block) into recv ([nranks][bytes]), on
// the communication stream, after the work recorded in ev_prod on `st`; completion is recorded
// in `done` (the compute stream waits on it before reading recv)
static neo_status comm_allgather(const neo_comm* cm, const void* send, void* recv, size_t bytes, cudaStream_t st,
                                 cudaEvent_t done) {
    CK(cudaEventRecord(cm->ev_prod, st));
    CK(cudaStreamWaitEvent(cm->cs, cm->ev_prod, 0));
    if (cm->nranks == 1) {
        if (recv != send) CK(cudaMemcpyAsync(recv, send, bytes, cudaMemcpyDeviceToDevice, cm->cs));
    } else if (cm->nccl) {
        ncclResult_t e = nccl_api().AllGather(send, recv, bytes, ncclUint8, cm->nccl, cm->cs);
        if (e != ncclSuccess) FAIL(NEO_ENCCL, std::string("ncclAllGather: ") + nccl_api().GetErrorString(e));
    } else {
        LocalGroup* G = cm->local;
        G->send[cm->rank] = send;
        CK(cudaEventRecord(G->ready[cm->rank], cm->cs));
        if (!G->barrier()) FAIL(NEO_ECUDA, "local group: a rank did not reach the exchange (barrier timeout)");
        for (int s = 0; s < G->n; ++s) {
            CK(cudaStreamWaitEvent(cm->cs, G->ready[s], 0));
            CK(cudaMemcpyAsync(static_cast<char*>(recv) + (size_t)s * bytes, G->send[s], bytes,
                               cudaMemcpyDeviceToDevice, cm->cs));
        }
        CK(cudaEventRecord(G->done[cm->rank], cm->cs));
        if (!G->barrier()) FAIL(NEO_ECUDA, "local group: a rank did not reach the exchange (barrier timeout)");
        for (int s = 0; s < G->n; ++s) CK(cudaStreamWaitEvent(cm->cs, G->done[s], 0));
    }
    CK(cudaEventRecord(done, cm->cs));
    return NEO_OK;
}

static neo_status comm_tables(neo_comm* cm) {
    const neo_ctx* c = cm->ctx;
    std::vector<uint8_t> all, bm;
    cm->up_tc.assign(c->num_q, {});
    cm->up_off.assign(c->num_q, {});
    cm->down_tc.assign(c->num_q, BConvTC{});
    cm->down_off.assign(c->num_q, 0);
    std::vector<u64> pm;
    for (int k = 0; k < c->num_p; ++k) pm.push_back(c->mod[c->num_q + k]);
    for (int l = 0; l < c->num_q; ++l) {
        ShardGeo g = shard_geo(c, cm->nranks, cm->rank, l);
        for (int j = 0; j < g.beta; ++j) {
            const std::vector<int>& dj = c->digits[l][j];
            std::vector<u64> sm, tm;
            for (int id : dj) sm.push_back(c->mod[id]);
            for (int t : g.mine)
                if (std::find(dj.begin(), dj.end(), t) == dj.end()) tm.push_back(c->mod[t]);
            BConvTC P;
            std::memset(&P, 0, sizeof(P));
            if (!tm.empty()) {
                if ((int)tm.size() > BCTC_MAX_OUT) FAIL(NEO_EUNSUPPORTED, "too many ModUp targets per rank");
                make_bconv_tc(sm, tm, P, bm);
                cm->up_off[l].push_back(all.size());
                all.insert(all.end(), bm.begin(), bm.end());
            } else {
                cm->up_off[l].push_back(0);
            }
            cm->up_tc[l].push_back(P);
        }
        if (!g.my_q.empty()) {
            std::vector<u64> qm;
            for (int i : g.my_q) qm.push_back(c->mod[i]);
            make_bconv_tc(pm, qm, cm->down_tc[l], bm);
            cm->down_off[l] = all.size();
            all.insert(all.end(), bm.begin(), bm.end());
        }
    }
    if (!all.empty()) {
        CK(cudaMalloc(&cm->d_bmat, all.size()));
        CK(cudaMemcpy(cm->d_bmat, all.data(), all.size(), cudaMemcpyHostToDevice));
    }
    return NEO_OK;
}

static neo_status comm_common(const neo_ctx* c, neo_comm* cm) {
    if (!c->use_tc) FAIL(NEO_EUNSUPPORTED, "the limb-sharded key-switch needs the tensor-core BConv tables");
    CK(cudaSetDevice(c->device));
    CK(cudaStreamCreateWithFlags(&cm->cs, cudaStreamNonBlocking));
    CK(cudaEventCreateWithFlags(&cm->ev_prod, cudaEventDisableTiming));
    CK(cudaEventCreateWithFlags(&cm->ev_p, cudaEventDisableTiming));
    cm->ev_gath.assign(c->dnum, nullptr);
    for (auto& e : cm->ev_gath) CK(cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    return comm_tables(cm);
}

extern "C" {

neo_status neo_comm_unique_id(uint8_t uid[128]) {
    if (!uid) FAIL(NEO_EINVAL, "null uid buffer");
    const NcclApi& A = nccl_api();
    if (!A.ok) FAIL(NEO_ENCCL, "libnccl.so.2 not found");
    ncclUniqueId id;
    ncclResult_t e = A.GetUniqueId(&id);
    if (e != ncclSuccess) FAIL(NEO_ENCCL, std::string("ncclGetUniqueId: ") + A.GetErrorString(e));
    static_assert(sizeof(ncclUniqueId) == 128, "ncclUniqueId is 128 bytes");
    std::memcpy(uid, &id, 128);
    return NEO_OK;
}

neo_status neo_comm_create(const neo_ctx* c, const uint8_t uid[128], int32_t nranks, int32_t rank, neo_comm** out) {
    TRY(check_ctx(c));
    if (!out || !uid) FAIL(NEO_EINVAL, "null argument");
    *out = nullptr;
    if (nranks < 1 || rank < 0 || rank >= nranks) FAIL(NEO_EINVAL, "need 0 <= rank < nranks");
    std::unique_ptr<neo_comm> cm(new (std::nothrow) neo_comm());
    if (!cm) FAIL(NEO_ENOMEM, "out of host memory");
    cm->ctx = c; cm->nranks = nranks; cm->rank = rank;
    TRY(comm_common(c, cm.get()));
    if (nranks > 1) {
        const NcclApi& A = nccl_api();
        if (!A.ok) FAIL(NEO_ENCCL, "libnccl.so.2 not found");
        ncclUniqueId id;
        std::memcpy(&id, uid, 128);
        ncclResult_t e = A.CommInitRank(&cm->nccl, nranks, id, rank);
        if (e != ncclSuccess) FAIL(NEO_ENCCL, std::string("ncclCommInitRank: ") + A.GetErrorString(e));
    }
    *out = cm.release();
    return NEO_OK;
}

neo_status neo_comm_create_local(const neo_ctx* c, int32_t nranks, neo_comm** comms) {
    TRY(check_ctx(c));
    if (!comms || nranks < 1 || nranks > 64) FAIL(NEO_EINVAL, "need 1 <= nranks <= 64 and an output array");
    LocalGroup* G = new (std::nothrow) LocalGroup();
    if (!G) FAIL(NEO_ENOMEM, "out of host memory");
    G->n = nranks;
    G->send.assign(nranks, nullptr);
    G->ready.assign(nranks, nullptr);
    G->done.assign(nranks, nullptr);
    for (int r = 0; r < nranks; ++r) {
        cudaEventCreateWithFlags(&G->ready[r], cudaEventDisableTiming);
        cudaEventCreateWithFlags(&G->done[r], cudaEventDisableTiming);
    }
    for (int r = 0; r < nranks; ++r) {
        comms[r] = nullptr;
        neo_comm* cm = new (std::nothrow) neo_comm();
        if (!cm) FAIL(NEO_ENOMEM, "out of host memory");
        cm->ctx = c; cm->nranks = nranks; cm->rank = r; cm->local = G;
        G->refs++;
        comms[r] = cm;
        neo_status s = comm_common(c, cm);
        if (s) return s;
    }
    return NEO_OK;
}

neo_status neo_comm_destroy(neo_comm* cm) {
    if (!cm) return NEO_OK;
    if (cm->nccl) nccl_api().CommDestroy(cm->nccl);
    if (cm->cs) cudaStreamDestroy(cm->cs);
    if (cm->ev_prod) cudaEventDestroy(cm->ev_prod);
    if (cm->ev_p) cudaEventDestroy(cm->ev_p);
    for (auto e : cm->ev_gath)
        if (e) cudaEventDestroy(e);
    if (cm->d_bmat) cudaFree(cm->d_bmat);
    if (cm->local && --cm->local->refs == 0) {
        for (auto e : cm->local->ready) cudaEventDestroy(e);
        for (auto e : cm->local->done) cudaEventDestroy(e);
        delete cm->local;
    }
    delete cm;
    return NEO_OK;
}

int32_t neo_comm_limbs(const neo_comm* cm, int32_t level, int32_t* q_ids, int32_t* p_ids, int32_t* n_p) {
    if (!cm || level < 0 || level >= cm->ctx->num_q) return -1;
    ShardGeo g = shard_geo(cm->ctx, cm->nranks, cm->rank, level);
    if (q_ids) for (size_t i = 0; i < g.my_q.size(); ++i) q_ids[i] = g.my_q[i];
    if (p_ids) for (size_t i = 0; i < g.my_p.size(); ++i) p_ids[i] = g.my_p[i];
    if (n_p) *n_p = (int32_t)g.my_p.size();
    return (int32_t)g.my_q.size();
}

size_t neo_workspace_size_sharded(const neo_comm* cm, int32_t level, int32_t batch) {
    if (!cm || level < 0 || level >= cm->ctx->num_q || batch <= 0) return 0;
    ShardGeo g = shard_geo(cm->ctx, cm->nranks, cm->rank, level);
    return shard_layout(cm->ctx, g, batch).total * sizeof(u64);
}

neo_status neo_keyswitch_sharded(const neo_ctx* c, const neo_comm* cm, const neo_evk* k, const uint64_t* d_local,
                                 int32_t level, uint64_t* out0, uint64_t* out1, int32_t batch, void* ws,
                                 size_t ws_bytes, neo_stream_t stream) {
    g_launches = 0;
    TRY(check_ctx(c));
    if (!cm || cm->ctx != c) FAIL(NEO_EINVAL, "communicator missing or from another context");
    if (!k || k->ctx != c || k->klss || k->galois) FAIL(NEO_EINVAL, "Hybrid evaluation key missing or from another context");
    if (level < 0 || level >= c->num_q) FAIL(NEO_EINVAL, "level out of range");
    if (batch <= 0 || batch > 32) FAIL(NEO_EINVAL, "batch must be in [1, 32]");
    const int l = level, B = batch, N = c->N;
    ShardGeo g = shard_geo(c, cm->nranks, cm->rank, l);
    const int nq = (int)g.my_q.size(), nm = (int)g.mine.size(), np = (int)g.my_p.size();
    if (nq > 0) { TRY(check_ptr(d_local, "d_local")); TRY(check_ptr(out0, "out0")); TRY(check_ptr(out1, "out1")); }
    ShardLayout Ly = shard_layout(c, g, B);
    if (!ws || ws_bytes < Ly.total * sizeof(u64)) FAIL(NEO_EINVAL, "workspace smaller than neo_workspace_size_sharded");
    cudaStream_t st = S(stream);
    u64* W64 = static_cast<u64*>(ws);
    u64 *ysend = W64 + Ly.ysend, *yall = W64 + Ly.yall, *up = W64 + Ly.up, *acc = W64 + Ly.acc;
    u64 *psend = W64 + Ly.psend, *pall = W64 + Ly.pall, *conv = W64 + Ly.conv, *tmp = W64 + Ly.tmp;
    if (g.W == 1) {                        // one rank: the gathered layouts are the send blocks
        yall = ysend;
        pall = psend;
    }
    int so[NEO_HOST_ROWS], dof[NEO_HOST_ROWS], pr[NEO_HOST_ROWS];
    auto qpos = [&](int id) { return (int)(std::find(g.my_q.begin(), g.my_q.end(), id) - g.my_q.begin()); };
    auto mpos = [&](int id) { return (int)(std::find(g.mine.begin(), g.mine.end(), id) - g.mine.begin()); };
    int launches = 0;

    // a3: INTT of the own Q limbs, ModUp's [d_i qhat_i^-1]_{q_i} folded in, straight into the
    // send block of each limb's digit: ysend[j][b][u]
    if (nq > 0) {
        TWD sc[NEO_MAX_ROWS];
        int n = 0;
        for (int j = 0; j < g.beta; ++j)
            for (size_t u = 0; u < g.dig_own[j].size(); ++u) {
                const int id = g.dig_own[j][u];
                const std::vector<int>& dj = c->digits[l][j];
                so[n] = qpos(id);
                dof[n] = j * B * g.maxd + (int)u;
                pr[n] = id;
                sc[n] = c->modup_tc[l][j].qhat_inv[std::find(dj.begin(), dj.end(), id) - dj.begin()];
                ++n;
            }
        TRY(ntt_rows(c, false, d_local, (long long)nq * N, so, ysend, (long long)g.maxd * N, dof, pr, n, tmp, B, st,
                     nullptr, false, sc));
        launches += g_launches;
    }
    // exchange #1, one all-gather per digit on the communication stream
    const size_t dbytes = (size_t)B * g.maxd * N * sizeof(u64);
    for (int j = 0; j < g.beta; ++j)
        TRY(comm_allgather(cm, ysend + (size_t)j * B * g.maxd * N, yall + (size_t)j * g.W * B * g.maxd * N, dbytes,
                           st, cm->ev_gath[j]));
    // a4/a5 per digit, as soon as its gather has landed
    for (int j = 0; j < g.beta; ++j) {
        CK(cudaStreamWaitEvent(st, cm->ev_gath[j], 0));
        const BConvTC& P = cm->up_tc[l][j];
        if (P.n_out == 0) continue;
        const std::vector<int>& dj = c->digits[l][j];
        BConvMulti M;
        M.centred = 0; M.dbg = nullptr; M.njobs = 1; M.pre_scaled = 1; M.lazy_out = 1;
        BConvIO io;
        io.in = yall + (size_t)j * g.W * B * g.maxd * N;
        io.out = up;
        io.in_bstride = (long long)g.maxd * N;
        io.out_bstride = (long long)g.beta * nm * N;
        for (size_t i = 0; i < dj.size(); ++i) {
            const int id = dj[i], w = id % g.W;
            // local index of id among its owner's limbs of digit j
            int u = 0;
            for (int t : dj) if (t < id && t % g.W == w) ++u;
            io.in_off[i] = w * B * g.maxd + u;
        }
        int n = 0;
        for (int t : g.mine)
            if (std::find(dj.begin(), dj.end(), t) == dj.end()) {
                io.out_off[n] = j * nm + mpos(t);
                so[n] = dof[n] = j * nm + mpos(t);
                pr[n] = t;
                ++n;
            }
        M.P[0] = P; M.io[0] = io; M.bmat[0] = cm->d_bmat + cm->up_off[l][j];
        LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, B, c->num_sms, st));
        ++launches;
        TRY(ntt_rows(c, true, up, (long long)g.beta * nm * N, so, up, (long long)g.beta * nm * N, dof, pr, n, tmp, B,
                     st, nullptr, true));
        launches += g_launches;
    }
    // a6: KeyIP over the own limbs; a digit's own Q limbs are read from d_local
    if (nm > 0) {
        KeyIPArgs A;
        A.galois = 0; A.accumulate = 0;
        A.d = d_local ? d_local : up; A.up = up; A.evk_lo = k->lo; A.evk_hi = k->hi; A.acc = acc; A.mods = c->d_mods;
        A.d_bstride = (long long)std::max(nq, 1) * N;
        A.up_bstride = (long long)g.beta * nm * N;
        A.acc_bstride = (long long)2 * nm * N;
        A.acc_cstride = (long long)nm * N;
        A.N = N; A.beta = g.beta; A.evk_limbs = c->num_q + c->num_p;
        for (int pos = 0; pos < nm; ++pos) {
            const int id = g.mine[pos];
            A.limb[pos] = id;
            for (int j = 0; j < g.beta; ++j) {
                const std::vector<int>& dj = c->digits[l][j];
                const bool own = std::find(dj.begin(), dj.end(), id) != dj.end();
                A.src_kind[j][pos] = own ? 0 : 1;
                A.src_off[j][pos] = own ? qpos(id) : j * nm + pos;
            }
        }
        LAUNCH(PK_KEYIP, st, launch_keyip(A, nm, B, st));
        ++launches;
    }
    // a7: INTT of the own P rows of acc (both components), P^_k^-1 folded, into the send block
    if (np > 0) {
        TWD sc[NEO_MAX_ROWS];
        for (int u = 0; u < np; ++u) {
            so[u] = nq + u;
            dof[u] = u;
            pr[u] = g.my_p[u];
            sc[u] = c->moddown_tc[l].qhat_inv[g.my_p[u] - c->num_q];
        }
        TRY(ntt_rows(c, false, acc, (long long)nm * N, so, psend, (long long)g.maxp * N, dof, pr, np, tmp, 2 * B, st,
                     nullptr, false, sc));
        launches += g_launches;
    }
    // exchange #2
    TRY(comm_allgather(cm, psend, pall, (size_t)2 * B * g.maxp * N * sizeof(u64), st, cm->ev_p));
    CK(cudaStreamWaitEvent(st, cm->ev_p, 0));
    if (nq == 0) {
        g_launches = launches;
        return NEO_OK;                                      // this rank owns P limbs only
    }
    // a8: ModDown BConv P -> own Q limbs, batch 2B
    {
        BConvMulti M;
        M.centred = 0; M.dbg = nullptr; M.njobs = 1; M.pre_scaled = 1; M.lazy_out = 1;
        BConvIO io;
        io.in = pall; io.out = conv;
        io.in_bstride = (long long)g.maxp * N;
        io.out_bstride = (long long)nq * N;
        for (int kk = 0; kk < g.P; ++kk) io.in_off[kk] = (kk % g.W) * 2 * B * g.maxp + kk / g.W;
        for (int i = 0; i < nq; ++i) io.out_off[i] = i;
        M.P[0] = cm->down_tc[l]; M.io[0] = io; M.bmat[0] = cm->d_bmat + cm->down_off[l];
        LAUNCH(PK_BCONV, st, launch_bconv_tc(M, N, 2 * B, c->num_sms, st));
        ++launches;
    }
    // a9 + a10: NTT of conv with the fused tail out_c = (acc_c - NTT(conv_c)) P^-1
    for (int i = 0; i < nq; ++i) { so[i] = dof[i] = i; pr[i] = g.my_q[i]; }
    RowEpi ep;
    ep.acc = acc;
    ep.acc_b = (long long)2 * nm * N;
    ep.acc_c = (long long)nm * N;
    ep.add0 = ep.add1 = nullptr;
    ep.add_b = 0;
    ep.add_galois = 0;
    ep.out0 = out0; ep.out1 = out1;
    ep.out_b = (long long)nq * N;
    for (int i = 0; i < nq; ++i) ep.pinv[i] = c->pinv[g.my_q[i]];
    TRY(ntt_rows(c, true, conv, (long long)nq * N, so, conv, (long long)nq * N, dof, pr, nq, tmp, 2 * B, st, &ep, true));
    g_launches = launches + g_launches;
    return NEO_OK;
}

}  // extern "C"
