// params.cpp -- host generation of the RNS parameters and device constant tables.
//
// Primes (rule Z4): q = k*2N + 1 for k from floor((2^W - 1)/2N) downward, W-bit, prime
// (deterministic Miller-Rabin); the first num_q are q_0.., the next num_p are p_0...
// psi (rule Z5): the minimal primitive 2N-th root of unity.
// Tables: NTT twiddles (ntt_tables.h), BConv constants per (level, digit) for ModUp
// (Eq. 2) and per level for ModDown (Table 2), P^-1 mod q_i, q_l^-1 mod q_i.
#include <algorithm>
#include <cmath>
#include <cstring>
#include <stdexcept>

#include <cstdlib>

#include "bconv_tc.h"
#include "context.h"
#include "ntt_tc.h"

namespace neo {

static inline u64 mulm(u64 a, u64 b, u64 m) { return (u64)((u128)a * b % m); }
static u64 powm(u64 a, u64 e, u64 m) {
    u64 r = 1 % m;
    a %= m;
    for (; e; e >>= 1, a = mulm(a, a, m))
        if (e & 1) r = mulm(r, a, m);
    return r;
}
static u64 invm(u64 a, u64 m) { return powm(a, m - 2, m); }   // m prime

static bool is_prime_u64(u64 n) {
    static const u64 bases[] = {2, 3, 5, 7, 11, 13, 17, 19, 23, 29, 31, 37};
    if (n < 2) return false;
    for (u64 b : bases)
        if (n % b == 0) return n == b;
    u64 d = n - 1;
    int s = 0;
    while (!(d & 1)) { d >>= 1; ++s; }
    for (u64 b : bases) {
        u64 x = powm(b, d, n);
        if (x == 1 || x == n - 1) continue;
        bool comp = true;
        for (int r = 1; r < s; ++r) {
            x = mulm(x, x, n);
            if (x == n - 1) { comp = false; break; }
        }
        if (comp) return false;
    }
    return true;
}

std::vector<u64> gen_primes(int log_n, int bits, int count) {
    u64 two_n = 2ull << log_n;
    u64 k = ((1ull << bits) - 1) / two_n;
    std::vector<u64> out;
    while ((int)out.size() < count) {
        if (k == 0) break;
        u64 q = k * two_n + 1;
        if ((q >> (bits - 1)) != 1) break;        // fell below W bits
        if (is_prime_u64(q)) out.push_back(q);
        --k;
    }
    return out;
}

u64 min_psi(u64 q, u64 n) {
    u64 e = (q - 1) / (2 * n);
    u64 psi0 = 0;
    for (u64 x = 2;; ++x) {
        psi0 = powm(x, e, q);
        if (powm(psi0, n, q) == q - 1) break;
    }
    u64 best = psi0, cur = psi0, sq = mulm(psi0, psi0, q);
    for (u64 i = 1; i < n; ++i) {
        cur = mulm(cur, sq, q);
        best = std::min(best, cur);
    }
    return best;
}

static TW mk_tw(u64 w, u64 q) { return TW{w, (u64)(((u128)w << 64) / q)}; }
static TWD mk_twd(u64 w, u64 q) { return TWD{(double)w, (double)w / (double)q}; }   // both exact < 2^53

static int brev(int x, int R) {
    int lg = 0;
    while ((1 << lg) < R) ++lg;
    int y = 0;
    for (int b = 0; b < lg; ++b) y |= ((x >> b) & 1) << (lg - 1 - b);
    return y;
}

// Fill one prime's twiddle block (formulas documented in ntt_tables.h).
static void fill_ntt_block(TWD* t, const NttLayout& L, u64 q, u64 psi, int N) {
    const int R = L.R, N1 = L.N1, N2 = L.N2;
    const u64 ipsi = invm(psi, q);
    auto P = [&](u64 base, long long e) { return powm(base, (u64)e, q); };
    const u64 psi1 = P(psi, N2), ipsi1 = P(ipsi, N2);
    const u64 rho = P(psi1, R), irho = P(ipsi1, R);
    const u64 om1 = P(psi1, 2 * R), iom1 = P(ipsi1, 2 * R);
    const u64 om2 = P(psi, 2 * N1), iom2 = P(ipsi, 2 * N1);
    const u64 om2R = P(om2, R), iom2R = P(iom2, R);
    const u64 ninv = invm((u64)N % q, q);
    for (int k = 0; k < R; ++k) {
        t[L.colf_neg + k] = mk_twd(P(rho, brev(k, R)), q);
        t[L.coli_neg + k] = mk_twd(P(irho, brev(k, R)), q);
    }
    for (int r = 0; r < R; ++r)
        for (int x = 0; x < R; ++x) {
            t[L.colf_tw1 + r * R + x] = mk_twd(P(psi1, (long long)(2 * x + 1) * r), q);
            t[L.coli_tw1 + r * R + x] = mk_twd(P(ipsi1, (long long)(2 * r + 1) * x), q);
            t[L.rowf_tw2 + r * R + x] = mk_twd(P(om2, (long long)x * r), q);
            t[L.rowi_tw2 + r * R + x] = mk_twd(P(iom2, (long long)x * r), q);
        }
    for (int j = 0; j < R / 2; ++j) {
        t[L.colf_cyc + j] = mk_twd(P(om1, j), q);
        t[L.coli_cyc + j] = mk_twd(P(iom1, j), q);
        t[L.rowf_cyc + j] = mk_twd(P(om2R, j), q);
        t[L.rowi_cyc + j] = mk_twd(P(iom2R, j), q);
    }
    // entry 0 of the negacyclic and cyclic tables (the unit twiddle, never read as one) carries
    // (q, fl(1/q)) for the kernels that stage these tables in shared memory
    const TWD qq{(double)q, 1.0 / (double)q};
    t[L.colf_neg] = t[L.coli_neg] = t[L.rowf_cyc] = t[L.rowi_cyc] = qq;
    const u64 two_n = 2ull * N;
    for (int n2 = 0; n2 < N2; ++n2)
        for (int r = 0; r < R; ++r) {
            u64 ea = ((u64)(2 * r + 1) * n2) % two_n;
            u64 eb = ((u64)2 * R * r * n2) % two_n;          // here r plays ib
            t[L.outf_a + n2 * R + r] = mk_twd(P(psi, ea), q);
            t[L.outf_b + n2 * R + r] = mk_twd(P(psi, eb), q);
            t[L.outi_a + n2 * R + r] = mk_twd(mulm(ninv, P(ipsi, ea), q), q);
            t[L.outi_b + n2 * R + r] = mk_twd(P(ipsi, eb), q);
        }
}

static ModQ mk_mod(u64 q) {
    ModQ m;
    m.q = q;
    m.mu = (u64)(((u128)1 << 98) / q);
    m.qd = (double)q;
    m.qinv = 1.0 / (double)q;
    return m;
}

// Algorithm 1 constants for src -> dst limb ids.
static BConvTab make_bconv(const neo_ctx* c, const std::vector<int>& src, const std::vector<int>& dst) {
    BConvTab b;
    std::memset(&b, 0, sizeof(b));
    b.n_in = (int)src.size();
    b.n_out = (int)dst.size();
    for (int i = 0; i < b.n_in; ++i) {
        u64 qi = c->mod[src[i]];
        b.qin[i] = qi;
        u64 qh = 1;                                          // qhat_i mod q_i
        for (int k = 0; k < b.n_in; ++k)
            if (k != i) qh = mulm(qh, c->mod[src[k]] % qi, qi);
        b.qhat_inv[i] = mk_tw(invm(qh, qi), qi);
    }
    for (int j = 0; j < b.n_out; ++j) {
        u64 t = c->mod[dst[j]];
        b.tmod[j] = mk_mod(t);
        for (int i = 0; i < b.n_in; ++i) {
            u64 f = 1;                                       // qhat_i mod t
            for (int k = 0; k < b.n_in; ++k)
                if (k != i) f = mulm(f, c->mod[src[k]] % t, t);
            b.f_lo[i][j] = (unsigned)(f & 0x3FFFF);
            b.f_hi[i][j] = (unsigned)(f >> 18);
        }
    }
    return b;
}

// Tensor-core BConv constants (bconv_tc.cu): B[n = 5t + b][k = 5i + a] =
// byte_b((2^(8a) qhat_i) mod t) in the SWIZZLE_NONE K-major core-matrix layout.
void make_bconv_tc(const std::vector<u64>& src, const std::vector<u64>& dst, BConvTC& P, std::vector<uint8_t>& bmat,
                   const std::vector<u64>* corr) {
    std::memset(&P, 0, sizeof(P));
    P.n_in = (int)src.size();
    P.n_out = (int)dst.size();
    // targets in parts of J = 9 (45 MMA columns, padded to 48): one TMEM job and one
    // tcgen05.ld batch per part in the epilogue
    // 48-bit targets (KLSS T primes at WordSize_T = 48) need 6 constant bytes: 8 targets per part
    u64 tmax = 0;
    for (u64 m : dst) tmax = std::max(tmax, m);
    P.nb = (tmax >> 40) ? 6 : 5;
    const int nb = P.nb;
    P.J = std::min(P.n_out, nb == 5 ? BCTC_PART_J : BCTC_PART_ROWS / 6);
    P.nparts = (P.n_out + P.J - 1) / P.J;
    P.ncols = ((nb * P.J + 15) / 16) * 16;
    bmat.assign((size_t)P.nparts * BCTC_PART_ROWS * 64, 0);
    for (int i = 0; i < P.n_in; ++i) {
        u64 qi = src[i], qh = 1;
        for (int k = 0; k < P.n_in; ++k)
            if (k != i) qh = mulm(qh, src[k] % qi, qi);
        P.qin[i] = (double)qi;
        P.qinv_in[i] = 1.0 / (double)qi;
        P.qhat_inv[i] = mk_twd(invm(qh, qi), qi);
    }
    for (int t = 0; t < P.n_out; ++t) {
        u64 m = dst[t];
        P.t[t] = (double)m;
        P.tinv[t] = 1.0 / (double)m;
        for (int i = 0; i < P.n_in; ++i) {
            u64 f = 1;                                          // qhat_i mod t
            for (int k = 0; k < P.n_in; ++k)
                if (k != i) f = mulm(f, src[k] % m, m);
            for (int a = 0; a < 5; ++a) {
                u64 v = mulm(f, (1ull << (8 * a)) % m, m);      // (2^(8a) qhat_i) mod t
                for (int b = 0; b < nb; ++b) {
                    const int h = t / P.J, n = nb * (t - h * P.J) + b, k = 5 * i + a;
                    size_t off = (size_t)h * BCTC_PART_ROWS * 64 + (size_t)(n / 8) * 512 + (k / 16) * 128 +
                                 (n % 8) * 16 + (k % 16);
                    bmat[off] = (uint8_t)((v >> (8 * b)) & 0xFF);
                }
            }
        }
        if (corr) {                                            // column k = 5 n_in: (-Q_in) mod t, unshifted
            const u64 v = (*corr)[t] % m;
            for (int b = 0; b < nb; ++b) {
                const int h = t / P.J, n = nb * (t - h * P.J) + b, k = 5 * P.n_in;
                size_t off = (size_t)h * BCTC_PART_ROWS * 64 + (size_t)(n / 8) * 512 + (k / 16) * 128 + (n % 8) * 16 +
                             (k % 16);
                bmat[off] = (uint8_t)((v >> (8 * b)) & 0xFF);
            }
        }
    }
}

// Build everything; throws std::runtime_error / returns status through abi.cpp.
neo_status build_context(neo_ctx* c, const neo_params_desc* d, std::string& err) {
    c->log_n = d->log_n;
    c->N = 1 << d->log_n;
    c->num_q = d->num_q;
    c->num_p = d->num_p;
    c->dnum = d->dnum;
    c->word_bits = d->word_bits;
    c->device = d->device;
    c->alpha = (c->num_q + c->dnum - 1) / c->dnum;
    const int nl = c->num_q + c->num_p;
    c->alpha_t = d->alpha_t > 0 ? d->alpha_t : 0;
    if (c->alpha_t && (d->q || d->p)) { err = "KLSS (alpha_t > 0) needs generated primes"; return NEO_EUNSUPPORTED; }
    if (d->q && d->p) {
        c->mod.assign(d->q, d->q + c->num_q);
        c->mod.insert(c->mod.end(), d->p, d->p + c->num_p);
        for (u64 m : c->mod)
            if (m % (2ull * c->N) != 1 || (m >> (c->word_bits - 1)) != 1 || !is_prime_u64(m)) {
                err = "explicit prime is not a word_bits-bit prime = 1 mod 2N";
                return NEO_EINVAL;
            }
    } else {
        c->word_bits_t = c->alpha_t ? (d->word_bits_t > 0 ? d->word_bits_t : c->word_bits) : 0;
        // T primes (K6): the Z4 rule at WordSize_T bits; at WordSize_T = word_bits the sequence
        // continues after q and p, otherwise it starts afresh (disjoint from Q and P by width)
        const bool same = c->word_bits_t == c->word_bits;
        c->mod = gen_primes(c->log_n, c->word_bits, nl + (c->alpha_t && same ? KLSS_MAX_T : 0));
        if ((int)c->mod.size() < nl) { err = "not enough NTT-friendly primes"; return NEO_ENOPRIME; }
        if (c->alpha_t && !same) {
            if (c->word_bits_t != 48) {
                err = "KLSS: WordSize_T must be word_bits or 48";
                return NEO_EUNSUPPORTED;
            }
            c->mod.resize(nl);
            std::vector<u64> tp = gen_primes(c->log_n, c->word_bits_t, KLSS_MAX_T);
            c->mod.insert(c->mod.end(), tp.begin(), tp.end());
        }
    }
    if (c->alpha_t) {
        // KLSS (reading K1-K3, Eq. 4): groups of alpha~ consecutive limbs of q_0..q_L, p_0..p_K;
        // alpha' = least number of T primes with T > 4 beta N B B~, B = alpha max_j Q_j (Algorithm 1's
        // non-centred digit integer), B~ = max_i P~_i.  Compared in log2 (a margin of 1e-9 bits is
        // checked; tests/ compare alpha' with the oracle's exact big-integer count).
        std::vector<int> ext;
        for (int i = 0; i < nl; ++i) ext.push_back(i);
        for (int i = 0; i < nl; i += c->alpha_t)
            c->klss_groups.push_back(std::vector<int>(ext.begin() + i, ext.begin() + std::min(nl, i + c->alpha_t)));
        auto lg = [&](int id) { return std::log2((long double)c->mod[id]); };
        long double lq = 0, lp = 0;
        for (int j = 0; j < c->dnum; ++j) {
            long double s = 0;
            for (int i = j * c->alpha; i < std::min((j + 1) * c->alpha, c->num_q); ++i) s += lg(i);
            lq = std::max(lq, s);
        }
        for (const auto& g : c->klss_groups) {
            long double s = 0;
            for (int id : g) s += lg(id);
            lp = std::max(lp, s);
        }
        const long double need = 2.0L + std::log2((long double)c->dnum) + c->log_n + std::log2((long double)c->alpha) + lq + lp;
        long double have = 0;
        int k = 0;
        while (have <= need && nl + k < (int)c->mod.size()) have += lg(nl + k++);
        if (have <= need || k > KLSS_MAX_T) { err = "KLSS: too many T primes"; return NEO_EUNSUPPORTED; }
        if (std::fabs((double)(have - need)) < 1e-9) { err = "KLSS: Eq. 4 bound too close to call in log2"; return NEO_EUNSUPPORTED; }
        if (nl > KLSS_MAX_EXT) { err = "KLSS: num_q + num_p must be <= 64"; return NEO_EUNSUPPORTED; }
        c->num_t = k;
    }
    c->mod.resize(nl + c->num_t);
    const int ntot = nl + c->num_t;
    c->psi.resize(ntot);
    c->h_mods.resize(ntot);
    for (int i = 0; i < ntot; ++i) {
        c->psi[i] = min_psi(c->mod[i], (u64)c->N);
        c->h_mods[i] = mk_mod(c->mod[i]);
    }
    c->L = make_ntt_layout(c->log_n);

    // ---- device tables
    std::vector<TWD> tab((size_t)ntot * c->L.total);
    for (int i = 0; i < ntot; ++i) fill_ntt_block(&tab[(size_t)i * c->L.total], c->L, c->mod[i], c->psi[i], c->N);
    if (cudaSetDevice(c->device) != cudaSuccess) { err = "cudaSetDevice failed"; return NEO_ECUDA; }
    if (cudaMalloc(&c->d_tab, tab.size() * sizeof(TWD)) != cudaSuccess ||
        cudaMalloc(&c->d_mods, ntot * sizeof(ModQ)) != cudaSuccess) {
        err = "cudaMalloc of constant tables failed";
        return NEO_ENOMEM;
    }
    if (cudaMemcpy(c->d_tab, tab.data(), tab.size() * sizeof(TWD), cudaMemcpyHostToDevice) != cudaSuccess ||
        cudaMemcpy(c->d_mods, c->h_mods.data(), ntot * sizeof(ModQ), cudaMemcpyHostToDevice) != cudaSuccess) {
        err = "cudaMemcpy of constant tables failed";
        return NEO_ECUDA;
    }
    c->ntt.tabd = c->d_tab;
    c->ntt.tab_stride = c->L.total;
    c->ntt.mods = c->d_mods;
    c->ntt.N = c->N;
    c->ntt.N1 = c->L.N1;
    c->ntt.N2 = c->L.N2;
    c->ntt.L = c->L;
    {
        int dev_sms = 0;
        cudaDeviceGetAttribute(&dev_sms, cudaDevAttrMultiProcessorCount, c->device);
        c->num_sms = dev_sms > 0 ? dev_sms : 148;
    }
    c->ntt.num_sms = c->num_sms;
    // tensor-core NTT tables (ntt_tc.cu): N = 2^16 and every prime in (2^35, 2^36)
    {
        std::vector<uint8_t> tct((size_t)ntot * NTC_PRIME_BYTES);
        bool ok = c->N == 65536;
        for (int i = 0; i < ntot && ok; ++i)
            ok = make_ntt_tc_block(&tct[(size_t)i * NTC_PRIME_BYTES], c->mod[i], c->psi[i], c->N);
        if (ok) {
            if (cudaMalloc(&c->d_ntt_tc, tct.size()) != cudaSuccess) { err = "cudaMalloc of NTT tables failed"; return NEO_ENOMEM; }
            if (cudaMemcpy(c->d_ntt_tc, tct.data(), tct.size(), cudaMemcpyHostToDevice) != cudaSuccess) {
                err = "cudaMemcpy of NTT tables failed";
                return NEO_ECUDA;
            }
            c->ntt.tct = c->d_ntt_tc;
            const char* e = std::getenv("NEO_NTT");
            c->ntt_impl = (e && std::string(e) == "tc") ? NEO_NTT_TC : NEO_NTT_FP64;
        }
    }

    // ---- BConv / ModDown / rescale constants per level
    std::vector<int> pids;
    for (int k = 0; k < c->num_p; ++k) pids.push_back(c->num_q + k);
    c->modup.resize(c->num_q);
    c->digits.resize(c->num_q);
    c->moddown.resize(c->num_q);
    c->ql_inv.resize(c->num_q);
    for (int l = 0; l < c->num_q; ++l) {
        std::vector<int> qids;
        for (int i = 0; i <= l; ++i) qids.push_back(i);
        for (int j = 0; j < c->beta(l); ++j) {
            std::vector<int> dj, tg;
            for (int i = j * c->alpha; i < std::min((j + 1) * c->alpha, l + 1); ++i) dj.push_back(i);
            for (int pos = 0; pos < c->ext(l); ++pos) {
                int id = c->ext_id(l, pos);
                if (std::find(dj.begin(), dj.end(), id) == dj.end()) tg.push_back(id);
            }
            c->digits[l].push_back(dj);
            c->modup[l].push_back(make_bconv(c, dj, tg));
            if (c->num_t) {
                std::vector<int> tids;
                for (int k = 0; k < c->num_t; ++k) tids.push_back(nl + k);
                c->klss_up.resize(c->num_q);
                c->klss_up[l].push_back(make_bconv(c, dj, tids));
            }
        }
        c->moddown[l] = make_bconv(c, pids, qids);
        for (int i = 0; i < l; ++i) c->ql_inv[l].push_back(mk_tw(invm(c->mod[l] % c->mod[i], c->mod[i]), c->mod[i]));
    }
    c->ds_inv.assign(c->num_q, {});
    c->ds_ql.assign(c->num_q, {});
    c->ds_qlinv_m.assign(c->num_q, TW{0, 0});
    for (int l = 2; l < c->num_q; ++l) {
        const u64 ql = c->mod[l], qm = c->mod[l - 1];
        c->ds_qlinv_m[l] = mk_tw(invm(ql % qm, qm), qm);
        for (int i = 0; i + 1 < l; ++i) {
            const u64 qi = c->mod[i];
            c->ds_inv[l].push_back(mk_tw(invm(mulm(ql % qi, qm % qi, qi), qi), qi));
            c->ds_ql[l].push_back(mk_tw(ql % qi, qi));
        }
    }
    // tensor-core BConv tables (used when alpha <= 12 and every conversion has <= 51 targets)
    {
        const char* e = std::getenv("NEO_BCONV");
        c->use_tc = !(e && std::string(e) == "cuda");
        // the epilogue's exact FP64 sum of the byte planes needs every Q / P modulus < 2^36
        // (bconv_tc.cu); 48-bit T targets take the 6-byte integer epilogue, 48-bit T inputs the
        // CUDA-core Recover Limbs
        for (int k = 0; k < nl; ++k)
            if (c->mod[k] >> 36) c->use_tc = false;
        c->klss_rec_tc_ok = true;
        for (int k = nl; k < ntot; ++k)
            if (c->mod[k] >> 36) c->klss_rec_tc_ok = false;
        std::vector<uint8_t> all, bm;
        c->modup_tc.resize(c->num_q);
        c->modup_boff.resize(c->num_q);
        c->moddown_tc.resize(c->num_q);
        c->moddown_boff.resize(c->num_q);
        std::vector<u64> pm;
        for (int k = 0; k < c->num_p; ++k) pm.push_back(c->mod[c->num_q + k]);
        bool fits = c->alpha <= BCTC_MAX_IN && c->num_p <= BCTC_MAX_IN;
        for (int l = 0; l < c->num_q && fits; ++l) {
            std::vector<u64> qm(c->mod.begin(), c->mod.begin() + l + 1);
            for (int j = 0; j < c->beta(l); ++j) {
                std::vector<u64> sm, tm;
                const std::vector<int>& dj = c->digits[l][j];
                for (int id : dj) sm.push_back(c->mod[id]);
                for (int pos = 0; pos < c->ext(l); ++pos) {
                    int id = c->ext_id(l, pos);
                    if (std::find(dj.begin(), dj.end(), id) == dj.end()) tm.push_back(c->mod[id]);
                }
                if ((int)tm.size() > BCTC_MAX_OUT) { fits = false; break; }
                BConvTC P;
                make_bconv_tc(sm, tm, P, bm);
                c->modup_tc[l].push_back(P);
                c->modup_boff[l].push_back(all.size());
                all.insert(all.end(), bm.begin(), bm.end());
            }
            if ((int)qm.size() > BCTC_MAX_OUT) { fits = false; break; }
            make_bconv_tc(pm, qm, c->moddown_tc[l], bm);
            c->moddown_boff[l] = all.size();
            all.insert(all.end(), bm.begin(), bm.end());
            if (c->num_t) {                                     // KLSS ModUp: digit -> T
                c->klss_up_tc.resize(c->num_q);
                c->klss_up_boff.resize(c->num_q);
                c->klss_rec_tc.resize(c->num_q);
                c->klss_rec_boff.resize(c->num_q);
                std::vector<u64> tm(c->mod.begin() + nl, c->mod.begin() + nl + c->num_t);
                if (5 * c->num_t >= 64) c->klss_rec_tc_ok = false;   // Recover's correction column: K = 5 alpha' + 1 <= 64
                for (size_t gi = 0; gi < c->klss_groups.size() && c->klss_rec_tc_ok; ++gi) {   // Recover Limbs: T -> group (centred)
                    std::vector<u64> dm, corr;
                    for (int id : c->klss_groups[gi])
                        if (id <= l || id >= c->num_q) {
                            const u64 pm = c->mod[id];
                            u64 T = 1;
                            for (u64 t : tm) T = mulm(T, t % pm, pm);
                            dm.push_back(pm);
                            corr.push_back((pm - T) % pm);
                        }
                    BConvTC P;
                    if (!dm.empty()) {
                        make_bconv_tc(tm, dm, P, bm, &corr);
                        c->klss_rec_boff[l].push_back(all.size());
                        all.insert(all.end(), bm.begin(), bm.end());
                    } else {
                        std::memset(&P, 0, sizeof(P));
                        c->klss_rec_boff[l].push_back(0);
                    }
                    c->klss_rec_tc[l].push_back(P);
                }
                for (int j = 0; j < c->beta(l); ++j) {
                    std::vector<u64> sm;
                    for (int id : c->digits[l][j]) sm.push_back(c->mod[id]);
                    BConvTC P;
                    make_bconv_tc(sm, tm, P, bm);
                    c->klss_up_tc[l].push_back(P);
                    c->klss_up_boff[l].push_back(all.size());
                    all.insert(all.end(), bm.begin(), bm.end());
                }
            }
        }
        if (!fits) c->use_tc = false;
        if (!all.empty()) {
            if (cudaMalloc(&c->d_bmat, all.size()) != cudaSuccess) { err = "cudaMalloc of BConv tables failed"; return NEO_ENOMEM; }
            if (cudaMemcpy(c->d_bmat, all.data(), all.size(), cudaMemcpyHostToDevice) != cudaSuccess) {
                err = "cudaMemcpy of BConv tables failed";
                return NEO_ECUDA;
            }
        }
    }
    if (c->num_t) {                                             // KLSS Recover Limbs constants
        RecTab R;
        std::memset(&R, 0, sizeof(R));
        for (int k = 0; k < c->num_t; ++k) {
            const u64 tk = c->mod[nl + k];
            u64 th = 1;
            for (int m = 0; m < c->num_t; ++m)
                if (m != k) th = mulm(th, c->mod[nl + m] % tk, tk);
            R.that_inv[k] = mk_tw(invm(th, tk), tk);
            R.tinv[k] = 1.0 / (double)tk;
        }
        for (int p = 0; p < nl; ++p) {
            const u64 pm = c->mod[p];
            u64 T = 1;
            for (int k = 0; k < c->num_t; ++k) {
                u64 th = 1;
                for (int m = 0; m < c->num_t; ++m)
                    if (m != k) th = mulm(th, c->mod[nl + m] % pm, pm);
                R.that_p[p][k] = mk_tw(th, pm);
                R.that_lo[p][k] = (unsigned)(th & 0x3FFFF);
                R.that_hi[p][k] = (unsigned)(th >> 18);
                T = mulm(T, c->mod[nl + k] % pm, pm);
            }
            R.T_p[p] = mk_tw(T, pm);
        }
        if (cudaMalloc(&c->d_rec, sizeof(RecTab)) != cudaSuccess ||
            cudaMemcpy(c->d_rec, &R, sizeof(RecTab), cudaMemcpyHostToDevice) != cudaSuccess) {
            err = "KLSS table upload failed";
            return NEO_ECUDA;
        }
    }
    c->pinv.resize(c->num_q);
    for (int i = 0; i < c->num_q; ++i) {
        u64 P = 1;
        for (int k = 0; k < c->num_p; ++k) P = mulm(P, c->mod[c->num_q + k] % c->mod[i], c->mod[i]);
        c->pinv[i] = mk_tw(invm(P, c->mod[i]), c->mod[i]);
    }
    return NEO_OK;
}

}  // namespace neo
