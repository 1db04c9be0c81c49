// bconv_tc.h -- tensor-core BConv (bconv_tc.cu): constants and launcher.
#pragma once
#include <cuda.h>   // CUtensorMap (the type only; the encoder is fetched through the runtime)

#include <vector>

#include "common.cuh"
#include "context.h"

namespace neo {

// Host: the pre-shifted byte matrix B[n = 5t + b][k = 5i + a] = byte_b(2^(8a) qhat_i mod t),
// stored in the SWIZZLE_NONE K-major core-matrix layout (ncols x 64 bytes).
// corr (optional, KLSS Recover Limbs): corr[t] = (-Q_in) mod t fills the extra K column 5 n_in,
// which the producers load with u = rint(sum_i y_i / q_i), so the GEMM returns the CENTRED lift
// sum_i y_i qhat_i - u Q_in (exact while |x| < Q_in / 4); needs 5 n_in < 64.
void make_bconv_tc(const std::vector<u64>& src_mod, const std::vector<u64>& dst_mod, BConvTC& P,
                   std::vector<uint8_t>& bmat, const std::vector<u64>* corr = nullptr);

size_t bconv_tc_smem(int ncols);

// Up to BCTC_MULTI_JOBS conversions with the same input/output batch geometry in one launch (e.g.
// the beta ModUp digits), with at most BCTC_MULTI_PARTS target parts in total (B matrices packed
// back to back in shared memory); B matrices from device memory.
constexpr int BCTC_MULTI_JOBS = 12;
constexpr int BCTC_MULTI_PARTS = 20;
struct BConvMulti {
    CUtensorMap tmap[BCTC_MULTI_JOBS];     // filled by launch_bconv_tc: 3-D map {N, rows, batch} of job j's input
    int use_tmap[BCTC_MULTI_JOBS];         // 1: one tensor TMA per tile (inputs rows contiguous), 0: per-row bulk copies
    int njobs;
    int pre_scaled;      // inputs already hold y_i = [c_i qhat_i^-1]_{q_i} (scale folded into the INTT)
    int lazy_out;        // write lazy doubles |x| < 2^40 for the next NTT instead of canonical u64
    int centred;         // B has the correction column of make_bconv_tc(corr): producers supply u
    BConvTC P[BCTC_MULTI_JOBS];
    BConvIO io[BCTC_MULTI_JOBS];
    const uint8_t* bmat[BCTC_MULTI_JOBS];
    unsigned long long* dbg;   // optional clock64 trace of CTA 0 (NEO_BCONV_DBG): [tile][8]
};
cudaError_t launch_bconv_tc(const BConvMulti& M, int N, int batch, int num_sms, cudaStream_t st);
// true if job P still fits a BConvMulti holding M.njobs jobs (job and part limits)
bool bconv_multi_fits(const BConvMulti& M, const BConvTC& P);
// One conversion with B passed by value (generic neo_bconv).
cudaError_t launch_bconv_tc_param(const BConvTC& P, const BConvIO& io, const BMatParam& bp, int N, int batch,
                                  int num_sms, cudaStream_t st);

}  // namespace neo
