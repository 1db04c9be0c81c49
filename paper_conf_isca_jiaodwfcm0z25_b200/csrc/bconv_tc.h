// bconv_tc.h -- tensor-core BConv (bconv_tc.cu): constants and launcher.
#pragma once
#include <vector>

#include "common.cuh"
#include "context.h"

namespace neo {

// Host: the pre-shifted byte matrix B[n = 5t + b][k = 5i + a] = byte_b(2^(8a) qhat_i mod t),
// stored in the SWIZZLE_NONE K-major core-matrix layout (ncols x 64 bytes).
void make_bconv_tc(const std::vector<u64>& src_mod, const std::vector<u64>& dst_mod, BConvTC& P,
                   std::vector<uint8_t>& bmat);

size_t bconv_tc_smem(int ncols);
// B from device memory (bmat) or by value (bp != nullptr).
cudaError_t launch_bconv_tc(const BConvTC& P, const BConvIO& io, const uint8_t* bmat, const BMatParam* bp, int N,
                            int batch, int num_sms, cudaStream_t st);

}  // namespace neo
