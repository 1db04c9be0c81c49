// ntt_tc.h -- the 4-step NTT with both radix-16 DFT stages of every pass on the 5th-gen
// tensor cores (ntt_tc.cu).  Same RowSet / TileMap / RowEpi interface as ntt.cu's FP64 passes.
#pragma once
#include <vector>

#include "common.cuh"
#include "ntt.h"

namespace neo {

// Pass types (the four 256-point passes of N = 2^16 = 256 x 256)
enum { TC_COL_FWD = 0, TC_ROW_FWD = 1, TC_ROW_INV = 2, TC_COL_INV = 3 };

// Per (prime, pass type) table block, in the exact shared-memory image the kernel uses:
//   S1 (7680 B): stage-1 B matrix, 80 rows (n = 16 b + o) x 96 bytes (K), SWIZZLE_NONE K-major
//   S2 (7680 B): stage-2 B matrix, same layout
//   T  (4096 B): inter-stage twiddles, TWD [p_a][o_a]
constexpr int NTC_BMAT = 80 * 96;
constexpr int NTC_TW = 16 * 16 * 16;
constexpr int NTC_PASS_BYTES = 2 * NTC_BMAT + NTC_TW;           // 19456
constexpr int NTC_PRIME_BYTES = 4 * NTC_PASS_BYTES;             // 77824

// Host: fill one prime's four pass blocks (N = 2^16 only).  Returns false if the prime is not
// supported (q must be in (2^35, 2^36) so that the exact FP64 epilogue bounds hold).
bool make_ntt_tc_block(uint8_t* dst, u64 q, u64 psi, int N);

// One pass, tensor-core form.  Requires N = 2^16 and a.tct != nullptr.
cudaError_t ntt_pass_tc(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st,
                        const RowEpi* epi = nullptr);

}  // namespace neo
