// ntt.h -- launch interface of the two NTT passes (see ntt.cu, ntt_tables.h).
#pragma once
#include "common.cuh"
#include "ntt_tables.h"

namespace neo {

struct NttArgs {
    const TWD* tabd;      // device: [limb id][L.total] twiddle blocks (w, w/q) in FP64
    long long tab_stride; // = L.total
    const ModQ* mods;     // device: per limb id
    int N, N1, N2;
    int num_sms;          // persistent grid = 2 CTAs per SM
    NttLayout L;
};

// One pass over batch x rs.n limb rows.  Forward NTT = column pass (src -> tmp) then row
// pass (tmp -> dst); inverse = row pass then column pass.  src and dst of one pass must
// not overlap.
cudaError_t ntt_pass(bool col, const RowSet& rs, const NttArgs& a, int batch, bool fwd, cudaStream_t st);

}  // namespace neo
