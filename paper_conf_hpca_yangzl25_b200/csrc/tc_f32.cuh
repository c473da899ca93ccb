// tc_f32.cuh — fp32 dW reductions of the FFMA-mode paths on tcgen05 (TF32 splitting), see tc_f32.cu.
#pragma once
#include <algorithm>

#include "common.cuh"

namespace buffalo {

// part[s][m][col] = sum_{r in split s} Z[r][m] F(r, col), F(r, col) = col < d_in ?
// self[gidx ? gidx[r] : r][col] : agg[r][col - d_in] (agg null: F = self only).  The
// k_dw_partial contract (without db, which the caller reduces separately).
struct TcfDw {
  int64_t n;
  int d_out, d_in;
  const float* Z; int64_t ldz;
  const void* self; int64_t lds; const int32_t* gidx;
  const float* agg; int64_t lda;
  float* part;
  int Dp; int64_t rows_per_split;            // set by tcf_dw
};
// 16-B row alignment the staging loads need (fp32: 4 elements, bf16: 8).
inline bool tcf_aligned(const void* p, int64_t ld, int elem) {
  return p == nullptr || ((((uintptr_t)p) % 16) == 0 && (ld * elem) % 16 == 0);
}
buffalo_status tcf_dw(TcfDw p, int S, bool self_bf16, cudaStream_t s);

}  // namespace buffalo
