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
// The same partials with fp32 self rows, operands loaded by TMA (MN-major); same split count S.
buffalo_status tcf_dw_tma(const TcfDw& p, int S, cudaStream_t s);

// C[r][n] = act(sum_k A1[gidx ? gidx[r] : r][k] B1(k, n) [r < m1] + sum_k A2[r][k] B2(k, n) +
// bias[n]) for n < N, 0 for N <= n < Np; B(k, n) = tb ? B[n][k] : B[k][n].  The k_gemm2_tc
// contract (sage.cu) with fp32 output; every pointer / pitch must pass tcf_aligned.
struct TcfGemm {
  int64_t M; int N, Np, K1, K2;
  const void* A1; int64_t lda1; const int32_t* gidx; int64_t m1;
  const float* A2; int64_t lda2;
  const float* B1; int64_t ldb1;
  const float* B2; int64_t ldb2;
  const float* bias; int relu;
  float* C; int64_t ldc;
};
// The tensor pipe accumulates in TMEM without IEEE rounding; over K = 2866 (Cora layer 1) that
// flips ReLU signs the fp32 FFMA path gets right, so longer K stays on the fallback kernels.
constexpr int kTcfMaxK = 512;
// exact: NS = 3 terms (operands represented exactly: the FFMA path's fp32 accuracy) instead of
// the 3xTF32 split (NS = 2) of the mma.sync path for short K.
buffalo_status tcf_gemm(const TcfGemm& p, bool a1_bf16, bool tb, bool exact, cudaStream_t s);

}  // namespace buffalo
