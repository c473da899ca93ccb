// tc_sage.cuh — tcgen05 (5th-gen tensor core) path of the fused SAGE layer.
#pragma once
#include "common.cuh"
#include "sage.cuh"

namespace buffalo {

int64_t tc_packed_bytes(int64_t d_in, int64_t d_out);
buffalo_status tc_pack_weights(const float* W, int d_in, int d_out, void* packed, cudaStream_t s);
int64_t tc_fwd_packed_bytes(int64_t d_in, int64_t d_out);
bool tc_fwd_supported(const FwdArgs& a);
buffalo_status tc_sage_fwd(const FwdArgs& a, cudaStream_t s);
int tc_dw_splits(int64_t n, int d_out, int d_in);
int64_t tc_bwd_db_parts();   // db partial rows of the bf16 backward's prepared dZ
int64_t tc_bwd_scratch_bytes(int64_t n_dst, int64_t n_src, int64_t e, int layer, int d_in, int d_out, bool last);
bool tc_bwd_supported(const BwdArgs& a);
buffalo_status tc_sage_bwd(const BwdArgs& a, cudaStream_t s);
buffalo_status tc_dw_tma(int64_t n, int S, const __nv_bfloat16* z, int64_t ldz, int d_out,
                         const __nv_bfloat16* self, int64_t lds, const int32_t* gidx, int64_t self_table_rows,
                         const __nv_bfloat16* agg, int64_t lda, int d_in, float* part, cudaStream_t s);
buffalo_status tc_gemm_tma(int64_t n_rows, int64_t self_rows, const int32_t* self_idx, const __nv_bfloat16* self,
                           int64_t ld_self, const __nv_bfloat16* agg,
                           int64_t ld_agg, int d_in, const uint8_t* wpk, int d_out, const float* bias, int relu,
                           int out_f32, void* out, int64_t ld_out, cudaStream_t s,
                           const int32_t* scale_rp = nullptr);

}  // namespace buffalo
