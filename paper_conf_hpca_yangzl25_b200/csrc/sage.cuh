// sage.cuh — internal interface of the GraphSAGE-mean layer kernels.
#pragma once
#include "common.cuh"

namespace buffalo {

struct FwdArgs {
  const buffalo_block* blk;
  bool layer1;       // input rows are global ids (features) via col_global / src_global
  bool in_bf16;      // dtype of h_src
  bool act_bf16;     // dtype of saved agg and (l < L) output
  bool out_f32;      // output logits in fp32 (last layer)
  int relu;
  int d_in, d_out;
  const void* h_src; int64_t ld_src;
  const float* W; const void* W_packed; const float* b;
  void* out; int64_t ld_out;
  void* agg; int64_t ld_agg;
  const buffalo_feature_shards* shards;   // layer 1 of a sharded feature table (else null)
};

struct BwdArgs {
  const buffalo_block* blk;
  bool layer1, in_bf16, act_bf16, last;
  int d_in, d_out;
  float* dh; int64_t ld_dh;
  const void* h_src; int64_t ld_src;
  const void* agg; int64_t ld_agg;
  const void* h_dst; int64_t ld_hdst;
  const float* W; const void* W_packed;
  float* dW; float* db;
  float* dh_src; int64_t ld_dh_src;
  void* scratch; int64_t scratch_bytes;
  const buffalo_feature_shards* shards;   // layer 1 of a sharded feature table (else null)
};

// GraphSAGE-pool (R28): FFMA path, fp32 activations.
struct PoolArgs {
  const buffalo_block* blk;
  bool layer1, in_bf16, last;
  int d_in, d_out;
  const void* h_src; int64_t ld_src;
  const float* W_pool; const float* b_pool;
  const float* W; const float* W_packed; const float* b;
  float* out; int64_t ld_out;
  float* agg; int64_t ld_agg;
  float* P; int32_t* arg; int64_t ld_pool;
  // backward
  float* dh; int64_t ld_dh;
  const float* h_dst; int64_t ld_hdst;
  float* dW_pool; float* db_pool; float* dW; float* db;
  float* dh_src; int64_t ld_dh_src;
  void* scratch; int64_t scratch_bytes;
};
int pool_dw_splits(int64_t n_rows, int d);
int64_t pool_bwd_scratch_bytes(int64_t n_dst, int64_t n_src, int d_in, int d_out);
buffalo_status pool_fwd_ffma(const PoolArgs& a, cudaStream_t s);
buffalo_status pool_bwd_ffma(const PoolArgs& a, cudaStream_t s);

// GraphSAGE-LSTM (R29): FFMA path, fp32 activations.
struct LstmArgs {
  const buffalo_block* blk;
  bool layer1, in_bf16, last;
  int d_in, d_out;
  const void* h_src; int64_t ld_src;
  const float* W_ih; const float* W_hh; const float* b_lstm;
  const float* W; const float* W_packed; const float* b;
  float* out; int64_t ld_out;
  float* agg; int64_t ld_agg;
  void* saved;
  float* dh; int64_t ld_dh;
  const float* h_dst; int64_t ld_hdst;
  float* dW_ih; float* dW_hh; float* db_lstm; float* dW; float* db;
  float* dh_src; int64_t ld_dh_src;
  void* scratch;
};
int lstm_dw_splits(int64_t n_rows, int d);
int64_t lstm_saved_bytes(int64_t n, int64_t e, int d);
int64_t lstm_bwd_scratch_bytes(int64_t n_dst, int64_t e, int layer, int d_in, int d_out);
buffalo_status lstm_fwd_ffma(const LstmArgs& a, cudaStream_t s);
buffalo_status lstm_bwd_ffma(const LstmArgs& a, cudaStream_t s);

// GAT (R30): one head per layer, FFMA path, fp32 activations.
struct GatArgs {
  const buffalo_block* blk;
  bool layer1, in_bf16, last;
  int d_in, d_out;
  const void* h_src; int64_t ld_src;
  const float* W; const float* a_l; const float* a_r; const float* b;
  float* out; int64_t ld_out;
  void* saved;
  float* dh; int64_t ld_dh;
  const float* h_dst; int64_t ld_hdst;
  float* dW; float* db; float* da_l; float* da_r;
  float* dh_src; int64_t ld_dh_src;
  void* scratch;
};
int gemm_splits(int64_t n_rows, int rows_out, int K);
int64_t gat_saved_bytes(int64_t n_src, int64_t n_dst, int64_t e, int d_out);
int64_t gat_bwd_scratch_bytes(int64_t n_src, int64_t n_dst, int64_t e, int d_in, int d_out);
buffalo_status gat_fwd_ffma(const GatArgs& a, cudaStream_t s);
buffalo_status gat_bwd_ffma(const GatArgs& a, cudaStream_t s);

int dw_splits(int64_t n_l, int d_out, int d_in);
int64_t bwd_scratch_bytes(int64_t n_dst, int64_t n_src, int layer, int d_in, int d_out);

buffalo_status sage_fwd_ffma(const FwdArgs& a, cudaStream_t s);
buffalo_status sage_bwd_ffma(const BwdArgs& a, cudaStream_t s);
buffalo_status launch_softmax_ce(const float* logits, int64_t ld, int64_t n, int classes,
                                 const int32_t* labels, const int32_t* ids, int64_t S,
                                 float* loss, float* dl, int64_t ldd, cudaStream_t s);
buffalo_status launch_sgd(float* p, float* g, int64_t n, float lr, cudaStream_t s);
buffalo_status launch_transpose_w(const float* W, int rows, int cols, float* Wt, cudaStream_t s);

}  // namespace buffalo
