/*
 * buffalo.h — C ABI of the B200-native hot path of Buffalo (Yang, Zhang, Li, HPCA'25).
 *
 * Paper text: /root/reference/PAPER.md (cited PAPER.md:<line>); readings R<n> are listed in
 * DESIGN.md §2.  Implemented by libbuffalo.so (sm_100a CUDA; no CPU fallback).
 *
 * Conventions (all entry points):
 *  - Pointers are DEVICE pointers unless the name ends in _h (host).  All device memory is
 *    allocated and owned by the caller; the library never calls cudaMalloc/cudaFree.
 *  - `stream` is a cudaStream_t passed as void*.  Work is stream-ordered; the only host
 *    synchronisations are the documented ones (data-dependent sizes).
 *  - Errors are returned as buffalo_status (never exceptions/abort).  Validation errors
 *    (INVALID_ARG, UNSUPPORTED, CAPACITY, BUDGET) leave the outputs (plan, blocks struct,
 *    accumulators) untouched, except *required_bytes_h; caller workspaces and arenas are scratch.
 *    After BUFFALO_ERR_CUDA the outputs are unspecified.  buffalo_last_error() gives a
 *    thread-local message.
 *  - Validated inputs: dims, fanouts, pointers, leading dimensions and alignment on every call;
 *    seed ids (in [0, N), distinct) in buffalo_bucketize and in buffalo_build_blocks without
 *    sizes_h; the CSR itself (O(N + nnz)) on request by buffalo_graph_validate.
 *  - Thread safety: no mutable global state affects results; per-thread state is the error
 *    message, the launch counter and the diagnostic profiler; a per-(kernel, device) cache of
 *    the shared-memory attribute is idempotent.
 *  - Deterministic: identical inputs and seed give bit-identical outputs.
 *  - Built for sm_100a only; on any other device BUFFALO_ERR_UNSUPPORTED.
 *  - A graph's node_map workspace must not be used by two streams at once.
 */
#ifndef BUFFALO_H
#define BUFFALO_H

#include <stddef.h>
#include <stdint.h>

#if defined(__GNUC__)
#define BUFFALO_API __attribute__((visibility("default")))
#else
#define BUFFALO_API
#endif

#ifdef __cplusplus
extern "C" {
#endif

typedef enum {
  BUFFALO_OK = 0,
  BUFFALO_ERR_INVALID_ARG = 1, /* null/misaligned pointer, bad dims, unsupported fanout > 32  */
  BUFFALO_ERR_BUDGET = 2,      /* Alg. 3: no K in [k_min, k_max] satisfies M_ctr            */
  BUFFALO_ERR_CAPACITY = 3,    /* caller buffer/arena too small; *required_bytes_h is set   */
  BUFFALO_ERR_CUDA = 4,        /* CUDA launch/runtime error; see buffalo_last_error()       */
  BUFFALO_ERR_UNSUPPORTED = 5  /* dtype/dim/arch combination not built (e.g. not sm_100a)   */
} buffalo_status;

enum { BUFFALO_FP32 = 0, BUFFALO_BF16 = 1 };            /* storage dtypes                  */
enum { BUFFALO_GEMM_FFMA = 0, BUFFALO_GEMM_BF16 = 1 };  /* Update GEMM: fp32 SIMT | tcgen05 */
/* model: GraphSAGE with aggregator MEAN / POOL / LSTM, or GAT (R20, R28, R29, R30) */
enum { BUFFALO_AGG_MEAN = 0, BUFFALO_AGG_POOL = 1, BUFFALO_AGG_LSTM = 2, BUFFALO_AGG_GAT = 3 };
enum { BUFFALO_MAX_LAYERS = 8, BUFFALO_MAX_FANOUT = 32, BUFFALO_MAX_DIM = 4096 };

/* Input graph (the batch's host graph): CSR, rows sorted ascending, symmetric,
 * no self loops or duplicates.  row_ptr int64[num_nodes+1], col int32[nnz].  node_map points
 * to the graph workspace (buffalo_graph_workspace_bytes): int32[num_nodes] node map, then the
 * relabel node bitmap and its word prefix; prepared once by buffalo_graph_prepare and
 * restored by every call that uses it. */
typedef struct {
  int64_t num_nodes, nnz;
  const int64_t* row_ptr;
  const int32_t* col;
  int32_t* node_map;
} buffalo_graph;

/* Sampling (R1, R2): fanout[l-1] is block l's fanout (<= 0: all neighbours, else <= 32);
 * block l uses hop h = L-l+1; cutoff_F is the degree-bucketing cut-off F;
 * seed keys Philox4x32-10 (per epoch: base + epoch). */
typedef struct {
  int32_t num_layers;
  int32_t fanout[BUFFALO_MAX_LAYERS];
  int32_t cutoff_F;
  uint64_t seed;
  /* Optional sample cache (all NULL: none).  cache[l-1] (for fanout[l-1] > 0, else ignored):
   * device int32 [num_nodes][fanout[l-1]], caller-owned.  buffalo_bucketize writes into it the
   * sampled neighbour list (ascending CSR position) of every node its first statistics pass
   * visits at block l — the whole receptive field of the seed batch — and buffalo_build_blocks
   * copies the rows from it instead of sampling again.  Contract: the cache was filled by
   * buffalo_bucketize on the same graph with a sampler of the same seed and fanouts, and the
   * groups built are groups of that batch; otherwise pass NULLs. */
  int32_t* cache[BUFFALO_MAX_LAYERS];
} buffalo_sampler;

/* A node-id-range sharded feature table (BASELINE.json configs[4], the IGB-shaped
 * 1024-d table of 205 GB that no single GPU holds; the paper's data-parallel mode, PAPER.md:
 * 458-471): rows [k * rows_per_shard, (k + 1) * rows_per_shard) live in shard k, a row-major
 * table with the model's feat_pitch.  shard[k] are device pointers valid in the calling process:
 * its own shard and the peers' shards opened with buffalo_ipc_open (NVLink peer mappings across
 * the GPUs of one NVSwitch box; on one GPU, memory of other processes or plain allocations).
 * Supported for feat_dtype BF16 with gemm_mode BF16 on sampled first blocks (fanout[0] > 0). */
enum { BUFFALO_MAX_SHARDS = 8 };
typedef struct {
  int32_t num_shards;
  int64_t rows_per_shard;
  const void* shard[BUFFALO_MAX_SHARDS];
} buffalo_feature_shards;

/* GraphSAGE-mean model (R20): dim[0] = input feature width, dim[L] = #classes.
 * feat_dtype: dtype of the global feature table (row pitch feat_pitch elements, 16-B aligned
 * rows).  gemm_mode FFMA keeps activations in fp32; BF16 stores activations (H_l, saved
 * h_agg) in bf16 and runs the Update GEMM on tcgen05 tensor cores (fp32 accumulate). */
typedef struct {
  int32_t num_layers;
  int32_t dim[BUFFALO_MAX_LAYERS + 1];
  int32_t feat_dtype;
  int32_t gemm_mode;
  int64_t feat_pitch;
  int32_t aggregator;       /* BUFFALO_AGG_MEAN (default) | _POOL | _LSTM (the last two: gemm_mode FFMA) */
  /* nullable: the feature table is sharded (see buffalo_feature_shards); layer-1 h_src is then
   * ignored, the Aggregate reads neighbour rows from their shards and also copies the dst rows'
   * own feature rows into the block's self_rows (the Update and dW operands: one tensor map
   * cannot span several allocations) */
  const buffalo_feature_shards* feat_shards;
} buffalo_model;

/* Scheduler parameters (Alg. 3): mem_budget = M_ctr in bytes (arena bytes
 * of one micro-batch, R15); C_ppm = average clustering coefficient x 10^6 (Eq. 1, <= 0: R = 1);
 * K searched in [max(k_min, num_gpus), k_max]; k_multiple > 1 (reading R31, rank-aware grouping
 * for data-parallel runs): only multiples of k_multiple are tried, so with k_multiple = num_gpus
 * the K groups can spread evenly over the ranks (the LPT rank assignment still decides; 0 or 1:
 * every K, the paper's loop). */
typedef int32_t (*buffalo_allgather_fn)(void* ctx, const void* send_h, void* recv_h, int64_t bytes);
typedef struct {
  int64_t mem_budget;
  int64_t C_ppm;
  int32_t k_min, k_max, num_gpus;
  int32_t k_multiple;
  /* Data-parallel scheduling: every rank calls buffalo_bucketize with the same
   * inputs and derives the same plan.  rank (0..num_gpus-1) = the caller's rank: the exact block
   * sizes (plan.group_sizes_h) are measured for its own groups only (other rows: -1).
   * allgather (nullable): host all-gather over the ranks — recv_h[r * bytes ...] receives rank
   * r's send_h, returns 0 on success; given, every statistics pass (the degree buckets, the K
   * loop's micro-bucket candidates) is shared out — each rank measures every num_gpus-th item —
   * and the int64 size rows exchanged, so the replicated scheduler work shrinks; the sampler's
   * cache is then not used (no rank visits the whole receptive field); every rank must call
   * bucketize in the same order.  NULL: every rank measures every item. */
  int32_t rank;
  buffalo_allgather_fn allgather;
  void* allgather_ctx;
} buffalo_sched;

/* Output of buffalo_bucketize.  Device arrays sized by the caller: group_of_seed[n_seeds],
 * group_seeds[n_seeds], group_offsets[k_max+1]; host arrays est_bytes_h[k_max],
 * rank_of_group_h[k_max], group_offsets_h[k_max+1], hist_h[cutoff_F+1]. */
typedef struct {
  int32_t* group_of_seed;   /* group of seeds[i]                                            */
  int32_t* group_seeds;     /* seeds grouped; inside a group by (bucket, micro-bucket), input order */
  int64_t* group_offsets;   /* group k = group_seeds[off[k] .. off[k+1])                     */
  int64_t* group_offsets_h;
  int64_t* est_bytes_h;     /* Eq. 2 estimate per group                       */
  int32_t* rank_of_group_h; /* LPT assignment of groups to num_gpus ranks (R24)              */
  int64_t* hist_h;          /* degree-bucket histogram of the seeds, [cutoff_F + 1]           */
  int64_t* group_sizes_h;   /* nullable host [k_max][2L+1]: exact block sizes of each group,
                               n_0..n_L then e_1..e_L (one extra statistics pass over the groups) */
  int32_t k_out;            /* number of non-empty groups                                     */
  int32_t k_tried;          /* the K at which Alg. 4 succeeded                               */
  int32_t exploded;         /* 1 if the degree-F bucket was split (R7)                       */
  int32_t num_items;
} buffalo_plan;

/* One block (bipartite layer) of a micro-batch, all views into the caller's arena.
 * src_global[0..n_dst) are the dst nodes (R3/R4).  row_ptr int32[n_dst+1] (CSR by dst,
 * neighbours in ascending CSR position), col_local int32[n_edges] (index into src),
 * col_global (block 1 only, else NULL) int32[n_edges], t_row_ptr/t_col: transposed block
 * (block >= 2 only, else NULL): for each src j the dst i with an edge to j, ascending.
 * cls_perm int32[n_dst]: the dst sorted by degree class min(D, 129), stable (degree bucketing of
 * the block, Alg. 2 l.6 PAPER.md:238); its tail lists the dst with D > 128 (long-tail cooperative
 * path): heavy = cls_perm + n_dst - n_heavy when the build read the sizes back, else n_heavy = -1
 * and heavy = NULL.  Sampled blocks (fanout > 0) of the mean model have no row past the fanout
 * and are walked in natural order: cls_perm = heavy = NULL, n_heavy = 0.  t_perm int32[n_src] (block >= 2 only): the src sorted by transposed degree
 * class; its tail holds those with more than 128 dst (n_heavy_t of them, or -1 if not counted).
 * Activations of the standard arena layout: agg (saved h_agg [n_dst][ld_agg]), out (H_l
 * [n_dst][ld_out], act dtype, or logits fp32 at l = L), dh (dH_l / dlogits fp32 [n_dst][ld_dh],
 * valid during the backward of layers l and l+1), bwd_scratch (bwd_scratch_bytes). */
typedef struct {
  int64_t n_dst, n_src, n_edges, n_heavy, n_heavy_t;
  int32_t *row_ptr, *col_local, *col_global, *src_global, *t_row_ptr, *t_col, *heavy, *cls_perm, *t_perm;
  void* agg;
  void* out;
  float* dh;
  void* bwd_scratch;
  int64_t ld_agg, ld_out, ld_dh, bwd_scratch_bytes;
  /* aggregator POOL only (else NULL / 0): P = ReLU(H_{l-1} W_pool^T + b_pool) fp32 [n_src][ld_pool]
   * and the argmax of the neighbour max, int32 [n_dst][ld_pool] (local src index, -1 where
   * the max is 0); block 1 then also carries its transpose (t_row_ptr, t_col, t_perm). */
  float* pool_P;
  int32_t* pool_arg;
  int64_t ld_pool;
  /* aggregator LSTM / GAT only (else NULL / 0): the layer's saved state — LSTM: gates, cell
   * states, per-edge source rows and packed positions, running h/c, degree-class counts (R29);
   * GAT: Z = H W^T, the attention scores el / er and the attention weights per edge (R30). */
  void* agg_saved;
  int64_t agg_saved_bytes;
  /* the sampling fanout the block was built with (<= 0: all neighbours).  A sampled block has no
   * row longer than the fanout (<= BUFFALO_MAX_FANOUT < 129), so the forward Aggregate walks its
   * rows in natural order (sequential row_ptr / col reads) instead of through cls_perm. */
  int64_t fanout;
  /* block 1 of a sharded feature table only (else NULL / 0): the dst rows' own feature rows,
   * bf16 [n_dst][ld_self], written by the layer-1 Aggregate, read by the Update and dW GEMMs */
  void* self_rows;
  int64_t ld_self;
} buffalo_block;

typedef struct {
  int32_t num_layers;
  buffalo_block layer[BUFFALO_MAX_LAYERS]; /* layer[l-1] = block l                          */
  int64_t arena_used;  /* bytes reserved at the bottom (blocks + activations)               */
  int64_t arena_peak;  /* high-water mark incl. build and backward scratch frames           */
  int64_t est_lo, est_hi; /* buffalo_estimate_mem of the built sizes                       */
} buffalo_blocks;

/* ------------------------------------------------------------------ graph workspace */
/* Bytes of the graph workspace: node map int32[N], bitmap uint32[ceil(N/32)], word prefix
 * int32[ceil(N/32)+1] and a scan workspace, each 256-B rounded (about 4.2 bytes per node). */
BUFFALO_API size_t buffalo_graph_workspace_bytes(int64_t num_nodes);
/* Sets g->node_map = workspace, fills the node map with INT32_MAX and clears the bitmap
 * (stream-ordered). */
BUFFALO_API buffalo_status buffalo_graph_prepare(buffalo_graph* g, void* workspace, size_t bytes, void* stream);

/* O(N + nnz) check of the CSR contract above on the device: row_ptr monotone from 0 to nnz, ids
 * in [0, N), rows strictly increasing (sorted, no duplicates), no self loops and, with
 * check_symmetric != 0, every (v, c) matched by (c, v) (binary search).  g must be prepared
 * (uses its workspace's scan space).  Synchronises once.  BUFFALO_ERR_INVALID_ARG names the
 * first violated rule.  The hot-path calls trust a validated graph (Alg. 3 input G, PAPER.md:
 * 261-265). */
BUFFALO_API buffalo_status buffalo_graph_validate(const buffalo_graph* g, int32_t check_symmetric, void* stream);

/* ------------------------------------------------------------------ a1-a3: scheduler */
/* Upper bound of the workspace buffalo_bucketize needs for n_seeds seeds. */
BUFFALO_API size_t buffalo_bucketize_workspace_bytes(const buffalo_graph* g, int64_t n_seeds,
                                         const buffalo_sampler* s, const buffalo_model* m);
/* Buffalo_Scheduler (Alg. 3) with DegreeBucketing (l.1), per-item I/O/D and
 * BucketMemEstimator (R13, R15, obtained by building each item's blocks on the GPU),
 * Eq. 1-2, SplitExplosionBucket (R7, R8) and MemBalancedGrouping (Alg. 4,
 * PAPER.md:313-326, R10-R12).  seeds: device int32[n_seeds] (distinct global ids).
 * Synchronises the stream (data-dependent sizes).  BUFFALO_ERR_INVALID_ARG if a seed id is
 * outside [0, N) or occurs twice; BUFFALO_ERR_BUDGET if no K fits M_ctr; BUFFALO_ERR_CAPACITY if
 * workspace_bytes is too small.  The plan is written only on success. */
BUFFALO_API buffalo_status buffalo_bucketize(const buffalo_graph* g, const int32_t* seeds, int64_t n_seeds,
                                 const buffalo_sampler* s, const buffalo_model* m,
                                 const buffalo_sched* sc, buffalo_plan* plan, void* workspace,
                                 size_t workspace_bytes, void* stream);

/* ------------------------------------------------------------------ a4-a6: blocks */
/* MicroBatchGenerator / BlockGenerate (Alg. 2 l.5 PAPER.md:237, §IV-E): the L
 * blocks of the micro-batch whose output nodes are group_seeds[0..n), built top-down, plus the
 * activation and backward buffers of the standard arena layout.  arena: device,
 * 256-B aligned.
 * sizes_h (nullable, host [2L+1]): the group's row of plan.group_sizes_h, i.e. the exact sizes
 *   n_0..n_L, e_1..e_L for this group and sampler.  Given, the arena need is checked up front
 *   (BUFFALO_ERR_CAPACITY with *required_bytes_h = the exact need) and the build runs without
 *   any host synchronisation; n_heavy / n_heavy_t / heavy are then left at -1 / NULL (kernels
 *   find the long rows at the tail of cls_perm / t_perm).  Sizes that do not match the group
 *   give undefined block contents (writes stay inside the arena).
 *   NULL: the group's ids are validated (in [0, N), distinct: BUFFALO_ERR_INVALID_ARG), then the
 *   sizes are read back while building (two to three synchronisations per layer);
 *   BUFFALO_ERR_CAPACITY then reports a lower bound of the need in *required_bytes_h.
 * *out is written only on success. */
BUFFALO_API buffalo_status buffalo_build_blocks(const buffalo_graph* g, const int32_t* group_seeds, int64_t n,
                                    const buffalo_sampler* s, const buffalo_model* m,
                                    buffalo_blocks* out, void* arena, size_t arena_bytes,
                                    int64_t* required_bytes_h, const int64_t* sizes_h, void* stream);

/* ------------------------------------------------------------------ a7: forward */
/* Packed copy of W_l [dim[l], 2*dim[l-1]] fp32 for the kernels (transposes / padded bf16). */
BUFFALO_API size_t buffalo_packed_weight_bytes(const buffalo_model* m, int32_t layer);
BUFFALO_API buffalo_status buffalo_pack_weights(const buffalo_model* m, int32_t layer, const float* W,
                                    void* packed, void* stream);

/* GraphSAGE-mean layer l (Aggregate + Update, Alg. 2 l.8-9, R20/R21):
 *   h_agg[i] = (sum_{e in row i} H[col[e]]) / D(i)   (0 if D(i) = 0),
 *   Z = [H[i] || h_agg[i]] W^T + b;  out = ReLU(Z) (act dtype) for l < L, Z (fp32) for l = L.
 * h_src: for layer 1 the global feature table (feat dtype, row pitch m->feat_pitch, rows
 * addressed by global id through col_global/src_global); for l > 1 H_{l-1} (act dtype, ld_src).
 * saved_agg receives h_agg (act dtype, ld_agg) for the backward.  W fp32 [d_out][2 d_in],
 * W_packed from buffalo_pack_weights, b fp32 [d_out]. */
BUFFALO_API buffalo_status buffalo_sage_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                const void* h_src, int64_t ld_src, const float* W,
                                const void* W_packed, const float* b, void* out, int64_t ld_out,
                                void* saved_agg, int64_t ld_agg, void* stream);

/* ------------------------------------------------------------------ a8: loss */
/* Partial loss of a group (Alg. 2 l.10, R19): loss_accum[0] += sum_i CE(softmax(Z_i), y_i) / S
 * and dlogits = (softmax(Z) - onehot(y)) / S, with y_i = labels[row_ids[i]].  dlogits (and so
 * every gradient) is deterministic; the loss scalar is a reported value accumulated with one
 * float atomic per CTA, so its last bits depend on the CTA completion order. */
BUFFALO_API buffalo_status buffalo_softmax_ce(const float* logits, int64_t ld, int64_t n, int32_t classes,
                                  const int32_t* labels, const int32_t* row_ids,
                                  int64_t batch_size, float* loss_accum, float* dlogits,
                                  int64_t ld_d, void* stream);

/* ------------------------------------------------------------------ a9: backward */
/* Scratch bytes buffalo_sage_bwd needs for block blk at layer l. */
BUFFALO_API size_t buffalo_sage_bwd_scratch_bytes(const buffalo_block* blk, int32_t layer,
                                      const buffalo_model* m);
/* Backward of layer l (Alg. 2 l.11-12).
 *   dZ_l = dH_l * 1[H_l > 0] (l < L) or dlogits (l = L)
 *   dW_accum += dZ^T [H[:n_dst] || h_agg];  db_accum += sum_i dZ[i]   (accumulated, R19)
 *   l > 1: dH_{l-1} = pad(dZ W_self) + (sum_{i: j in N(i)} dZ[i] / D(i)) W_neigh
 * FFMA mode: dh_dst holds dH_l fp32 (l < L; masked IN PLACE using h_dst) or dlogits (l = L);
 * dh_src receives dH_{l-1} fp32.
 * BF16 mode: dh_dst holds dlogits fp32 at l = L; for l < L it holds the layer's prepared
 * backward input as written by the layer above: bf16 dZ_l [n_dst][p(d_l)], then at byte offset
 * R(2 n_dst p(d_l)) fp32 column-sum partials of dZ_l [888][d_l] (summed in row order for db).
 * For l >= 2 the layer computes Ys = dZ W_self and Yn = (dZ W_neigh) / D over its n_dst rows
 * (tcgen05), then the transposed Aggregate dH_{l-1}[j] = [j < n_dst] Ys[j] + sum_{i in T(j)} Yn[i]
 * over the n_src rows with the layer-below epilogue fused: ReLU' with h_src = H_{l-1}, bf16
 * dZ_{l-1} into dh_src and its column-sum partials, i.e. dh_src receives the same prepared form
 * of layer l-1 and must hold R(2 n_src p(d_{l-1})) + R(4 * 888 * d_{l-1}) bytes.
 * Pass dh_src = NULL for layer 1 (features are not trained).
 * Streams: in BF16 mode the layer's dW / db reductions and the long-tail rows of the transposed
 * Aggregate run on two library-owned non-blocking side streams (one pair per device, created
 * on first use), forked from and joined back into `stream` with events before the call returns:
 * the call stays ordered on `stream` for the caller (and for CUDA graph capture). */
BUFFALO_API buffalo_status buffalo_sage_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                float* dh_dst, int64_t ld_dh, const void* h_src, int64_t ld_src,
                                const void* saved_agg, int64_t ld_agg, const void* h_dst,
                                int64_t ld_hdst, const float* W, const void* W_packed,
                                float* dW_accum, float* db_accum, float* dh_src,
                                int64_t ld_dh_src, void* scratch, size_t scratch_bytes, void* stream);

/* ------------------------------------------------------------------ GraphSAGE-pool */
/* the pooling aggregator (the paper's aggregator list "mean, pool or
 * LSTM"; "applicable to any aggregators", :386; GraphSAGE [16]), reading R28.
 * Forward of block `layer` (model.aggregator = BUFFALO_AGG_POOL, gemm_mode FFMA, fp32):
 *   P = ReLU(H_{l-1} W_pool^T + b_pool) over the block's n_src input rows (layer 1: feature rows
 *   via src_global), h_agg[i][k] = max over i's sampled neighbours j of P[j][k] (0 if D = 0),
 *   arg[i][k] = that j, the first in CSR order (-1 where the max is 0), then the Update of
 *   buffalo_sage_fwd: out = [H_self || h_agg] W^T + b (ReLU for l < L).
 * W_pool fp32 [d_{l-1}][d_{l-1}] row-major, b_pool fp32 [d_{l-1}]; W / W_packed / b / out /
 * saved_agg as buffalo_sage_fwd; P, arg: the block's pool_P / pool_arg (ld_pool >= pitch).
 * Deterministic (every reduction order depends only on the row).  Errors: INVALID_ARG (nulls,
 * leading dimensions), UNSUPPORTED (aggregator != POOL or gemm_mode != FFMA). */
BUFFALO_API buffalo_status buffalo_pool_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                const void* h_src, int64_t ld_src, const float* W_pool,
                                const float* b_pool, const float* W, const void* W_packed,
                                const float* b, void* out, int64_t ld_out, void* saved_agg,
                                int64_t ld_agg, float* P, int32_t* arg, int64_t ld_pool,
                                void* stream);
/* Backward of buffalo_pool_fwd (gradients accumulated in place, +=):
 *   dZ = dh_dst * 1[h_dst > 0] (l < L, in place; l = L: dh_dst = dlogits);
 *   dW += dZ^T [H_self || h_agg], db += sum dZ;  dh_agg = dZ W_neigh;
 *   dP[j][k] = sum of dh_agg[i][k] over the dst i with arg[i][k] = j, ascending i through the
 *   transposed block (deterministic);  dQ = dP * 1[P > 0];  dW_pool += dQ^T H_{l-1},
 *   db_pool += sum dQ;  dh_src (l >= 2, NULL at l = 1) = dQ W_pool + pad(dZ W_self).
 * scratch: the block's bwd_scratch (buffalo_sage_bwd_scratch_bytes). */
BUFFALO_API buffalo_status buffalo_pool_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                float* dh_dst, int64_t ld_dh, const void* h_src, int64_t ld_src,
                                const void* saved_agg, int64_t ld_agg, const void* h_dst,
                                int64_t ld_hdst, const float* P, const int32_t* arg, int64_t ld_pool,
                                const float* W_pool, const float* W, float* dW_pool_accum,
                                float* db_pool_accum, float* dW_accum, float* db_accum,
                                float* dh_src, int64_t ld_dh_src, void* scratch,
                                size_t scratch_bytes, void* stream);

/* ------------------------------------------------------------------ GraphSAGE-LSTM */
/* the LSTM aggregator, the paper's memory-intensive case (PAPER.md:56,
 * :63, :125 "degree bucketing ... is crucial for memory-intensive aggregators (e.g., LSTM)",
 * :351, Table III :479-497), reading R29.  For block `layer` (model.aggregator = LSTM, gemm_mode
 * FFMA, fp32): an LSTM of hidden size d = d_{l-1} (gates i, f, g, o; W_ih, W_hh fp32 [4d][d]
 * row-major, b_lstm fp32 [4d] = b_ih + b_hh) runs over each dst row's sampled neighbours in CSR
 * order from zero state; h_agg = its last hidden state (0 for D = 0); then the Update of
 * buffalo_sage_fwd.  The dst rows are processed in degree-class order (the block's cls_perm:
 * the degree buckets of Alg. 2 l.6), so step t is one batched gate GEMM over the rows with
 * D > t.  saved = the block's agg_saved (kept for the backward).  Synchronises the stream once
 * (an 520-byte read of the degree-class counts sizes the per-step launches).  Errors:
 * UNSUPPORTED (a row with more than 128 neighbours; aggregator/gemm_mode), INVALID_ARG. */
BUFFALO_API buffalo_status buffalo_lstm_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                const void* h_src, int64_t ld_src, const float* W_ih,
                                const float* W_hh, const float* b_lstm, const float* W,
                                const void* W_packed, const float* b, void* out, int64_t ld_out,
                                void* saved_agg, int64_t ld_agg, void* agg_saved,
                                size_t agg_saved_bytes, void* stream);
/* Backward (back-propagation through the neighbour sequences; gradients accumulated, +=):
 * dZ, dW, db as buffalo_sage_bwd; dh_agg = dZ W_neigh; per step t = T-1..0 the gate gradients,
 * dW_ih += sum dG x^T, dW_hh += sum dG h_{t-1}^T, db_lstm += sum dG (deterministic split
 * reductions); dh_src (l >= 2) = pad(dZ W_self) + sum over each src's edges (ascending dst) of
 * W_ih^T dG.  Synchronises once (the step table).  scratch: the block's bwd_scratch. */
BUFFALO_API buffalo_status buffalo_lstm_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                float* dh_dst, int64_t ld_dh, const void* h_src, int64_t ld_src,
                                const void* saved_agg, int64_t ld_agg, const void* h_dst,
                                int64_t ld_hdst, void* agg_saved, size_t agg_saved_bytes,
                                const float* W_ih, const float* W_hh, const float* W,
                                float* dW_ih_accum, float* dW_hh_accum, float* db_lstm_accum,
                                float* dW_accum, float* db_accum, float* dh_src, int64_t ld_dh_src,
                                void* scratch, size_t scratch_bytes, void* stream);

/* ------------------------------------------------------------------ GAT */
/* GAT, the paper's second model (Table IV :499-513), on the
 * same blocks, reading R30: one attention head per layer.  For block `layer` (model.aggregator =
 * GAT, gemm_mode FFMA, fp32; W fp32 [d_l][d_{l-1}], a_l, a_r, b fp32 [d_l]): Z = H W^T over the
 * block's src rows; s_ij = LeakyReLU_0.2(a_l . Z[j] + a_r . Z[i]); alpha = softmax over i's
 * sampled neighbours; out_i = sum_j alpha_ij Z[j] + b (b for D = 0); ELU for l < L, logits at
 * l = L.  gat_saved = the block's agg_saved (Z, scores, alpha per edge).  Every reduction order
 * depends only on the row (deterministic).  Block 1 carries its transpose (the backward needs
 * dZ over all src rows for dW). */
BUFFALO_API buffalo_status buffalo_gat_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                               const void* h_src, int64_t ld_src, const float* W, const float* a_l,
                               const float* a_r, const float* b, void* out, int64_t ld_out,
                               void* gat_saved, size_t gat_saved_bytes, void* stream);
/* Backward (accumulated, +=): dOut = dH * ELU'(out) (in place), db += sum dOut; per dst the
 * softmax backward; per src (transposed block, ascending dst) dZ; da_l, da_r, dW = dZ^T H by
 * deterministic split reductions; dh_src (l >= 2) = dZ W.  scratch: the block's bwd_scratch. */
BUFFALO_API buffalo_status buffalo_gat_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                               float* dh_dst, int64_t ld_dh, const void* h_src, int64_t ld_src,
                               const void* h_dst, int64_t ld_hdst, void* gat_saved,
                               size_t gat_saved_bytes, const float* W, const float* a_l,
                               const float* a_r, float* dW_accum, float* db_accum, float* da_l_accum,
                               float* da_r_accum, float* dh_src, int64_t ld_dh_src, void* scratch,
                               size_t scratch_bytes, void* stream);

/* ------------------------------------------------------------------ a10: optimizer */
/* SGD (Alg. 2 l.13, R18): param -= lr * grad; grad = 0 (ready for the next epoch). */
BUFFALO_API buffalo_status buffalo_sgd_step(float* param, float* grad, int64_t n, float lr, void* stream);

/* ------------------------------------------------------------------ memory model */
/* BucketMemEstimator reading R15: exact arena bytes of a micro-batch with
 * layer sizes n[0..L] and e[0..L-1] (e[l-1] = edges of block l).  hi = capacity that always
 * suffices (the scheduler's M_est), lo = bytes the backward is certain to touch; the measured
 * arena peak lies in [lo, hi].  Pure host function. */
BUFFALO_API buffalo_status buffalo_estimate_mem(int32_t num_layers, const int64_t* n, const int64_t* e,
                                    const buffalo_model* m, int64_t* lo_bytes_h,
                                    int64_t* hi_bytes_h);

/* ------------------------------------------------------------------ C of Eq. 1 */
/* The average clustering coefficient C of Eq. 1 (PAPER.md:363 R = min(1, I / (D * O * C));
 * an offline property of the input graph, "page 142 of [27]"), exactly, by
 * triangle counting (reading R27: C = (1/N) * sum_v 2 T_v / (d_v (d_v - 1)), 0 for d_v < 2).
 * Graph as for every call (symmetric, sorted, simple CSR); node_map is not used.  Workspace:
 * caller-owned device buffer of buffalo_clustering_workspace_bytes(g) bytes (the degree-oriented
 * graph: int32[N+1] + int32[nnz/2+1], scan state, 593 doubles), any content.
 * Errors: INVALID_ARG (null pointers, N <= 0), CAPACITY (workspace too small),
 * UNSUPPORTED (nnz/2 or N >= 2^31: the oriented graph uses int32 offsets). */
BUFFALO_API size_t buffalo_clustering_workspace_bytes(const buffalo_graph* g);
/* T int64[num_nodes] (device, overwritten): T[v] = number of triangles through v, i.e. of
 * adjacent pairs among v's neighbours.  Exact integers (bit-exact, any launch order). */
BUFFALO_API buffalo_status buffalo_triangles(const buffalo_graph* g, int64_t* T, void* workspace,
                                 size_t workspace_bytes, void* stream);
/* *C_h = C from T (device, as written by buffalo_triangles), float64 summed in a fixed order
 * (deterministic); *C_ppm_h (nullable) = llround(C * 10^6), the buffalo_sched.C_ppm input.
 * Synchronises the stream once (the 8-byte result). */
BUFFALO_API buffalo_status buffalo_avg_clustering(const buffalo_graph* g, const int64_t* T, double* C_h,
                                      int64_t* C_ppm_h, void* workspace, size_t workspace_bytes,
                                      void* stream);

/* ------------------------------------------------------------------ feature shards over IPC */
/* Cross-process sharing of a feature shard (one process per GPU): the owner exports
 * a device pointer as a handle (cudaIpcGetMemHandle of the driver allocation that contains it,
 * followed by the pointer's 8-byte offset inside that allocation), the handles are exchanged over
 * the process group (torch.distributed), every peer opens them (cudaIpcOpenMemHandle with lazy
 * peer access: NVLink P2P loads on an NVSwitch box) and closes them (with the same handle) when
 * done.  handle_h: host buffer of BUFFALO_IPC_HANDLE_BYTES.  Errors: INVALID_ARG (nulls, pointer
 * outside a device allocation), CUDA (driver refusal). */
enum { BUFFALO_IPC_HANDLE_BYTES = 72 };
BUFFALO_API buffalo_status buffalo_ipc_export(const void* dev_ptr, void* handle_h);
BUFFALO_API buffalo_status buffalo_ipc_open(const void* handle_h, void** dev_ptr_out_h);
BUFFALO_API buffalo_status buffalo_ipc_close(const void* handle_h, void* dev_ptr);

/* Number of kernels this thread has launched through the library (for bench accounting). */
BUFFALO_API int64_t buffalo_launch_count(void);

/* Diagnostics (bench roofline): time every launch of one kernel family with CUDA events on the
 * stream it is launched on.  family "gat_attn": k_gat_attn (GAT softmax + weighted neighbour
 * sum; per row 16 B + the output row, per edge 12 B of index / score / alpha + the Z row).
 * family "lstm_gates": the LSTM gate GEMM of every step; its
 * "algorithmic bytes" are FLOPs (2 x rows x 4d x (d + d)).  family "pool_max": k_pool_max, the GraphSAGE-pool neighbour max
 * (per row 12 B + the max and argmax rows, per edge the index and the pooled fp32 row).
 * family "gather": k_gather_rows, the Aggregate of the forward (mean
 * of neighbour rows) and of the backward (sum of dZ/D rows over the transposed block).
 * counters: caller's device buffer of max_launches uint64 (edges each launch aggregated);
 * launches beyond min(max_launches, 4096) are not timed.  Not thread-safe; one family at a time.
 * buffalo_profile_end synchronises the device and returns the summed launch time, the number of
 * timed launches and their algorithmic bytes: per aggregated edge the 4-B index and the source
 * row (pitch x element size), per row the 4-B permutation entry, two 4-B row_ptr reads and the
 * bf16 output row. */
BUFFALO_API buffalo_status buffalo_profile_begin(const char* family, void* counters, int64_t max_launches,
                                     void* stream);
BUFFALO_API buffalo_status buffalo_profile_end(double* ms_total_h, int64_t* launches_h, double* algo_bytes_h);
BUFFALO_API const char* buffalo_status_str(buffalo_status s);
BUFFALO_API const char* buffalo_last_error(void);

#ifdef __cplusplus
}
#endif
#endif /* BUFFALO_H */
