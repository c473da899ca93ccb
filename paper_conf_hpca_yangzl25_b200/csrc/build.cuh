// build.cuh — internal interface of block generation and seed bucketing.
#pragma once
#include <algorithm>
#include <cstring>

#include "common.cuh"
#include "primitives.cuh"

namespace buffalo {

// t1: block 1 also gets its transpose (GraphSAGE-pool's backward scatters through it, R28).
int64_t build_frame_bytes(int64_t n_dst, int64_t e, int layer, bool sizes_only, bool t1 = false);

// Graph workspace (buffalo_graph_workspace_bytes): node_map int32[N] (INT32_MAX when idle), the
// relabel bitmap uint32[W] (zero when idle), its word prefix int32[W + 1] and a scan workspace,
// W = ceil(N / 32).
struct GraphWs {
  uint32_t* bits;
  int32_t* prefix;
  int32_t* scan_ws;
  int64_t words;
};
inline int64_t graph_ws_words(int64_t N) { return ceil_div(N > 0 ? N : 1, 32); }
inline int64_t graph_ws_bytes(int64_t N) {
  const int64_t W = graph_ws_words(N);
  return R(4 * (N > 0 ? N : 1)) + R(4 * W) + R(4 * (W + 1)) + R(4 * scan_ws_elems(W + 1));
}
inline GraphWs graph_ws(const buffalo_graph* g) {
  const int64_t N = g->num_nodes, W = graph_ws_words(N);
  char* q = (char*)g->node_map + R(4 * (N > 0 ? N : 1));
  GraphWs w;
  w.bits = (uint32_t*)q; q += R(4 * W);
  w.prefix = (int32_t*)q; q += R(4 * (W + 1));
  w.scan_ws = (int32_t*)q;
  w.words = W;
  return w;
}

// Builds block `layer` (1-based) whose dst are dst[0..n_dst).  sizes_only: only row_ptr and
// src_global are produced (scheduler statistics).  Allocates from A (bottom: persistent block
// arrays; top frame: scratch).  known = {e_l, n_{l-1}} (exact, from the plan): no host
// synchronisation, n_heavy / n_heavy_t are left at -1; else the stream is synchronised to read
// the sizes (twice, three times for layers >= 2).
buffalo_status build_layer(const buffalo_graph* g, const int32_t* dst, int64_t n_dst, int32_t f,
                           uint32_t hop, uint64_t seed, int layer, bool sizes_only, Arena& A,
                           buffalo_block* blk, cudaStream_t s, const int64_t* known = nullptr,
                           bool t1 = false, const int32_t* cache = nullptr, bool dst_perm = true);

// Input validation: ids in [0, N) and distinct (err_dev |= 1 / 2, stream-ordered, graph
// bitmap left cleared); ids_error maps the word to a status; validate_graph checks the CSR
// (synchronises once).
buffalo_status check_ids(const buffalo_graph* g, const int32_t* ids, int64_t n, int32_t* err_dev, cudaStream_t s);
buffalo_status ids_error(int32_t err, const char* what);
buffalo_status validate_graph(const buffalo_graph* g, int sym, cudaStream_t s);

// Degree bucketing of the seeds (Alg. 3 l.1): bucket[i] = min(D(seed_i), F); order = seed
// positions grouped by bucket (stable); sorted_ids = seeds[order]; hist_h[0..F].
buffalo_status seed_bucketing(const buffalo_graph* g, const int32_t* seeds, int64_t n, int32_t fL,
                              int32_t F, uint8_t* bucket, int32_t* order, int32_t* sorted_ids,
                              int32_t* counts, int32_t* ws, int32_t* starts_dev, int64_t* hist_h,
                              cudaStream_t s);

// Exact per-item block sizes (n[0..L], e[0..L-1]) of up to 256 items (they may overlap): item
// k is sorted_ids[item_start_h[k] .. + item_count_h[k]).  ws: mask_stats_bytes(N, L) bytes; the
// masks are left zeroed (masks_clean = true on the next call saves a memset).  Uses (and
// leaves cleared) the graph workspace's node bitmap.  Synchronises once per layer.
int64_t mask_stats_bytes(int64_t N, int L);
buffalo_status mask_stats(const buffalo_graph* g, const int32_t* sorted_ids, const int64_t* item_start_h,
                          const int64_t* item_count_h, int nitems, const buffalo_sampler* sp, int L, char* ws,
                          int64_t ws_bytes,
                          bool masks_clean, int64_t (*n_h)[BUFFALO_MAX_LAYERS + 1],
                          int64_t (*e_h)[BUFFALO_MAX_LAYERS], cudaStream_t s, int cache_mode = 1);

}  // namespace buffalo
