// build.cu — block generation and seed degree bucketing (a1).
//
// BlockGenerate / MicroBatchGenerator (Alg. 2 l.5; §IV-E):
// for every dst row of the layer, in parallel at the node level ("tracking neighbors happens
// in parallel at the node level"): count -> scan -> sample/slice -> relabel into
// a bipartite block (dst prefix + first occurrence, R3/R4) -> transpose for the backward.
#include "build.cuh"

#include <cooperative_groups.h>
namespace cg = cooperative_groups;
#include "philox.cuh"
#include "primitives.cuh"

namespace buffalo {

// ------------------------------------------------------------------ a4: count D per dst
// D(i) = min(deg(dst[i]), f) (all neighbours for f <= 0), evaluated inside the row_ptr scan.
struct LoadDeg {
  const int32_t* dst;
  const int64_t* grow;
  int32_t f;
  __device__ __forceinline__ int32_t operator()(int64_t i) const {
    const int64_t v = dst[i];
    const int64_t deg = grow[v + 1] - grow[v];
    return (int32_t)((f > 0 && deg > f) ? f : deg);
  }
};

// ------------------------------------------------------------------ a4: sample / slice
// A warp serves 32/SEG destination rows (SEG lanes each, SEG >= f).  deg <= f or f <= 0: the
// segment copies the CSR row.  Otherwise Floyd's algorithm (R2): lane t of the segment computes
// r_t = floor(x_t (j_t + 1) / 2^32), j_t = deg - f + t; the sequential membership test runs as
// f ballot steps (all lanes execute them, so sampling and copying segments may share a warp);
// the chosen positions are ranked (sorted ascending) inside the segment.
// emit(slot, k, u): neighbour number k (ascending CSR position) of the warp's row `slot` is u.
template <int SEG, class RowFn, class Emit>
__device__ __forceinline__ void sample_warp_rows(int64_t w, int64_t n, RowFn row_of, const int64_t* __restrict__ grow,
                                                 const int32_t* __restrict__ gcol, int32_t f, uint32_t hop,
                                                 uint64_t seed, Emit emit) {
  constexpr int G = 32 / SEG;
  const int lane = threadIdx.x & 31, g = lane / SEG, sl = lane % SEG;
  const int64_t slot = w * G + g;
  uint32_t v = 0;
  int64_t beg = 0, deg = 0;
  if (slot < n) {
    v = (uint32_t)row_of(slot);
    beg = grow[v];
    deg = grow[v + 1] - beg;
  }
  const bool samp = slot < n && f > 0 && deg > f;
  if (__any_sync(0xffffffffu, samp)) {
    const uint32_t j = (uint32_t)(deg - f) + (uint32_t)sl;
    uint32_t r = 0;
    if (samp && sl < f) r = __umulhi(sample_draw(seed, v, hop, (uint32_t)sl), j + 1u);
    int32_t S = -1;
    const unsigned segmask = (SEG == 32) ? 0xffffffffu : (((1u << SEG) - 1u) << (g * SEG));
    for (int t = 0; t < f; ++t) {
      const int32_t cand = (int32_t)__shfl_sync(0xffffffffu, r, g * SEG + t);
      const unsigned present = __ballot_sync(0xffffffffu, sl < t && S == cand) & segmask;
      if (sl == t) S = present ? (int32_t)((uint32_t)(deg - f) + (uint32_t)t) : cand;
    }
    int rank = 0;
    for (int u = 0; u < f; ++u) {
      const int32_t su = __shfl_sync(0xffffffffu, S, g * SEG + u);
      rank += (su < S) ? 1 : 0;
    }
    if (samp && sl < f) emit(slot, rank, gcol[beg + S]);
  }
  if (slot < n && !samp)
    for (int64_t k = sl; k < deg; k += SEG) emit(slot, (int32_t)k, gcol[beg + k]);
}

struct DstRows {
  const int32_t* dst;
  __device__ __forceinline__ int64_t operator()(int64_t i) const { return dst[i]; }
};

// The first step of the relabel (R3) fused into the fills: every written neighbour u is looked
// up in the node map (the layer's dst were entered by k_set_map before the fill), the result
// kept in mapped[pos] (the dst prefix id, or INT32_MAX), and a non-dst u is marked in the node
// bitmap.  mapped == null: fill only (no relabel).
struct MarkCtx {
  const int32_t* node_map;
  uint32_t* bits;
  int32_t* mapped;
  __device__ __forceinline__ void operator()(int64_t pos, int32_t u) const {
    if (!mapped) return;
    const int32_t m = node_map[u];
    mapped[pos] = m;
    if (m != INT32_MAX) return;                                  // a dst: keeps its prefix id
    const uint32_t b = 1u << (u & 31);
    if (!(bits[u >> 5] & b)) atomicOr(&bits[u >> 5], b);
  }
};

template <int SEG>
__global__ void __launch_bounds__(256) k_sample_fill(const int32_t* __restrict__ dst, int64_t n,
                                                     const int64_t* __restrict__ grow,
                                                     const int32_t* __restrict__ gcol, int32_t f,
                                                     uint32_t hop, uint64_t seed,
                                                     const int32_t* __restrict__ row_ptr,
                                                     int32_t* __restrict__ out, int64_t cap, MarkCtx mk) {
  pdl_wait();
  constexpr int G = 32 / SEG;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * G < n; w += warps)
    sample_warp_rows<SEG>(w, n, DstRows{dst}, grow, gcol, f, hop, seed, [&](int64_t slot, int32_t k, int32_t u) {
      const int64_t pos = (int64_t)row_ptr[slot] + k;
      if (pos < cap) {
        out[pos] = u;
        mk(pos, u);
      }
    });
}

// Rows from the sample cache (filled by the scheduler's statistics pass): SEG lanes per row,
// lane k copies entry k of the row's cached list (D = min(deg, f) entries, CSR order).
template <int SEG>
__global__ void __launch_bounds__(256) k_cache_fill(const int32_t* __restrict__ dst, int64_t n,
                                                    const int32_t* __restrict__ cache, int32_t f,
                                                    const int32_t* __restrict__ row_ptr, int32_t* __restrict__ out,
                                                    int64_t cap, MarkCtx mk) {
  pdl_wait();
  // kR rows per lane group and iteration: their row_ptr / dst -> cache row -> node map chains
  // are in flight together (one chain per iteration left the kernel latency-bound)
  constexpr int G = 32 / SEG, kR = 4;
  const int lane = threadIdx.x & 31, g = lane / SEG, sl = lane % SEG;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * G < n; w += kR * warps) {
    int32_t b[kR], u[kR], mm[kR];
#pragma unroll
    for (int r = 0; r < kR; ++r) {
      const int64_t slot = (w + r * warps) * G + g;
      u[r] = -1;
      b[r] = 0;
      if (slot < n) {
        b[r] = __ldg(row_ptr + slot);
        const int32_t D = __ldg(row_ptr + slot + 1) - b[r];
        if (sl < D && b[r] + sl < cap) u[r] = __ldg(cache + (int64_t)__ldg(dst + slot) * f + sl);
      }
    }
#pragma unroll
    for (int r = 0; r < kR; ++r) mm[r] = (u[r] >= 0 && mk.mapped) ? __ldg(mk.node_map + u[r]) : 0;
#pragma unroll
    for (int r = 0; r < kR; ++r) {
      if (u[r] < 0) continue;
      const int64_t pos = (int64_t)b[r] + sl;
      out[pos] = u[r];
      if (!mk.mapped) continue;
      mk.mapped[pos] = mm[r];
      if (mm[r] != INT32_MAX) continue;                            // a dst: keeps its prefix id
      const uint32_t bit = 1u << (u[r] & 31);
      if (!(mk.bits[u[r] >> 5] & bit)) atomicOr(&mk.bits[u[r] >> 5], bit);
    }
  }
}

static inline int sample_seg(int32_t f) { return (f > 0 && f <= 8) ? 8 : (f > 0 && f <= 16) ? 16 : 32; }

template <class... Args>
static void launch_sample_fill(int seg, int64_t n, cudaStream_t s, Args... args) {
  const int G = 32 / seg;
  const int grid = grid_for(ceil_div(n, G) * 32, 256, 16);
  if (seg == 8) launch_pdl(k_sample_fill<8>, dim3(grid), dim3(256), 0, s, args...);
  else if (seg == 16) launch_pdl(k_sample_fill<16>, dim3(grid), dim3(256), 0, s, args...);
  else launch_pdl(k_sample_fill<32>, dim3(grid), dim3(256), 0, s, args...);
}

// ------------------------------------------------------------------ a5: relabel
// Local src ids (R3): the dst keep their positions 0..n_dst-1 (node_map[dst[i]] = i); the other
// distinct neighbours follow in ascending global id.  They are marked in a node bitmap; an
// exclusive popcount scan over its words gives each word's first local id, so that
// local(u) = n_dst + prefix[u / 32] + popc(bits[u / 32] & below(u % 32)).
__global__ void k_set_map(const int32_t* __restrict__ src, int64_t n, int32_t* __restrict__ node_map) {
  pdl_wait();
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    node_map[src[j]] = (int32_t)j;
}
__global__ void k_reset_map(const int32_t* __restrict__ src, int64_t n, int32_t* __restrict__ node_map) {
  pdl_wait();
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
    node_map[src[j]] = INT32_MAX;
}
// mapped (nullable): node_map[u] per edge, kept for k_col_local (a coalesced re-read instead of a
// second random node-map lookup).
struct PopcWord {
  const uint32_t* bits;
  __device__ __forceinline__ int32_t operator()(int64_t w) const { return __popc(bits[w]); }
};
// Scan store: the word's exclusive prefix.
struct StorePrefix {
  int32_t* prefix;
  __device__ __forceinline__ void operator()(int64_t w, int32_t excl, int32_t) const { prefix[w] = excl; }
};
// The marked nodes appended to src (at src + n_dst) in ascending id: thread per bitmap word.
__global__ void k_emit_bits(const uint32_t* __restrict__ bits, const int32_t* __restrict__ prefix, int64_t words,
                            int32_t* __restrict__ src, int64_t cap) {
  pdl_wait();
  for (int64_t w = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; w < words; w += (int64_t)gridDim.x * blockDim.x) {
    uint32_t m = bits[w];
    int32_t r = m ? prefix[w] : 0;
    while (m) {
      const int b = __ffs(m) - 1;
      m &= m - 1;
      if (r < cap) src[r] = (int32_t)(w * 32 + b);
      ++r;
    }
  }
}
// col_local of every edge (holding node_map[u] from k_mark_bits on entry); tcnt (layers >= 2,
// zeroed): transposed row lengths counted on the way.
__global__ void k_col_local(const int32_t* __restrict__ colg, int64_t e, const int32_t* __restrict__ node_map,
                            const uint32_t* __restrict__ bits, const int32_t* __restrict__ prefix, int32_t n_dst,
                            int32_t* __restrict__ col_local, int32_t* __restrict__ tcnt) {
  pdl_wait();
  // kR edges per thread and iteration (coalesced per r): their bitmap / prefix lookups in flight together
  constexpr int kR = 4;
  (void)node_map;                        // looked up by the fill already (col_local holds node_map[u])
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * kR;
  for (int64_t k0 = blockIdx.x * (int64_t)blockDim.x * kR + threadIdx.x; k0 < e; k0 += stride) {
    int32_t u[kR], m[kR], c[kR];
#pragma unroll
    for (int r = 0; r < kR; ++r) {
      const int64_t k = k0 + (int64_t)r * blockDim.x;
      u[r] = -1;
      m[r] = 0;
      if (k < e) {
        u[r] = __ldg(colg + k);
        m[r] = col_local[k];                                    // node_map[u], kept by the fill
      }
    }
#pragma unroll
    for (int r = 0; r < kR; ++r) {
      c[r] = m[r];
      if (u[r] >= 0 && m[r] == INT32_MAX) {
        const int32_t w = u[r] >> 5;
        c[r] = n_dst + __ldg(prefix + w) + __popc(__ldg(bits + w) & ((1u << (u[r] & 31)) - 1u));
      }
    }
#pragma unroll
    for (int r = 0; r < kR; ++r) {
      const int64_t k = k0 + (int64_t)r * blockDim.x;
      if (k < e) {
        col_local[k] = c[r];
        if (tcnt) atomicAdd(&tcnt[c[r]], 1);
      }
    }
  }
}

// ------------------------------------------------------------------ a6: heavy rows, transpose
struct HeavyFlag {
  const int32_t* rp;
  __device__ __forceinline__ int32_t operator()(int64_t i) const {
    return (rp[i + 1] - rp[i]) > kHeavyT ? 1 : 0;
  }
};
struct NoStore {
  __device__ __forceinline__ void operator()(int64_t, int32_t, int32_t) const {}
};
// Degree class of a dst row (degree bucketing of the block, Alg. 2 l.6): min(D, kHeavyT + 1).
struct DegClass {
  const int32_t* rp;
  __device__ __forceinline__ int operator()(int64_t i) const {
    const int32_t D = rp[i + 1] - rp[i];
    return D > kHeavyT ? kHeavyT + 1 : D;
  }
};
struct EmitPerm {
  int32_t* perm;
  __device__ __forceinline__ void operator()(int64_t i, int32_t pos) const { perm[pos] = (int32_t)i; }
};

// Transposed fill: edge (i -> col_local[e]) lands at an atomic cursor of its src row.
__global__ void __launch_bounds__(256) k_tfill(const int32_t* __restrict__ rp, const int32_t* __restrict__ col_local,
                                               int64_t n, int32_t* __restrict__ cursor, int32_t* __restrict__ tcol) {
  pdl_wait();
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n; i += warps)
    for (int32_t k = rp[i] + lane; k < rp[i + 1]; k += 32) tcol[atomicAdd(&cursor[col_local[k]], 1)] = (int32_t)i;
}
// Ascending sort of the transposed rows with 2..128 entries.  t_perm lists the rows by length
// (stable partition by min(len, 129); cls_start(c) = first position of class c, read from the
// scanned partition counts), so rows are taken in bands: len 2..8 eight lanes per row, 9..16
// sixteen, 17..128 a warp with up to four entries per lane.  rank = number of smaller entries
// of the row (entries are distinct).
template <int SEG, int V>
__device__ __forceinline__ void tsort_segment(const int32_t* __restrict__ trp, int32_t* __restrict__ tcol, int32_t j,
                                              bool valid) {
  const int lane = threadIdx.x & 31, g = lane / SEG, sl = lane % SEG;
  int32_t b = 0, len = 0;
  if (valid) {
    b = trp[j];
    len = trp[j + 1] - b;
  }
  int32_t v[V];
  int rank[V];
#pragma unroll
  for (int k = 0; k < V; ++k) {
    v[k] = (sl + SEG * k < len) ? tcol[b + sl + SEG * k] : INT32_MAX;
    rank[k] = 0;
  }
  const int tmax = SEG == 32 ? len : SEG * V;      // one row per warp at SEG = 32: len is uniform
  for (int t = 0; t < tmax; ++t) {
    const int32_t x = __shfl_sync(0xffffffffu, v[t / SEG], g * SEG + (t % SEG));
#pragma unroll
    for (int k = 0; k < V; ++k) rank[k] += x < v[k] ? 1 : 0;
  }
  __syncwarp();
#pragma unroll
  for (int k = 0; k < V; ++k)
    if (sl + SEG * k < len) tcol[b + rank[k]] = v[k];
}

__global__ void __launch_bounds__(256) k_tsort_banded(const int32_t* __restrict__ perm, const int32_t* __restrict__ trp,
                                                      int32_t* __restrict__ tcol, const int32_t* __restrict__ cls_off,
                                                      int64_t ntiles) {
  pdl_wait();
  const int64_t sA = cls_off[2 * ntiles], sB = cls_off[9 * ntiles], sC = cls_off[17 * ntiles];
  const int64_t sH = cls_off[(kHeavyT + 1) * ntiles];
  const int64_t wA = (sB - sA + 3) / 4, wB = (sC - sB + 1) / 2, wC = sH - sC;
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w < wA + wB + wC; w += warps) {
    if (w < wA) {
      const int64_t p = sA + w * 4 + lane / 8;
      tsort_segment<8, 1>(trp, tcol, p < sB ? perm[p] : 0, p < sB);
    } else if (w < wA + wB) {
      const int64_t p = sB + (w - wA) * 2 + lane / 16;
      tsort_segment<16, 1>(trp, tcol, p < sC ? perm[p] : 0, p < sC);
    } else {
      const int64_t p = sC + (w - wA - wB);
      tsort_segment<32, 4>(trp, tcol, perm[p], true);
    }
  }
}
// Long transposed rows (> 128 entries): CTA per row; the row is staged in `stage` (same
// offsets as t_col), then every entry is written at its rank among the staged values.
__global__ void __launch_bounds__(256) k_tsort_heavy(const int32_t* __restrict__ perm, int64_t n,
                                                     const int32_t* __restrict__ trp,
                                                     int32_t* __restrict__ tcol, int32_t* __restrict__ stage) {
  pdl_wait();
  for (int64_t hh = blockIdx.x; hh < n; hh += gridDim.x) {
  const int32_t j = perm[n - 1 - hh];          // heavy rows: the tail of the degree-class perm
  const int32_t b = trp[j], len = trp[j + 1] - b;
  if (len <= kHeavyT) break;
  for (int32_t k = threadIdx.x; k < len; k += blockDim.x) stage[b + k] = tcol[b + k];
  __syncthreads();
  for (int32_t k = threadIdx.x; k < len; k += blockDim.x) {
    const int32_t x = stage[b + k];
    int32_t r = 0;
    for (int32_t t = 0; t < len; ++t) r += stage[b + t] < x ? 1 : 0;
    tcol[b + r] = x;
  }
  __syncthreads();
  }
}
// Long transposed rows, counting sort through a shared-memory bitmap over the dst range (the
// entries are distinct dst indices < n_dst): set the bits, then every thread emits its slice
// of words at the slice's popcount prefix.  O(len + n_dst / 32) per row.
constexpr int kBitsortMaxWords = 40 * 1024;      // 160 KB of shared memory (n_dst <= 1.31 M)
__global__ void __launch_bounds__(256) k_tsort_heavy_bits(const int32_t* __restrict__ perm, int64_t n,
                                                          const int32_t* __restrict__ trp,
                                                          int32_t* __restrict__ tcol, int32_t words) {
  pdl_wait();
  extern __shared__ uint32_t bm[];
  __shared__ int32_t sw[33];
  const int per = (words + blockDim.x - 1) / blockDim.x;
  const int w0 = min(words, (int)threadIdx.x * per), w1 = min(words, w0 + per);
  for (int64_t hh = blockIdx.x; hh < n; hh += gridDim.x) {
    const int32_t j = perm[n - 1 - hh];          // heavy rows: the tail of the degree-class perm
    const int32_t b = trp[j], len = trp[j + 1] - b;
    if (len <= kHeavyT) break;
    for (int w = threadIdx.x; w < words; w += blockDim.x) bm[w] = 0u;
    __syncthreads();
    for (int32_t k = threadIdx.x; k < len; k += blockDim.x) {
      const int32_t x = tcol[b + k];
      atomicOr(&bm[x >> 5], 1u << (x & 31));
    }
    __syncthreads();
    int32_t cnt = 0;
    for (int w = w0; w < w1; ++w) cnt += __popc(bm[w]);
    int32_t total;
    int32_t r = block_exclusive_sum<256>(cnt, sw, &total);
    for (int w = w0; w < w1; ++w) {
      uint32_t m = bm[w];
      while (m) {
        const int bit = __ffs(m) - 1;
        m &= m - 1;
        tcol[b + r++] = w * 32 + bit;
      }
    }
    __syncthreads();
  }
}
// ------------------------------------------------------------------ host side
static buffalo_status d2h_i32(const int32_t* d, int32_t* h, cudaStream_t s) {
  BF_CUDA(cudaMemcpyAsync(h, d, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  return BUFFALO_OK;
}

int64_t build_frame_bytes(int64_t n_dst, int64_t e, int layer, bool sizes_only, bool t1) {
  const int64_t pc = part_count_elems(e);
  if (sizes_only) {
    const int64_t scan_len = std::max<int64_t>(n_dst + e + 1, pc + 1);
    return R(64) + R(4 * scan_ws_elems(scan_len)) + R(4 * e);
  }
  const int64_t pne = part_count_elems(n_dst + e);   // bounds the partitions of n_dst, n_src, e
  const int64_t scan_len = std::max<int64_t>(n_dst + e + 1, pne + 1);
  int64_t fr = R(64) + R(4 * scan_ws_elems(scan_len)) + R(4 * (pne + 1));
  if (layer >= 2) fr += R(4 * e) + R(4 * (n_dst + e));        // col_global + transposed-fill cursors
  else if (t1) fr += R(4 * (n_dst + e));                       // block 1: cursors (col_global persists)
  return fr;
}

buffalo_status build_layer(const buffalo_graph* g, const int32_t* dst, int64_t n_dst, int32_t f,
                           uint32_t hop, uint64_t seed, int layer, bool sizes_only, Arena& A,
                           buffalo_block* blk, cudaStream_t s, const int64_t* known, bool t1,
                           const int32_t* cache, bool dst_perm) {
  memset(blk, 0, sizeof(*blk));
  blk->n_dst = n_dst;
  blk->fanout = f;
  int32_t* rp = (int32_t*)A.take(4 * (n_dst + 1));
  int32_t* perm = sizes_only ? nullptr : (int32_t*)A.take(4 * n_dst);
  // frame 1: totals + scan workspace for the count scan and the heavy compaction
  char* fr = A.push_frame(R(64) + R(4 * scan_ws_elems(n_dst + 1)));
  if (A.overflow) return BUFFALO_ERR_CAPACITY;
  int32_t* totals = (int32_t*)fr;
  int32_t* ws = (int32_t*)(fr + R(64));
  BF_CHECK(device_scan(LoadDeg{dst, g->row_ptr, f}, StoreArr{rp}, n_dst, ws, rp + n_dst, s));
  int64_t e = 0, nh = -1;
  if (known) {
    e = known[0];                                                  // exact sizes from the plan: no sync
  } else {
    int32_t e32 = 0, nh32 = 0;
    if (!sizes_only) {
      BF_CHECK(device_count(HeavyFlag{rp}, n_dst, totals, s));
      BF_CHECK(d2h_i32(totals, &nh32, s));
    }
    BF_CHECK(d2h_i32(rp + n_dst, &e32, s));
    BF_CUDA(cudaStreamSynchronize(s));                             // sync 1: e_l, n_heavy
    e = e32;
    nh = nh32;
  }
  blk->n_edges = e;
  blk->row_ptr = rp;
  if (!dst_perm) {                 // sampled block of the mean model: no row past the fanout
    perm = nullptr;
    nh = 0;
  }
  blk->cls_perm = perm;
  blk->n_heavy = nh;
  blk->heavy = (perm && nh >= 0) ? perm + (n_dst - nh) : nullptr;

  // frame 2
  const int64_t pc = sizes_only ? part_count_elems(e) : part_count_elems(n_dst + e);
  const int64_t scan_len = std::max<int64_t>(n_dst + e + 1, pc + 1);
  int32_t* col_local = (!sizes_only) ? (int32_t*)A.take(4 * e) : nullptr;
  int32_t* colg_persist = (!sizes_only && layer == 1) ? (int32_t*)A.take(4 * e) : nullptr;
  fr = A.push_frame(build_frame_bytes(n_dst, e, layer, sizes_only, t1));
  if (A.overflow) return BUFFALO_ERR_CAPACITY;
  totals = (int32_t*)fr;
  char* q = fr + R(64);
  ws = (int32_t*)q; q += R(4 * scan_ws_elems(scan_len));
  int32_t* colg = colg_persist;
  if (!colg) { colg = (int32_t*)q; q += R(4 * e); }
  int32_t* counts = nullptr;
  if (!sizes_only) {
    counts = (int32_t*)q;
    q += R(4 * (pc + 1));
    // degree classes of the dst rows: stable counting sort by min(D, kHeavyT + 1)
    if (perm) BF_CHECK(stable_partition(DegClass{rp}, EmitPerm{perm}, n_dst, counts, ws, s));
  }
  // relabel (R3): dst prefix, then the other neighbours in ascending global id; the dst enter
  // the node map first so that the fill marks the other neighbours in the bitmap as it writes
  const GraphWs gw = graph_ws(g);
  if (n_dst > 0) {
    launch_pdl(k_set_map, dim3(grid_for(n_dst, 256)), dim3(256), 0, s, dst, n_dst, g->node_map);
    BF_LAUNCHED("k_set_map");
  }
  const MarkCtx mk{g->node_map, gw.bits, col_local};
  if (n_dst > 0 && cache && f > 0) {                             // rows sampled by the scheduler
    const int seg = sample_seg(f), G = 32 / seg;
    const int grid = grid_for(ceil_div(n_dst, G) * 32, 256, 16);
    if (seg == 8) launch_pdl(k_cache_fill<8>, dim3(grid), dim3(256), 0, s, dst, n_dst, cache, f, (const int32_t*)rp, colg, e, mk);
    else if (seg == 16) launch_pdl(k_cache_fill<16>, dim3(grid), dim3(256), 0, s, dst, n_dst, cache, f, (const int32_t*)rp, colg, e, mk);
    else launch_pdl(k_cache_fill<32>, dim3(grid), dim3(256), 0, s, dst, n_dst, cache, f, (const int32_t*)rp, colg, e, mk);
    BF_LAUNCHED("k_cache_fill");
  } else if (n_dst > 0) {
    launch_sample_fill(sample_seg(f), n_dst, s, dst, n_dst, g->row_ptr, g->col, f, hop, seed, (const int32_t*)rp,
                       colg, e, mk);
    BF_LAUNCHED("k_sample_fill");
  }
  int64_t n_src = 0;
  if (known) {
    n_src = known[1];
  } else {
    BF_CHECK(device_count(PopcWord{gw.bits}, gw.words, totals, s));
    int32_t nn32 = 0;
    BF_CHECK(d2h_i32(totals, &nn32, s));
    BF_CUDA(cudaStreamSynchronize(s));                             // sync 2: n_{l-1}
    n_src = n_dst + nn32;
  }
  // from here on the graph workspace is dirty: an early return must restore it
  auto restore_ws = [&]() -> buffalo_status {
    if (n_dst > 0) {
      launch_pdl(k_reset_map, dim3(grid_for(n_dst, 256)), dim3(256), 0, s, dst, n_dst, g->node_map);
      BF_LAUNCHED("k_reset_map");
    }
    BF_CUDA(cudaMemsetAsync(gw.bits, 0, sizeof(uint32_t) * gw.words, s));
    return BUFFALO_OK;
  };
  int32_t* src = (int32_t*)A.take(4 * n_src);
  if (A.overflow) {
    BF_CHECK(restore_ws());
    return BUFFALO_ERR_CAPACITY;
  }
  if (n_dst > 0) BF_CUDA(cudaMemcpyAsync(src, dst, sizeof(int32_t) * n_dst, cudaMemcpyDeviceToDevice, s));
  BF_CHECK(device_scan(PopcWord{gw.bits}, StorePrefix{gw.prefix}, gw.words, gw.scan_ws, totals + 2, s));
  launch_pdl(k_emit_bits, dim3(grid_for(gw.words, 256)), dim3(256), 0, s, gw.bits, gw.prefix, gw.words, src + n_dst, n_src - n_dst);
  BF_LAUNCHED("k_emit_bits");
  blk->n_src = n_src;
  blk->src_global = src;
  blk->col_global = colg_persist;
  const bool transpose = !sizes_only && (layer >= 2 || t1);
  int32_t *trp = nullptr, *tcol = nullptr, *tperm = nullptr;
  if (transpose) {
    trp = (int32_t*)A.take(4 * (n_src + 1));
    tcol = (int32_t*)A.take(4 * e);
    tperm = (int32_t*)A.take(4 * n_src);
    if (A.overflow) {
      BF_CHECK(restore_ws());
      return BUFFALO_ERR_CAPACITY;
    }
    BF_CUDA(cudaMemsetAsync(trp, 0, sizeof(int32_t) * (n_src + 1), s));
  }
  if (!sizes_only) {
    if (e > 0) {
      launch_pdl(k_col_local, dim3(grid_for(e, 256)), dim3(256), 0, s, colg, e, g->node_map, gw.bits, gw.prefix, (int32_t)n_dst,
                                                   col_local, trp);
      BF_LAUNCHED("k_col_local");
    }
    blk->col_local = col_local;
  }
  BF_CHECK(restore_ws());
  blk->n_heavy_t = -1;
  if (transpose) {
    // transposed block: t_row_ptr from the counts taken in k_col_local; t_col by an
    // atomic-cursor fill followed by an ascending sort of every transposed row (entries are
    // distinct dst indices, so the sorted row equals the stable order of the dst-ordered
    // edges); degree classes of the src rows.
    int32_t* cursor = (int32_t*)q; q += R(4 * (n_dst + e));
    BF_CHECK(scan_inplace(trp, n_src, ws, s));
    BF_CHECK(stable_partition(DegClass{trp}, EmitPerm{tperm}, n_src, counts, ws, s));
    int64_t nht = -1;
    if (!known) {
      BF_CHECK(device_count(HeavyFlag{trp}, n_src, totals + 1, s));
      int32_t nht32 = 0;
      BF_CHECK(d2h_i32(totals + 1, &nht32, s));
      BF_CUDA(cudaStreamSynchronize(s));                           // n_heavy_t (informational)
      nht = nht32;
    }
    if (e > 0) {
      BF_CUDA(cudaMemcpyAsync(cursor, trp, sizeof(int32_t) * n_src, cudaMemcpyDeviceToDevice, s));
      launch_pdl(k_tfill, dim3(grid_for(n_dst * 32, 256, 16)), dim3(256), 0, s, rp, col_local, n_dst, cursor, tcol);
      BF_LAUNCHED("k_tfill");
      if (n_src > 0) {
        launch_pdl(k_tsort_banded, dim3(grid_for(n_src * 8, 256, 16)), dim3(256), 0, s, tperm, trp, tcol, counts, part_tiles(n_src));
        BF_LAUNCHED("k_tsort_banded");
      }
      const int hg = heavy_tail_grid(nht, e);
      if (hg > 0) {
        const int64_t words = ceil_div(n_dst, 32);
        if (words <= kBitsortMaxWords) {
          BF_CHECK(set_max_smem_once<k_tsort_heavy_bits>(kBitsortMaxWords * 4));
          launch_pdl(k_tsort_heavy_bits, dim3(hg), dim3(256), words * 4, s, tperm, n_src, trp, tcol, (int32_t)words);
          BF_LAUNCHED("k_tsort_heavy_bits");
        } else {
          launch_pdl(k_tsort_heavy, dim3(hg), dim3(256), 0, s, tperm, n_src, trp, tcol, cursor);
          BF_LAUNCHED("k_tsort_heavy");
        }
      }
    }
    blk->t_row_ptr = trp;
    blk->t_col = tcol;
    blk->t_perm = tperm;
    blk->n_heavy_t = nht;
  }
  A.pop_frame();
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ input validation
// Id lists (seeds, group seeds; Alg. 3's input G is a set of nodes): every id
// in [0, N) and none twice.  Duplicates are found through the graph workspace's node bitmap,
// which k_clear_ids leaves all-zero again (its between-calls invariant).
__global__ void k_check_ids(const int32_t* __restrict__ ids, int64_t n, int64_t N, uint32_t* __restrict__ bits,
                            int32_t* __restrict__ err) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = ids[i];
    if (v < 0 || v >= N) {
      atomicOr(err, 1);
      continue;
    }
    const uint32_t m = 1u << (v & 31);
    if (atomicOr(bits + (v >> 5), m) & m) atomicOr(err, 2);
  }
}
__global__ void k_clear_ids(const int32_t* __restrict__ ids, int64_t n, int64_t N, uint32_t* __restrict__ bits) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t v = ids[i];
    if (v >= 0 && v < N) bits[v >> 5] = 0u;
  }
}
buffalo_status check_ids(const buffalo_graph* g, const int32_t* ids, int64_t n, int32_t* err_dev, cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  const GraphWs gw = graph_ws(g);
  k_check_ids<<<grid_for(n, 256), 256, 0, s>>>(ids, n, g->num_nodes, gw.bits, err_dev);
  BF_LAUNCHED("k_check_ids");
  k_clear_ids<<<grid_for(n, 256), 256, 0, s>>>(ids, n, g->num_nodes, gw.bits);
  BF_LAUNCHED("k_clear_ids");
  return BUFFALO_OK;
}
buffalo_status ids_error(int32_t err, const char* what) {
  if (err & 1) {
    set_error("%s: a node id is outside [0, num_nodes)", what);
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (err & 2) {
    set_error("%s: a node id occurs twice (the batch is a set of nodes)", what);
    return BUFFALO_ERR_INVALID_ARG;
  }
  return BUFFALO_OK;
}

// The graph's CSR (include/buffalo.h: rows sorted ascending, simple, symmetric): a warp per
// node walks its row.  Error bits: 1 row_ptr not a monotone offset array from 0 to nnz, 2 an
// id outside [0, N), 4 a row not strictly increasing (unsorted or duplicate entries), 8 a self
// loop, 16 an edge (v, c) without (c, v) (checked only with `sym`, by binary search of row c).
__global__ void __launch_bounds__(256) k_validate_csr(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                      int64_t N, int64_t nnz, int sym, int32_t* __restrict__ err) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  if (blockIdx.x == 0 && threadIdx.x == 0 && (rp[0] != 0 || rp[N] != nnz)) atomicOr(err, 1);
  for (int64_t v = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; v < N; v += warps) {
    const int64_t b = rp[v], e = rp[v + 1];
    if (b < 0 || e < b || e > nnz) {
      if (lane == 0) atomicOr(err, 1);
      continue;
    }
    int bad = 0;
    for (int64_t k = b + lane; k < e; k += 32) {
      const int32_t c = col[k];
      if (c < 0 || c >= N) {
        bad |= 2;
        continue;
      }
      if (c == v) bad |= 8;
      if (k > b && col[k - 1] >= c) bad |= 4;
      if (sym) {
        int64_t lo = rp[c], hi = rp[c + 1];
        if (lo < 0 || hi < lo || hi > nnz) {
          bad |= 1;
          continue;
        }
        while (lo < hi) {                               // first entry >= v in row c
          const int64_t mid = (lo + hi) >> 1;
          if (col[mid] < v) lo = mid + 1; else hi = mid;
        }
        if (lo == rp[c + 1] || col[lo] != v) bad |= 16;
      }
    }
    bad = __reduce_or_sync(0xffffffffu, bad);
    if (lane == 0 && bad) atomicOr(err, bad);
  }
}

buffalo_status validate_graph(const buffalo_graph* g, int sym, cudaStream_t s) {
  const GraphWs gw = graph_ws(g);
  int32_t* err_dev = gw.scan_ws;                 // scratch between calls
  BF_CUDA(cudaMemsetAsync(err_dev, 0, sizeof(int32_t), s));
  k_validate_csr<<<grid_for(g->num_nodes * 32, 256), 256, 0, s>>>(g->row_ptr, g->col, g->num_nodes, g->nnz, sym,
                                                                  err_dev);
  BF_LAUNCHED("k_validate_csr");
  int32_t err = 0;
  BF_CUDA(cudaMemcpyAsync(&err, err_dev, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  BF_CUDA(cudaStreamSynchronize(s));
  static const char* what[5] = {"row_ptr is not a monotone offset array from 0 to nnz",
                                "a column id is outside [0, num_nodes)",
                                "a row is not strictly increasing (unsorted or duplicate entries)",
                                "a self loop", "the graph is not symmetric"};
  for (int k = 0; k < 5; ++k)
    if (err & (1 << k)) {
      set_error("graph_validate: %s", what[k]);
      return BUFFALO_ERR_INVALID_ARG;
    }
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ a1: seed bucketing
__global__ void k_seed_bucket(const int32_t* __restrict__ seeds, int64_t n, const int64_t* __restrict__ grow,
                              int64_t N, int32_t fL, int32_t F, uint8_t* __restrict__ bucket) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    int64_t v = seeds[i];
    if (v < 0 || v >= N) { bucket[i] = 0; continue; }     // rejected by k_check_ids (no read)
    int64_t deg = grow[v + 1] - grow[v];
    int64_t D = (fL > 0 && deg > fL) ? fL : deg;
    bucket[i] = (uint8_t)(D < F ? D : F);
  }
}
struct BucketKey {
  const uint8_t* b;
  __device__ __forceinline__ int operator()(int64_t i) const { return b[i]; }
};
struct BucketEmit {
  const int32_t* seeds;
  int32_t* order;
  int32_t* sorted_ids;
  __device__ __forceinline__ void operator()(int64_t i, int32_t pos) const {
    order[pos] = (int32_t)i;
    sorted_ids[pos] = seeds[i];
  }
};
// starts[b] = exclusive offset of bin b (b = 0..nbins), read from the scanned partition counts.
__global__ void k_bin_starts(const int32_t* counts, int64_t ntiles, int nbins, int32_t total, int32_t* starts) {
  int b = threadIdx.x;
  if (b < nbins) starts[b] = counts[(int64_t)b * ntiles];
  if (b == nbins) starts[b] = total;
}

buffalo_status seed_bucketing(const buffalo_graph* g, const int32_t* seeds, int64_t n, int32_t fL,
                              int32_t F, uint8_t* bucket, int32_t* order, int32_t* sorted_ids,
                              int32_t* counts, int32_t* ws, int32_t* starts_dev, int64_t* hist_h,
                              cudaStream_t s) {
  if (n <= 0) {
    for (int b = 0; b <= F; ++b) hist_h[b] = 0;
    return BUFFALO_OK;
  }
  // input validation (include/buffalo.h): ids in [0, N), no id twice; the error word is read
  // back with the bucket starts (one synchronisation)
  int32_t* err_dev = starts_dev + 257;
  BF_CUDA(cudaMemsetAsync(err_dev, 0, sizeof(int32_t), s));
  BF_CHECK(check_ids(g, seeds, n, err_dev, s));
  k_seed_bucket<<<grid_for(n, 256), 256, 0, s>>>(seeds, n, g->row_ptr, g->num_nodes, fL, F, bucket);
  BF_LAUNCHED("k_seed_bucket");
  BF_CHECK(stable_partition(BucketKey{bucket}, BucketEmit{seeds, order, sorted_ids}, n, counts, ws, s));
  k_bin_starts<<<1, 256, 0, s>>>(counts, part_tiles(n), F + 1, (int32_t)n, starts_dev);
  BF_LAUNCHED("k_bin_starts");
  int32_t st[258];
  BF_CUDA(cudaMemcpyAsync(st, starts_dev, sizeof(int32_t) * (F + 2), cudaMemcpyDeviceToHost, s));
  BF_CUDA(cudaMemcpyAsync(st + 257, err_dev, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
  BF_CUDA(cudaStreamSynchronize(s));
  BF_CHECK(ids_error(st[257], "seeds"));
  for (int b = 0; b <= F; ++b) hist_h[b] = st[b + 1] - st[b];
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ a2: item statistics
// Block sizes of up to 256 items (seed ranges, possibly overlapping) at once, by propagating
// item bitmasks top-down: a node's mask at layer l-1 is the OR of the masks of the layer-l
// nodes that have it as a dst (prefix) or a sampled neighbour.  Because a node's sample depends
// only on (seed, node, hop) (R2), item k's node set at every layer is exactly the one of its own
// blocks, so n_l(k) = #nodes with bit k, e_l(k) = sum of D over them — the sizes build_layer
// would give.  A mask is W 64-bit words per node (W = 1, 2 or 4 by the item count); the nodes
// of each layer are collected through the graph workspace's node bitmap (ascending ids).

// Seed masks: position i (of the union range starting at base) gets the bit of every item
// [start_k, end_k) that contains it (items of different K candidates overlap).
template <int W>
__global__ void __launch_bounds__(256) k_mask_seed(const int32_t* __restrict__ ids, int64_t base, int64_t n,
                                                   const int64_t* __restrict__ item_se, int nitems,
                                                   unsigned long long* __restrict__ m, int32_t* __restrict__ act) {
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int64_t pos = base + i;
    unsigned long long mask[W];
#pragma unroll
    for (int w = 0; w < W; ++w) mask[w] = 0;
    for (int k = 0; k < nitems; ++k)
      if (pos >= item_se[2 * k] && pos < item_se[2 * k + 1]) mask[k >> 6] |= 1ull << (k & 63);
    const int32_t v = ids[pos];
#pragma unroll
    for (int w = 0; w < W; ++w) m[(int64_t)v * W + w] = mask[w];
    act[i] = v;
  }
}

// Per-item counters of a warp's nodes: lane k accumulates items k + 32 j (j < 2W) in registers;
// the block's sums are flushed once at the end.
template <int W>
struct ItemCounters {
  uint32_t n[2 * W];
  unsigned long long e[2 * W];
  __device__ ItemCounters() {
#pragma unroll
    for (int j = 0; j < 2 * W; ++j) { n[j] = 0; e[j] = 0; }
  }
};

template <int W>
__device__ __forceinline__ void flush_item_counters(const ItemCounters<W>& c, unsigned long long* __restrict__ gn,
                                                    unsigned long long* __restrict__ ge,
                                                    unsigned long long* sn, unsigned long long* se) {
  const int lane = threadIdx.x & 31;
#pragma unroll
  for (int j = 0; j < 2 * W; ++j) {
    if (c.n[j]) atomicAdd(&sn[lane + 32 * j], (unsigned long long)c.n[j]);
    if (ge && c.e[j]) atomicAdd(&se[lane + 32 * j], c.e[j]);
  }
  __syncthreads();
  for (int k = threadIdx.x; k < 64 * W; k += blockDim.x) {
    if (sn[k]) atomicAdd(&gn[k], sn[k]);
    if (ge && se[k]) atomicAdd(&ge[k], se[k]);
  }
}

// ORs the nonzero words of mask into node u's mask and marks u in the layer's node bitmap.
template <int W>
__device__ __forceinline__ void mask_or(unsigned long long* __restrict__ m_out, uint32_t* __restrict__ bits, int32_t u,
                                        const unsigned long long (&mask)[W]) {
#pragma unroll
  for (int w = 0; w < W; ++w)
    if (mask[w]) atomicOr(&m_out[(int64_t)u * W + w], mask[w]);
  const uint32_t b = 1u << (u & 31);
  if (!(bits[u >> 5] & b)) atomicOr(&bits[u >> 5], b);
}

// One layer: 32/SEG active nodes of layer l per warp; accumulates n_l, e_l per item and ORs
// each node's mask into layer l-1 for the node itself and its sampled neighbours.
template <int SEG, int W>
__global__ void __launch_bounds__(256, (W >= 4 ? 4 : 6)) k_mask_layer(const int32_t* __restrict__ act, int64_t n_act,
                                                    const unsigned long long* __restrict__ m_in,
                                                    unsigned long long* __restrict__ m_out, uint32_t* __restrict__ bits,
                                                    const int64_t* __restrict__ grow, const int32_t* __restrict__ gcol,
                                                    int32_t f, uint32_t hop, uint64_t seed,
                                                    unsigned long long* __restrict__ gn, unsigned long long* __restrict__ ge,
                                                    int32_t* __restrict__ cache, int cache_read) {
  constexpr int G = 32 / SEG;
  __shared__ unsigned long long sn[64 * W], se[64 * W];
  for (int k = threadIdx.x; k < 64 * W; k += blockDim.x) { sn[k] = 0; se[k] = 0; }
  __syncthreads();
  const int lane = threadIdx.x & 31, g = lane / SEG;
  ItemCounters<W> cnt;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * G < n_act; w += warps) {
    const int64_t slot = w * G + g;
    int32_t v = 0;
    unsigned long long mask[W];
#pragma unroll
    for (int q = 0; q < W; ++q) mask[q] = 0;
    int32_t D = 0;
    if (slot < n_act) {
      v = act[slot];
#pragma unroll
      for (int q = 0; q < W; ++q) mask[q] = m_in[(int64_t)v * W + q];
      const int64_t deg = grow[v + 1] - grow[v];
      D = (int32_t)((f > 0 && deg > f) ? f : deg);
    }
#pragma unroll
    for (int q = 0; q < G; ++q) {
      const uint32_t Dq = (uint32_t)__shfl_sync(0xffffffffu, D, q * SEG);
#pragma unroll
      for (int j = 0; j < 2 * W; ++j) {
        const unsigned long long mq = __shfl_sync(0xffffffffu, mask[j >> 1], q * SEG);
        if ((mq >> (lane + 32 * (j & 1))) & 1ull) { cnt.n[j] += 1; cnt.e[j] += Dq; }
      }
    }
    if (slot < n_act && (lane % SEG) == 0) mask_or<W>(m_out, bits, v, mask);
    if (cache_read) {                                            // rows cached by the first pass
      if (slot < n_act && (lane % SEG) < D) {
        const int32_t u = cache[(int64_t)v * f + (lane % SEG)];
        mask_or<W>(m_out, bits, u, mask);
      }
    } else {
      sample_warp_rows<SEG>(w, n_act, DstRows{act}, grow, gcol, f, hop, seed, [&](int64_t s_, int32_t k, int32_t u) {
        if (cache) cache[(int64_t)act[s_] * f + k] = u;         // sample cache for the build (f > 0)
        unsigned long long ms[W];
#pragma unroll
        for (int q = 0; q < W; ++q) ms[q] = m_in[(int64_t)act[s_] * W + q];
        mask_or<W>(m_out, bits, u, ms);
      });
    }
  }
  flush_item_counters<W>(cnt, gn, ge, sn, se);
}

// Clears the masks of the active list; with gn, first counts per item how many active nodes
// carry its bit (one ballot per item bit, counted in registers).
template <int W>
__global__ void __launch_bounds__(256) k_mask_count(const int32_t* __restrict__ act, int64_t n_act,
                                                    unsigned long long* __restrict__ m,
                                                    unsigned long long* __restrict__ gn) {
  __shared__ unsigned long long sn[64 * W];
  for (int k = threadIdx.x; k < 64 * W; k += blockDim.x) sn[k] = 0;
  __syncthreads();
  const int lane = threadIdx.x & 31;
  ItemCounters<W> cnt;
  // Each thread adds its nodes' masks into bit-sliced counters (plane p holds bit p of the count
  // of every item: a ripple-carry add of P word operations per node); every 2^P - 1 nodes, and
  // at the end, the planes are reduced over the warp with one ballot per (plane, item bit).  The
  // loop trip count is warp-uniform (threads past n_act add zero masks), so the flushes are too.
  constexpr int P = W >= 4 ? 5 : 8;
  constexpr int kFlush = (1 << P) - 1;
  unsigned long long plane[P][W];
#pragma unroll
  for (int p = 0; p < P; ++p)
#pragma unroll
    for (int q = 0; q < W; ++q) plane[p][q] = 0ull;
  int since = 0;
  auto flush = [&]() {
#pragma unroll
    for (int q = 0; q < W; ++q)
#pragma unroll
      for (int h = 0; h < 2; ++h)
#pragma unroll
        for (int p = 0; p < P; ++p) {
          const unsigned word = (unsigned)(plane[p][q] >> (32 * h));
          if (__any_sync(0xffffffffu, word != 0u)) {
#pragma unroll
            for (int k = 0; k < 32; ++k) {
              const unsigned b = __ballot_sync(0xffffffffu, (word >> k) & 1u);
              if (lane == k) cnt.n[2 * q + h] += (uint32_t)__popc(b) << p;
            }
          }
        }
#pragma unroll
    for (int p = 0; p < P; ++p)
#pragma unroll
      for (int q = 0; q < W; ++q) plane[p][q] = 0ull;
  };
  // U nodes per thread and iteration (coalesced act loads, U independent mask loads in flight:
  // one dependent act -> mask chain per node measured ~10 us per iteration at papers scale)
  constexpr int U = W >= 4 ? 2 : 4;
  const int64_t stride = (int64_t)gridDim.x * blockDim.x * U;
  for (int64_t i0 = blockIdx.x * (int64_t)blockDim.x * U; i0 < n_act; i0 += stride) {
    int32_t v[U];
#pragma unroll
    for (int u = 0; u < U; ++u) {
      const int64_t i = i0 + threadIdx.x + (int64_t)u * blockDim.x;
      v[u] = i < n_act ? __ldg(act + i) : -1;
    }
    unsigned long long mask[U][W];
#pragma unroll
    for (int u = 0; u < U; ++u)
#pragma unroll
      for (int q = 0; q < W; ++q) mask[u][q] = v[u] >= 0 ? m[(int64_t)v[u] * W + q] : 0ull;
#pragma unroll
    for (int u = 0; u < U; ++u)
      if (v[u] >= 0) {
#pragma unroll
        for (int q = 0; q < W; ++q) m[(int64_t)v[u] * W + q] = 0ull;
      }
    if (gn) {
#pragma unroll
      for (int u = 0; u < U; ++u)
#pragma unroll
        for (int q = 0; q < W; ++q) {
          unsigned long long c = mask[u][q];
#pragma unroll
          for (int p = 0; p < P; ++p) {
            const unsigned long long t = plane[p][q] & c;
            plane[p][q] ^= c;
            c = t;
          }
        }
      since += U;
      if (since > kFlush - U) {
        flush();
        since = 0;
      }
    }
  }
  if (gn) {
    flush();
    flush_item_counters<W>(cnt, gn, nullptr, sn, nullptr);
  }
}

constexpr int kMaskMaxItems = 256;
constexpr int kMaskMaxW = kMaskMaxItems / 64;

int64_t mask_stats_bytes(int64_t N, int L) {
  return 2 * R(8 * kMaskMaxW * N) + 2 * R(4 * N) + R(8 * kMaskMaxItems * (2 * L + 1)) + R(64) +
         R(16 * kMaskMaxItems);
}

template <int W>
static buffalo_status mask_stats_w(const buffalo_graph* g, const int32_t* sorted_ids, int64_t lo_pos, int64_t n_seed,
                                   const int64_t* se, int nitems, const buffalo_sampler* sp, int L,
                                   unsigned long long* const* m, int32_t* const* act, unsigned long long* accn,
                                   unsigned long long* acce, cudaStream_t s, int cache_mode) {
  const GraphWs gw = graph_ws(g);
  if (n_seed > 0) {
    k_mask_seed<W><<<grid_for(n_seed, 256), 256, 0, s>>>(sorted_ids, lo_pos, n_seed, se, nitems, m[0], act[0]);
    BF_LAUNCHED("k_mask_seed");
  }
  int64_t n_act = n_seed;
  int cur = 0;
  int32_t* total = gw.prefix + gw.words;          // the prefix array's spare last element
  for (int l = L; l >= 1; --l) {
    int32_t na = 0;
    if (n_act > 0) {
      const int32_t fl = sp->fanout[l - 1];
      int32_t* cache = (fl > 0 && cache_mode > 0) ? sp->cache[l - 1] : nullptr;
      const int cread = cache && cache_mode == 2;
      const int seg = sample_seg(fl);
      const int grid = grid_for(ceil_div(n_act, 32 / seg) * 32, 256, 16);
      const uint32_t hop = (uint32_t)(L - l + 1);
      if (seg == 8)
        k_mask_layer<8, W><<<grid, 256, 0, s>>>(act[cur], n_act, m[cur], m[cur ^ 1], gw.bits, g->row_ptr, g->col, fl,
                                               hop, sp->seed, accn + 64 * W * l, acce + 64 * W * (l - 1), cache, cread);
      else if (seg == 16)
        k_mask_layer<16, W><<<grid, 256, 0, s>>>(act[cur], n_act, m[cur], m[cur ^ 1], gw.bits, g->row_ptr, g->col, fl,
                                                hop, sp->seed, accn + 64 * W * l, acce + 64 * W * (l - 1), cache, cread);
      else
        k_mask_layer<32, W><<<grid, 256, 0, s>>>(act[cur], n_act, m[cur], m[cur ^ 1], gw.bits, g->row_ptr, g->col, fl,
                                                hop, sp->seed, accn + 64 * W * l, acce + 64 * W * (l - 1), cache, cread);
      BF_LAUNCHED("k_mask_layer");
      // masks of layer l are no longer needed: clear them for reuse by layer l-2
      k_mask_count<W><<<grid_for(n_act, 256), 256, 0, s>>>(act[cur], n_act, m[cur], nullptr);
      BF_LAUNCHED("k_mask_count");
      // layer l-1's nodes, ascending: popcount scan of the node bitmap, emit, clear
      BF_CHECK(device_scan(PopcWord{gw.bits}, StorePrefix{gw.prefix}, gw.words, gw.scan_ws, total, s));
      k_emit_bits<<<grid_for(gw.words, 256), 256, 0, s>>>(gw.bits, gw.prefix, gw.words, act[cur ^ 1], g->num_nodes);
      BF_LAUNCHED("k_emit_bits");
      BF_CUDA(cudaMemsetAsync(gw.bits, 0, sizeof(uint32_t) * gw.words, s));
      BF_CUDA(cudaMemcpyAsync(&na, total, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
      BF_CUDA(cudaStreamSynchronize(s));
    }
    n_act = na;
    cur ^= 1;
  }
  if (n_act > 0) {
    k_mask_count<W><<<grid_for(n_act, 256), 256, 0, s>>>(act[cur], n_act, m[cur], accn);
    BF_LAUNCHED("k_mask_count");
  }
  return BUFFALO_OK;
}

buffalo_status mask_stats(const buffalo_graph* g, const int32_t* sorted_ids, const int64_t* item_start_h,
                          const int64_t* item_count_h, int nitems, const buffalo_sampler* sp, int L, char* ws,
                          int64_t ws_bytes,
                          bool masks_clean, int64_t (*n_h)[BUFFALO_MAX_LAYERS + 1],
                          int64_t (*e_h)[BUFFALO_MAX_LAYERS], cudaStream_t s, int cache_mode) {
  const int64_t N = g->num_nodes;
  if (ws_bytes < mask_stats_bytes(N, L)) {
    set_error("bucketize workspace too small for the item statistics");
    return BUFFALO_ERR_CAPACITY;
  }
  if (nitems < 1 || nitems > kMaskMaxItems) {
    set_error("mask_stats: %d items (1..%d)", nitems, kMaskMaxItems);
    return BUFFALO_ERR_INVALID_ARG;
  }
  const int W = nitems <= 64 ? 1 : nitems <= 128 ? 2 : 4;
  char* q = ws;
  unsigned long long* m[2] = {(unsigned long long*)q, (unsigned long long*)(q + R(8 * kMaskMaxW * N))};
  q += 2 * R(8 * kMaskMaxW * N);
  int32_t* act[2] = {(int32_t*)q, (int32_t*)(q + R(4 * N))};
  q += 2 * R(4 * N);
  unsigned long long* acc = (unsigned long long*)q; q += R(8 * kMaskMaxItems * (2 * L + 1));
  q += R(64);
  int64_t* se = (int64_t*)q;
  if (!masks_clean) {
    BF_CUDA(cudaMemsetAsync(m[0], 0, 2 * R(8 * kMaskMaxW * N), s));
  }
  const int stride = 64 * W;                      // items per accumulator row
  BF_CUDA(cudaMemsetAsync(acc, 0, sizeof(unsigned long long) * stride * (2 * L + 1), s));
  int64_t se_h[2 * kMaskMaxItems];
  int64_t lo_pos = INT64_MAX, hi_pos = 0;
  for (int k = 0; k < nitems; ++k) {
    se_h[2 * k] = item_start_h[k];
    se_h[2 * k + 1] = item_start_h[k] + item_count_h[k];
    if (item_count_h[k] > 0) {
      lo_pos = std::min(lo_pos, se_h[2 * k]);
      hi_pos = std::max(hi_pos, se_h[2 * k + 1]);
    }
  }
  if (lo_pos > hi_pos) lo_pos = hi_pos = 0;
  BF_CUDA(cudaMemcpyAsync(se, se_h, sizeof(int64_t) * 2 * nitems, cudaMemcpyHostToDevice, s));
  const int64_t n_seed = hi_pos - lo_pos;
  // acc layout: n[l] at acc + stride*l (l = 0..L), e[l-1] at acc + stride*(L+1) + stride*(l-1)
  unsigned long long* accn = acc;
  unsigned long long* acce = acc + stride * (L + 1);
  if (W == 1)
    BF_CHECK(mask_stats_w<1>(g, sorted_ids, lo_pos, n_seed, se, nitems, sp, L, m, act, accn, acce, s, cache_mode));
  else if (W == 2)
    BF_CHECK(mask_stats_w<2>(g, sorted_ids, lo_pos, n_seed, se, nitems, sp, L, m, act, accn, acce, s, cache_mode));
  else
    BF_CHECK(mask_stats_w<4>(g, sorted_ids, lo_pos, n_seed, se, nitems, sp, L, m, act, accn, acce, s, cache_mode));
  static thread_local unsigned long long host[kMaskMaxItems * (2 * BUFFALO_MAX_LAYERS + 1)];
  BF_CUDA(cudaMemcpyAsync(host, acc, sizeof(unsigned long long) * stride * (2 * L + 1), cudaMemcpyDeviceToHost, s));
  BF_CUDA(cudaStreamSynchronize(s));
  for (int k = 0; k < nitems; ++k) {
    for (int l = 0; l <= L; ++l) n_h[k][l] = (int64_t)host[stride * l + k];
    for (int l = 1; l <= L; ++l) e_h[k][l - 1] = (int64_t)host[stride * (L + 1) + stride * (l - 1) + k];
  }
  return BUFFALO_OK;
}

}  // namespace buffalo
