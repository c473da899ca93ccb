// primitives.cuh — device-wide scan and stable bin partition used by block generation and
// bucketing.  Functor-driven so that flags/keys are computed on the fly (no flag arrays).
#pragma once
#include "common.cuh"

namespace buffalo {

constexpr int kScanThreads = 512;
constexpr int kScanPerThread = kScanTile / kScanThreads;  // 32
static_assert(kScanPerThread * kScanThreads == kScanTile, "scan tile");

inline int64_t scan_ws_elems(int64_t n) { return ceil_div(n > 0 ? n : 1, kScanTile) + 2; }

template <int NT>
__device__ __forceinline__ int32_t block_exclusive_sum(int32_t v, int32_t* smem_warp, int32_t* total) {
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  int32_t x = v;
#pragma unroll
  for (int o = 1; o < 32; o <<= 1) {
    int32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) smem_warp[warp] = x;
  __syncthreads();
  if (warp == 0) {
    int32_t w = lane < NT / 32 ? smem_warp[lane] : 0;
    int32_t s = w;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      int32_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < NT / 32) smem_warp[lane] = s - w;
    if (lane == NT / 32 - 1) smem_warp[32] = s;
  }
  __syncthreads();
  int32_t r = smem_warp[warp] + x - v;
  *total = smem_warp[32];
  __syncthreads();
  return r;
}

// Pass 1: per-tile sums.
template <class Load>
__global__ void __launch_bounds__(kScanThreads) k_scan_reduce(Load ld, int64_t n, int32_t* tile_sums) {
  __shared__ int32_t sw[33];
  const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanPerThread;
  int32_t s = 0;
#pragma unroll 4
  for (int k = 0; k < kScanPerThread; ++k) {
    int64_t i = base + k;
    if (i < n) s += ld(i);
  }
  int32_t tot;
  block_exclusive_sum<kScanThreads>(s, sw, &tot);
  if (threadIdx.x == 0) tile_sums[blockIdx.x] = tot;
}

// Pass 2: exclusive scan of the tile sums (single block); total -> *total_out.
__global__ void __launch_bounds__(1024) k_scan_tiles(int32_t* tile_sums, int64_t ntiles, int32_t* total_out);

// Pass 3: rescan every tile with its offset; st(i, exclusive_prefix, value).
template <class Load, class Store>
__global__ void __launch_bounds__(kScanThreads) k_scan_apply(Load ld, Store st, int64_t n,
                                                             const int32_t* tile_offsets) {
  __shared__ int32_t sw[33];
  const int64_t base = (int64_t)blockIdx.x * kScanTile + (int64_t)threadIdx.x * kScanPerThread;
  int32_t v[kScanPerThread];
  int32_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanPerThread; ++k) {
    int64_t i = base + k;
    v[k] = i < n ? ld(i) : 0;
    s += v[k];
  }
  int32_t tot;
  int32_t run = block_exclusive_sum<kScanThreads>(s, sw, &tot) + tile_offsets[blockIdx.x];
#pragma unroll
  for (int k = 0; k < kScanPerThread; ++k) {
    int64_t i = base + k;
    if (i < n) st(i, run, v[k]);
    run += v[k];
  }
}

// Device-wide exclusive scan driven by functors.  ws: int32[scan_ws_elems(n)].
// The total is written to *total_out (device).
template <class Load, class Store>
buffalo_status device_scan(Load ld, Store st, int64_t n, int32_t* ws, int32_t* total_out,
                           cudaStream_t s) {
  int64_t ntiles = ceil_div(n > 0 ? n : 1, kScanTile);
  k_scan_reduce<<<(unsigned)ntiles, kScanThreads, 0, s>>>(ld, n, ws);
  BF_LAUNCHED("k_scan_reduce");
  k_scan_tiles<<<1, 1024, 0, s>>>(ws, ntiles, total_out);
  BF_LAUNCHED("k_scan_tiles");
  k_scan_apply<<<(unsigned)ntiles, kScanThreads, 0, s>>>(ld, st, n, ws);
  BF_LAUNCHED("k_scan_apply");
  return BUFFALO_OK;
}

struct LoadArr {
  const int32_t* a;
  __device__ int32_t operator()(int64_t i) const { return a[i]; }
};
struct StoreArr {
  int32_t* a;
  __device__ void operator()(int64_t i, int32_t excl, int32_t) const { a[i] = excl; }
};

// In-place exclusive scan of a[0..n) with the total stored at a[n].
inline buffalo_status scan_inplace(int32_t* a, int64_t n, int32_t* ws, cudaStream_t s) {
  return device_scan(LoadArr{a}, StoreArr{a}, n, ws, a + n, s);
}

// ------------------------------------------------------------------ stable bin partition
// Stable counting partition of n items into <= 256 bins (one LSD radix pass).
constexpr int kPartThreads = 256;
constexpr int kPartTile = 4096;

inline int64_t part_tiles(int64_t n) { return ceil_div(n > 0 ? n : 1, kPartTile); }
inline int64_t part_count_elems(int64_t n) { return 256 * part_tiles(n); }

template <class Key>
__global__ void __launch_bounds__(kPartThreads) k_part_hist(Key key, int64_t n, int32_t* counts,
                                                            int64_t ntiles) {
  __shared__ int32_t h[256];
  h[threadIdx.x] = 0;
  __syncthreads();
  const int64_t t0 = (int64_t)blockIdx.x * kPartTile;
  for (int k = threadIdx.x; k < kPartTile; k += kPartThreads) {
    int64_t i = t0 + k;
    if (i < n) atomicAdd(&h[key(i)], 1);
  }
  __syncthreads();
  counts[(int64_t)threadIdx.x * ntiles + blockIdx.x] = h[threadIdx.x];
}

// emit(i, pos): item i goes to position pos (stable: input order inside a bin).
template <class Key, class Emit>
__global__ void __launch_bounds__(kPartThreads) k_part_scatter(Key key, Emit emit, int64_t n,
                                                               const int32_t* offsets, int64_t ntiles) {
  constexpr int NW = kPartThreads / 32;
  __shared__ int32_t base[256];
  __shared__ int32_t wcnt[NW][256];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  base[threadIdx.x] = offsets[(int64_t)threadIdx.x * ntiles + blockIdx.x];
  const int64_t t0 = (int64_t)blockIdx.x * kPartTile;
  for (int r = 0; r < kPartTile / kPartThreads; ++r) {
#pragma unroll
    for (int w = 0; w < NW; ++w) wcnt[w][threadIdx.x] = 0;
    __syncthreads();
    const int64_t i = t0 + (int64_t)r * kPartThreads + threadIdx.x;
    const bool valid = i < n;
    const int b = valid ? key(i) : 256 + lane;   // invalid lanes never match valid ones
    const unsigned peers = __match_any_sync(0xffffffffu, b);
    const int rank = __popc(peers & ((1u << lane) - 1u));
    if (valid && rank == 0) wcnt[warp][b] = __popc(peers);
    __syncthreads();
    if (valid) {
      int32_t off = base[b] + rank;
      for (int w = 0; w < warp; ++w) off += wcnt[w][b];
      emit(i, off);
    }
    __syncthreads();
    int32_t add = 0;
#pragma unroll
    for (int w = 0; w < NW; ++w) add += wcnt[w][threadIdx.x];
    base[threadIdx.x] += add;
    __syncthreads();
  }
}

// counts: int32[part_count_elems(n) + 1]; scan_ws: int32[scan_ws_elems(part_count_elems(n)+1)]
template <class Key, class Emit>
buffalo_status stable_partition(Key key, Emit emit, int64_t n, int32_t* counts, int32_t* scan_ws,
                                cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  int64_t nt = part_tiles(n);
  k_part_hist<<<(unsigned)nt, kPartThreads, 0, s>>>(key, n, counts, nt);
  BF_LAUNCHED("k_part_hist");
  BF_CHECK(scan_inplace(counts, 256 * nt, scan_ws, s));
  k_part_scatter<<<(unsigned)nt, kPartThreads, 0, s>>>(key, emit, n, counts, nt);
  BF_LAUNCHED("k_part_scatter");
  return BUFFALO_OK;
}

}  // namespace buffalo
