// primitives.cuh — device-wide scan and stable bin partition used by block generation and
// bucketing.  Functor-driven so that flags/keys are computed on the fly (no flag arrays).
#pragma once
#include "common.cuh"

namespace buffalo {

// Single-pass decoupled look-back scan: each CTA (dynamic tile id) loads its tile with
// coalesced functor evaluations into shared memory, scans it, publishes its aggregate, looks
// back over its predecessors' published values and applies the store functor in coalesced
// order.  Workspace: a zeroed status word (flag | value) per tile + a tile counter.
constexpr int kScanThreads = 512;
constexpr int kScanItems = 8;
static_assert(kScanItems * kScanThreads == kScanTile, "scan tile");

inline int64_t scan_ws_elems(int64_t n) { return 2 * (ceil_div(n > 0 ? n : 1, kScanTile) + 2); }

__device__ __forceinline__ int scan_pad(int i) { return i + (i >> 5); }

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

constexpr uint64_t kFlagAgg = 1ull << 32, kFlagPrefix = 2ull << 32;

template <class Load, class Store>
__global__ void __launch_bounds__(kScanThreads) k_scan_lookback(Load ld, Store st, int64_t n,
                                                                unsigned long long* status,
                                                                unsigned int* counter, int32_t* total_out) {
  pdl_wait();
  __shared__ int32_t sv[kScanTile + kScanTile / 32];
  __shared__ int32_t sx[kScanTile + kScanTile / 32];
  __shared__ int32_t sw[33];
  __shared__ int32_t s_prefix;
  __shared__ unsigned int s_tile;
  if (threadIdx.x == 0) s_tile = atomicAdd(counter, 1u);
  __syncthreads();
  const int64_t tile = s_tile;
  const int64_t base = tile * kScanTile;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    const int li = k * kScanThreads + threadIdx.x;
    const int64_t i = base + li;
    sv[scan_pad(li)] = i < n ? ld(i) : 0;
  }
  __syncthreads();
  int32_t v[kScanItems];
  int32_t sum = 0;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    v[k] = sv[scan_pad(threadIdx.x * kScanItems + k)];
    sum += v[k];
  }
  int32_t agg;
  int32_t run = block_exclusive_sum<kScanThreads>(sum, sw, &agg);
  if (threadIdx.x == 0) {
    volatile unsigned long long* vs = status;
    if (tile == 0) {
      __threadfence();
      vs[0] = kFlagPrefix | (uint32_t)agg;
      s_prefix = 0;
    } else {
      vs[tile] = kFlagAgg | (uint32_t)agg;
      __threadfence();
      int32_t excl = 0;
      int64_t p = tile - 1;
      while (true) {
        unsigned long long w = vs[p];
        if ((w >> 32) == 0) continue;        // not yet published: spin
        excl += (int32_t)(uint32_t)w;
        if ((w >> 32) == 2) break;
        --p;
      }
      __threadfence();
      vs[tile] = kFlagPrefix | (uint32_t)(excl + agg);
      s_prefix = excl;
    }
    if (base + kScanTile >= n && total_out) *total_out = s_prefix + agg;
  }
  __syncthreads();
  run += s_prefix;
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    sx[scan_pad(threadIdx.x * kScanItems + k)] = run;
    run += v[k];
  }
  __syncthreads();
#pragma unroll
  for (int k = 0; k < kScanItems; ++k) {
    const int li = k * kScanThreads + threadIdx.x;
    const int64_t i = base + li;
    if (i < n) st(i, sx[scan_pad(li)], sv[scan_pad(li)]);
  }
}

// Device-wide exclusive scan driven by functors.  ws: int32[scan_ws_elems(n)] (any content).
// The total is written to *total_out (device).
template <class Load, class Store>
buffalo_status device_scan(Load ld, Store st, int64_t n, int32_t* ws, int32_t* total_out,
                           cudaStream_t s) {
  const int64_t ntiles = ceil_div(n > 0 ? n : 1, kScanTile);
  BF_CUDA(cudaMemsetAsync(ws, 0, sizeof(unsigned long long) * (ntiles + 1), s));
  unsigned long long* status = reinterpret_cast<unsigned long long*>(ws);
  unsigned int* counter = reinterpret_cast<unsigned int*>(status + ntiles);
  launch_pdl(k_scan_lookback<Load, Store>, dim3((unsigned)ntiles), dim3(kScanThreads), 0, s, ld, st, n, status, counter,
             total_out);
  BF_LAUNCHED("k_scan_lookback");
  return BUFFALO_OK;
}

// Integer count (sum of a 0/1 or small functor) over [0, n) into *total (zeroed first).
template <class Load>
__global__ void __launch_bounds__(256) k_count_sum(Load ld, int64_t n, int32_t* total) {
  pdl_wait();
  int32_t s = 0;
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
    s += ld(i);
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  if ((threadIdx.x & 31) == 0 && s) atomicAdd(total, s);
}
template <class Load>
buffalo_status device_count(Load ld, int64_t n, int32_t* total, cudaStream_t s) {
  BF_CUDA(cudaMemsetAsync(total, 0, sizeof(int32_t), s));
  if (n <= 0) return BUFFALO_OK;
  launch_pdl(k_count_sum<Load>, dim3(grid_for(n, 256)), dim3(256), 0, s, ld, n, total);
  BF_LAUNCHED("k_count_sum");
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
// Stable counting partition of n items into <= 256 bins (one LSD radix pass).  Tiles of
// kPartTile items, one 1024-thread CTA each (four rounds of 1024 items per tile).
constexpr int kPartThreads = 1024;
constexpr int kPartTile = 4096;

inline int64_t part_tiles(int64_t n) { return ceil_div(n > 0 ? n : 1, kPartTile); }
inline int64_t part_count_elems(int64_t n) { return 256 * part_tiles(n); }

template <class Key>
__global__ void __launch_bounds__(kPartThreads) k_part_hist(Key key, int64_t n, int32_t* counts,
                                                            int64_t ntiles) {
  pdl_wait();
  __shared__ int32_t h[256];
  if (threadIdx.x < 256) h[threadIdx.x] = 0;
  __syncthreads();
  const int64_t t0 = (int64_t)blockIdx.x * kPartTile;
  for (int k = threadIdx.x; k < kPartTile; k += kPartThreads) {
    int64_t i = t0 + k;
    if (i < n) atomicAdd(&h[key(i)], 1);
  }
  __syncthreads();
  if (threadIdx.x < 256) counts[(int64_t)threadIdx.x * ntiles + blockIdx.x] = h[threadIdx.x];
}

// emit(i, pos): item i goes to position pos (stable: input order inside a bin).
template <class Key, class Emit>
__global__ void __launch_bounds__(kPartThreads) k_part_scatter(Key key, Emit emit, int64_t n,
                                                               const int32_t* offsets, int64_t ntiles) {
  pdl_wait();
  constexpr int NW = kPartThreads / 32;
  __shared__ int32_t base[256];
  __shared__ int32_t wcnt[NW][256];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  if (threadIdx.x < 256) base[threadIdx.x] = offsets[(int64_t)threadIdx.x * ntiles + blockIdx.x];
  const int64_t t0 = (int64_t)blockIdx.x * kPartTile;
  for (int r = 0; r < kPartTile / kPartThreads; ++r) {
    for (int k = threadIdx.x; k < NW * 256; k += kPartThreads) (&wcnt[0][0])[k] = 0;
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
    if (threadIdx.x < 256) {
      int32_t add = 0;
#pragma unroll 8
      for (int w = 0; w < NW; ++w) add += wcnt[w][threadIdx.x];
      base[threadIdx.x] += add;
    }
    __syncthreads();
  }
}

// counts: int32[part_count_elems(n) + 1]; scan_ws: int32[scan_ws_elems(part_count_elems(n)+1)]
template <class Key, class Emit>
buffalo_status stable_partition(Key key, Emit emit, int64_t n, int32_t* counts, int32_t* scan_ws,
                                cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  int64_t nt = part_tiles(n);
  launch_pdl(k_part_hist<Key>, dim3((unsigned)nt), dim3(kPartThreads), 0, s, key, n, counts, nt);
  BF_LAUNCHED("k_part_hist");
  BF_CHECK(scan_inplace(counts, 256 * nt, scan_ws, s));
  launch_pdl(k_part_scatter<Key, Emit>, dim3((unsigned)nt), dim3(kPartThreads), 0, s, key, emit, n, counts, nt);
  BF_LAUNCHED("k_part_scatter");
  return BUFFALO_OK;
}

}  // namespace buffalo
