// cluster.cu — exact triangle counting and the average clustering coefficient C of Eq. 1
// ("C is the average clustering coefficient [27]", an offline property
// of the input graph; reading R27: Newman's local coefficient 2 T_v / (d_v (d_v - 1)), 0 for
// d_v < 2, averaged over all nodes).
//
// Design (B200): the graph is oriented by the total order rank(v) = (d_v, v), keeping for each
// node only its higher-ranked neighbours (out-degree <= sqrt(2 nnz), rows stay sorted by id).
// Every triangle {v, u, w} with rank v < u < w is then found exactly once, at v: for each u in
// out(v), for each w in out(u), test w in out(v).  A warp owns one v at a time (dynamic node
// grabbing for load balance); the (u, w) candidate pairs of 32 consecutive u are flattened
// over the lanes (segment found by a 5-step shuffle search of the warp's prefix of |out(u)|),
// so the out(u) reads are coalesced whatever the degrees; out(v) is staged in shared memory
// when it fits and binary-searched.  Each hit adds 1 to T_w (global atomic), to a per-warp
// shared counter of u (flushed once per 32 u) and to a register count of v (flushed once).
// C is reduced in float64 in a fixed order (fixed grid, fixed tree), so it is deterministic.
#include <algorithm>

#include "common.cuh"
#include "primitives.cuh"

namespace buffalo {

namespace {

constexpr int kTriWarps = 8;          // warps per CTA of k_tri
constexpr int kTriStage = 1024;       // out(v) entries staged in shared memory per warp
constexpr int kNodesPerGrab = 8;      // nodes taken per dynamic-scheduling atomic
constexpr int kCcBlocks = 592;        // fixed grid of the C reduction (4 x 148; determinism)
constexpr int kCcThreads = 256;

__device__ __forceinline__ bool ranks_above(int64_t du, int32_t u, int64_t dv, int32_t v) {
  return du > dv || (du == dv && u > v);
}

// out_deg[v] = #{u in N(v) : rank(u) > rank(v)}; warp per node.
__global__ void __launch_bounds__(256) k_orient_count(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                      int64_t N, int32_t* __restrict__ odeg) {
  const int lane = lane_id();
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t v = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; v < N; v += nw) {
    const int64_t a = rp[v], b = rp[v + 1], dv = b - a;
    int32_t c = 0;
    for (int64_t e = a + lane; e < b; e += 32) {
      const int32_t u = col[e];
      c += ranks_above(rp[u + 1] - rp[u], u, dv, (int32_t)v);
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) c += __shfl_xor_sync(0xffffffffu, c, o);
    if (lane == 0) odeg[v] = c;
  }
}

// ocol[optr[v] ..] = the higher-ranked neighbours of v in CSR (ascending id) order.
__global__ void __launch_bounds__(256) k_orient_fill(const int64_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                     int64_t N, const int32_t* __restrict__ optr,
                                                     int32_t* __restrict__ ocol) {
  const int lane = lane_id();
  const int64_t nw = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t v = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; v < N; v += nw) {
    const int64_t a = rp[v], b = rp[v + 1], dv = b - a;
    int32_t pos = optr[v];
    for (int64_t e0 = a; e0 < b; e0 += 32) {
      const int64_t e = e0 + lane;
      int32_t u = -1;
      bool keep = false;
      if (e < b) {
        u = col[e];
        keep = ranks_above(rp[u + 1] - rp[u], u, dv, (int32_t)v);
      }
      const unsigned m = __ballot_sync(0xffffffffu, keep);
      if (keep) ocol[pos + __popc(m & ((1u << lane) - 1u))] = u;
      pos += __popc(m);
    }
  }
}

__device__ __forceinline__ bool sorted_contains(const int32_t* a, int32_t n, int32_t x) {
  int32_t lo = 0, hi = n;
  while (lo < hi) {
    const int32_t mid = (lo + hi) >> 1;
    if (a[mid] < x) lo = mid + 1; else hi = mid;
  }
  return lo < n && a[lo] == x;
}

__global__ void __launch_bounds__(kTriWarps * 32) k_tri(const int32_t* __restrict__ optr, const int32_t* __restrict__ ocol,
                                                       int64_t N, unsigned long long* __restrict__ T,
                                                       unsigned long long* __restrict__ next) {
  __shared__ int32_t s_out[kTriWarps][kTriStage];
  __shared__ uint32_t s_cnt[kTriWarps][32];
  const int lane = lane_id(), warp = threadIdx.x >> 5;
  while (true) {
    unsigned long long base = 0;
    if (lane == 0) base = atomicAdd(next, (unsigned long long)kNodesPerGrab);
    base = __shfl_sync(0xffffffffu, base, 0);
    if ((int64_t)base >= N) break;
    const int64_t vend = std::min<int64_t>((int64_t)base + kNodesPerGrab, N);
    for (int64_t v = (int64_t)base; v < vend; ++v) {
      const int32_t a0 = optr[v], a = optr[v + 1] - a0;
      if (a < 2) continue;                                   // a triangle needs u, w in out(v)
      const int32_t* ov = ocol + a0;
      if (a <= kTriStage) {
        for (int j = lane; j < a; j += 32) s_out[warp][j] = ov[j];
        __syncwarp();
        ov = s_out[warp];
      }
      const int32_t lo_id = ov[0], hi_id = ov[a - 1];
      uint32_t cv = 0;
      for (int32_t j0 = 0; j0 < a; j0 += 32) {
        const int32_t j = j0 + lane;
        int32_t u = -1, st = 0, b = 0;
        if (j < a) {
          u = ov[j];
          st = optr[u];
          b = optr[u + 1] - st;
        }
        int32_t incl = b;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const int32_t y = __shfl_up_sync(0xffffffffu, incl, o);
          if (lane >= o) incl += y;
        }
        const int32_t excl = incl - b;
        const int32_t P = __shfl_sync(0xffffffffu, incl, 31);
        s_cnt[warp][lane] = 0;
        __syncwarp();
        for (int32_t p0 = 0; p0 < P; p0 += 32) {
          const int32_t p = p0 + lane;
          // segment of p: the smallest k with incl_k > p
          int k = 0;
#pragma unroll
          for (int step = 16; step; step >>= 1) {
            const int32_t y = __shfl_sync(0xffffffffu, incl, k + step - 1);
            if (y <= p) k += step;
          }
          const int32_t stk = __shfl_sync(0xffffffffu, st, k);
          const int32_t exk = __shfl_sync(0xffffffffu, excl, k);
          if (p < P) {
            const int32_t w = ocol[stk + (p - exk)];
            if (w >= lo_id && w <= hi_id && sorted_contains(ov, a, w)) {
              ++cv;
              atomicAdd(&s_cnt[warp][k], 1u);
              atomicAdd(&T[w], 1ull);
            }
          }
        }
        __syncwarp();
        const uint32_t cu = s_cnt[warp][lane];
        if (j < a && cu) atomicAdd(&T[u], (unsigned long long)cu);
        __syncwarp();
      }
#pragma unroll
      for (int o = 16; o; o >>= 1) cv += __shfl_xor_sync(0xffffffffu, cv, o);
      if (lane == 0 && cv) atomicAdd(&T[v], (unsigned long long)cv);
      __syncwarp();
    }
  }
}

// Fixed-order float64 sum of the local coefficients: grid-stride per thread, then a shared
// tree per CTA (kCcBlocks partials), then one CTA sums the partials the same way.
__device__ __forceinline__ double cta_tree_sum(double x, double* sh) {
  sh[threadIdx.x] = x;
  __syncthreads();
  for (int s = kCcThreads / 2; s; s >>= 1) {
    if ((int)threadIdx.x < s) sh[threadIdx.x] += sh[threadIdx.x + s];
    __syncthreads();
  }
  return sh[0];
}

__global__ void __launch_bounds__(kCcThreads) k_cc_partial(const int64_t* __restrict__ rp,
                                                           const int64_t* __restrict__ T, int64_t N,
                                                           double* __restrict__ partial) {
  __shared__ double sh[kCcThreads];
  double acc = 0.0;
  for (int64_t v = blockIdx.x * (int64_t)kCcThreads + threadIdx.x; v < N; v += (int64_t)kCcBlocks * kCcThreads) {
    const int64_t d = rp[v + 1] - rp[v];
    if (d >= 2) {
      const double dd = (double)d;
      acc += 2.0 * (double)T[v] / (dd * (dd - 1.0));
    }
  }
  const double s = cta_tree_sum(acc, sh);
  if (threadIdx.x == 0) partial[blockIdx.x] = s;
}

__global__ void __launch_bounds__(kCcThreads) k_cc_final(const double* __restrict__ partial, int64_t N,
                                                         double* __restrict__ out) {
  __shared__ double sh[kCcThreads];
  double acc = 0.0;
  for (int i = threadIdx.x; i < kCcBlocks; i += kCcThreads) acc += partial[i];
  const double s = cta_tree_sum(acc, sh);
  if (threadIdx.x == 0) out[0] = s / (double)N;
}

struct LoadI32 {
  const int32_t* a;
  __device__ __forceinline__ int32_t operator()(int64_t i) const { return a[i]; }
};
struct StoreExcl {
  int32_t* a;
  __device__ __forceinline__ void operator()(int64_t i, int32_t excl, int32_t) const { a[i] = excl; }
};

struct ClusterWs {
  int32_t* optr;        // [N+1]  out-degrees, scanned in place to offsets
  int32_t* ocol;        // [nnz/2 + 1]
  int32_t* scan;        // [scan_ws_elems(N)]
  unsigned long long* next;
  double* partial;      // [kCcBlocks + 1] (the last slot is C)
};

int64_t cluster_ws_bytes(int64_t N, int64_t nnz) {
  return R(4 * (N + 1)) + R(4 * (nnz / 2 + 1)) + R(4 * scan_ws_elems(N + 1)) + R(8) + R(8 * (kCcBlocks + 1));
}

ClusterWs cluster_ws(void* base, int64_t N, int64_t nnz) {
  char* p = (char*)base;
  ClusterWs w;
  w.optr = (int32_t*)p; p += R(4 * (N + 1));
  w.ocol = (int32_t*)p; p += R(4 * (nnz / 2 + 1));
  w.scan = (int32_t*)p; p += R(4 * scan_ws_elems(N + 1));
  w.next = (unsigned long long*)p; p += R(8);
  w.partial = (double*)p;
  return w;
}

buffalo_status validate_cluster(const buffalo_graph* g, void* ws, size_t ws_bytes) {
  BF_CHECK(require_sm100());
  if (!g || !g->row_ptr || (!g->col && g->nnz > 0) || g->num_nodes <= 0 || g->nnz < 0 || !ws) {
    set_error("clustering: null graph/workspace or empty graph");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (g->nnz / 2 >= INT32_MAX || g->num_nodes >= INT32_MAX) {
    set_error("clustering: oriented graph needs nnz/2 < 2^31 and N < 2^31");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if ((int64_t)ws_bytes < cluster_ws_bytes(g->num_nodes, g->nnz)) {
    set_error("clustering: workspace %zu B < %lld B", ws_bytes, (long long)cluster_ws_bytes(g->num_nodes, g->nnz));
    return BUFFALO_ERR_CAPACITY;
  }
  return BUFFALO_OK;
}

}  // namespace

}  // namespace buffalo

using namespace buffalo;

extern "C" {

size_t buffalo_clustering_workspace_bytes(const buffalo_graph* g) {
  if (!g || g->num_nodes <= 0) return 0;
  return (size_t)cluster_ws_bytes(g->num_nodes, g->nnz);
}

buffalo_status buffalo_triangles(const buffalo_graph* g, int64_t* T, void* ws, size_t ws_bytes, void* stream) {
  BF_CHECK(validate_cluster(g, ws, ws_bytes));
  if (!T) return BUFFALO_ERR_INVALID_ARG;
  cudaStream_t s = (cudaStream_t)stream;
  const int64_t N = g->num_nodes;
  ClusterWs w = cluster_ws(ws, N, g->nnz);
  const int orient_grid = grid_for(N * 32, 256);
  k_orient_count<<<orient_grid, 256, 0, s>>>(g->row_ptr, g->col, N, w.optr);
  BF_LAUNCHED("k_orient_count");
  int32_t* optr = w.optr;
  BF_CHECK(device_scan(LoadI32{optr}, StoreExcl{optr}, N, w.scan, optr + N, s));   // in place
  k_orient_fill<<<orient_grid, 256, 0, s>>>(g->row_ptr, g->col, N, w.optr, w.ocol);
  BF_LAUNCHED("k_orient_fill");
  BF_CUDA(cudaMemsetAsync(T, 0, sizeof(int64_t) * N, s));
  BF_CUDA(cudaMemsetAsync(w.next, 0, sizeof(unsigned long long), s));
  k_tri<<<148 * 8, kTriWarps * 32, 0, s>>>(w.optr, w.ocol, N, (unsigned long long*)T, w.next);
  BF_LAUNCHED("k_tri");
  return BUFFALO_OK;
}

buffalo_status buffalo_avg_clustering(const buffalo_graph* g, const int64_t* T, double* C_h, int64_t* C_ppm_h,
                                      void* ws, size_t ws_bytes, void* stream) {
  BF_CHECK(validate_cluster(g, ws, ws_bytes));
  if (!T || !C_h) return BUFFALO_ERR_INVALID_ARG;
  cudaStream_t s = (cudaStream_t)stream;
  ClusterWs w = cluster_ws(ws, g->num_nodes, g->nnz);
  k_cc_partial<<<kCcBlocks, kCcThreads, 0, s>>>(g->row_ptr, T, g->num_nodes, w.partial);
  BF_LAUNCHED("k_cc_partial");
  k_cc_final<<<1, kCcThreads, 0, s>>>(w.partial, g->num_nodes, w.partial + kCcBlocks);
  BF_LAUNCHED("k_cc_final");
  BF_CUDA(cudaMemcpyAsync(C_h, w.partial + kCcBlocks, sizeof(double), cudaMemcpyDeviceToHost, s));
  BF_CUDA(cudaStreamSynchronize(s));
  if (C_ppm_h) *C_ppm_h = (int64_t)llround(*C_h * 1e6);
  return BUFFALO_OK;
}

}  // extern "C"
