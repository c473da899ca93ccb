// api.cu — the C ABI (include/buffalo.h): validation, arena layout, the scheduler's K loop
// (Alg. 3/4) and the memory model (R15).  Host code; all compute is in build.cu / sage.cu /
// tc_sage.cu kernels.
#include <cuda.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstring>
#include <string>
#include <vector>

#include "build.cuh"
#include "common.cuh"
#include "primitives.cuh"
#include "sage.cuh"
#include "tc_sage.cuh"

namespace buffalo {

static thread_local std::string g_err;
static std::atomic<int64_t> g_launches{0};

void set_error(const char* fmt, ...) {
  char buf[1024];
  va_list ap;
  va_start(ap, fmt);
  vsnprintf(buf, sizeof(buf), fmt, ap);
  va_end(ap);
  g_err = buf;
}
void count_launch(int n) { g_launches += n; }

// ------------------------------------------------------------------ kernel timing (diagnostic)
namespace {
struct Profiler {
  bool on = false;
  std::string family;
  unsigned long long* counters = nullptr;   // caller's device buffer, one per launch
  int64_t max_launches = 0;
  std::vector<cudaEvent_t> ev;
  std::vector<double> fixed, per_edge;
};
thread_local Profiler g_prof;   // per host thread (launch sites record on the calling thread)
}  // namespace

ProfSlot prof_begin_launch(const char* family, cudaStream_t s) {
  ProfSlot slot{nullptr, -1};
  if (!g_prof.on || g_prof.family != family || (int64_t)g_prof.fixed.size() >= g_prof.max_launches) return slot;
  if (2 * g_prof.fixed.size() >= g_prof.ev.size()) return slot;   // event pool exhausted
  slot.index = (int)g_prof.fixed.size();
  slot.edges_dev = g_prof.counters + slot.index;
  g_prof.fixed.push_back(0.0);
  g_prof.per_edge.push_back(0.0);
  cudaEventRecord(g_prof.ev[2 * slot.index], s);
  return slot;
}
void prof_end_launch(const ProfSlot& slot, cudaStream_t s, double fixed_bytes, double bytes_per_edge) {
  if (slot.index < 0) return;
  cudaEventRecord(g_prof.ev[2 * slot.index + 1], s);
  g_prof.fixed[slot.index] = fixed_bytes;
  g_prof.per_edge[slot.index] = bytes_per_edge;
}

buffalo_status check_cuda(const char* what) {
  cudaError_t e = cudaGetLastError();
  if (e != cudaSuccess) {
    set_error("%s: %s", what, cudaGetErrorString(e));
    return BUFFALO_ERR_CUDA;
  }
  return BUFFALO_OK;
}

buffalo_status require_sm100() {
  int dev = 0;
  BF_CUDA(cudaGetDevice(&dev));
  int major = 0, minor = 0;
  BF_CUDA(cudaDeviceGetAttribute(&major, cudaDevAttrComputeCapabilityMajor, dev));
  BF_CUDA(cudaDeviceGetAttribute(&minor, cudaDevAttrComputeCapabilityMinor, dev));
  if (major != 10 || minor != 0) {
    set_error("libbuffalo is built for sm_100a only (device %d is sm_%d%d)", dev, major, minor);
    return BUFFALO_ERR_UNSUPPORTED;
  }
  return BUFFALO_OK;
}

__global__ void k_fill_i32(int32_t* a, int64_t n, int32_t v) {
  for (int64_t k = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; k < n; k += (int64_t)gridDim.x * blockDim.x)
    a[k] = v;
}

// ------------------------------------------------------------------ memory model (R15)
// Restated from DESIGN.md §5; must agree with the arena that buffalo_build_blocks lays out.
static int64_t bwd_scratch_for(const buffalo_model* m, int64_t n_dst, int64_t n_src, int64_t e, int l) {
  if (m->aggregator == BUFFALO_AGG_POOL) return pool_bwd_scratch_bytes(n_dst, n_src, m->dim[l - 1], m->dim[l]);
  if (m->aggregator == BUFFALO_AGG_LSTM) return lstm_bwd_scratch_bytes(n_dst, e, l, m->dim[l - 1], m->dim[l]);
  if (m->aggregator == BUFFALO_AGG_GAT) return gat_bwd_scratch_bytes(n_src, n_dst, e, m->dim[l - 1], m->dim[l]);
  if (m->gemm_mode == BUFFALO_GEMM_BF16)
    return tc_bwd_scratch_bytes(n_dst, n_src, e, l, m->dim[l - 1], m->dim[l], l == m->num_layers);
  return bwd_scratch_bytes(n_dst, n_src, l, m->dim[l - 1], m->dim[l]);
}

// dH_l slot of the backward region: fp32 dH (FFMA) / dlogits; in BF16 mode layers l < L hold
// bf16 dZ_l plus the column-sum partials of the fused transposed Aggregate that wrote it.
static int64_t dh_slot_bytes(const buffalo_model* m, int64_t n, int l) {
  if (m->gemm_mode == BUFFALO_GEMM_BF16 && l < m->num_layers)     // bf16 dZ_l + its db partial rows
    return R(n * pitch_of(m->dim[l]) * 2) + R((int64_t)4 * tc_bwd_db_parts() * m->dim[l]);
  return R(n * pitch_of(m->dim[l]) * 4);                          // fp32 dH / dlogits
}

static void mem_model(int L, const int64_t* n, const int64_t* e, const buffalo_model* m,
                      int64_t* lo, int64_t* hi) {
  const int64_t s = m->gemm_mode == BUFFALO_GEMM_BF16 ? 2 : 4;
  const bool pool = m->aggregator == BUFFALO_AGG_POOL || m->aggregator == BUFFALO_AGG_GAT;  // R28/R30: block 1
                                                                                              // keeps a transpose too
  int64_t blocks = 0, build = 0, acts = 0, bwd = 0;
  for (int l = 1; l <= L; ++l) {
    const int64_t nl = n[l], nm = n[l - 1], el = e[l - 1];
    blocks += R(4 * (nl + 1)) + R(4 * nl) + R(4 * el) + R(4 * nm);
    blocks += (l == 1) ? R(4 * el) : R(4 * (nm + 1)) + R(4 * el) + R(4 * nm);
    if (l == 1 && pool) blocks += R(4 * (nm + 1)) + R(4 * el) + R(4 * nm);
    build = std::max(build, build_frame_bytes(nl, el, l, false, pool));
  }
  for (int l = 1; l <= L; ++l) {
    if (m->aggregator != BUFFALO_AGG_GAT) acts += R(n[l] * pitch_of(m->dim[l - 1]) * s);   // saved h_agg
    if (l < L) acts += R(n[l] * pitch_of(m->dim[l]) * s);
  }
  if (m->aggregator == BUFFALO_AGG_GAT)
    for (int l = 1; l <= L; ++l) acts += gat_saved_bytes(n[l - 1], n[l], e[l - 1], m->dim[l]);
  acts += R(n[L] * pitch_of(m->dim[L]) * 4);
  if (m->feat_shards) acts += R(n[1] * pitch_of(m->dim[0]) * 2);     // block 1's self_rows copy
  if (m->aggregator == BUFFALO_AGG_LSTM)
    for (int l = 1; l <= L; ++l) acts += R(lstm_saved_bytes(n[l], e[l - 1], m->dim[l - 1]));
  if (m->aggregator == BUFFALO_AGG_POOL)
    for (int l = 1; l <= L; ++l)   // P [n_{l-1}] and argmax [n_l] rows of width pitch(d_{l-1})
      acts += R(n[l - 1] * pitch_of(m->dim[l - 1]) * 4) + R(n[l] * pitch_of(m->dim[l - 1]) * 4);
  for (int l = L; l >= 1; --l) {
    int64_t f = dh_slot_bytes(m, n[l], l);
    if (l >= 2) f += dh_slot_bytes(m, n[l - 1], l - 1);
    f += bwd_scratch_for(m, n[l], n[l - 1], e[l - 1], l);
    bwd = std::max(bwd, f);
  }
  *lo = blocks + acts + bwd;
  *hi = blocks + acts + std::max(bwd, build);
}

static buffalo_status validate_model(const buffalo_model* m) {
  if (!m || m->num_layers < 1 || m->num_layers > BUFFALO_MAX_LAYERS) {
    set_error("model: num_layers must be in [1, %d]", BUFFALO_MAX_LAYERS);
    return BUFFALO_ERR_INVALID_ARG;
  }
  for (int l = 0; l <= m->num_layers; ++l)
    if (m->dim[l] < 1 || m->dim[l] > BUFFALO_MAX_DIM) {
      set_error("model: dim[%d] = %d out of range", l, m->dim[l]);
      return BUFFALO_ERR_INVALID_ARG;
    }
  if (m->feat_dtype != BUFFALO_FP32 && m->feat_dtype != BUFFALO_BF16) return BUFFALO_ERR_INVALID_ARG;
  if (m->gemm_mode != BUFFALO_GEMM_FFMA && m->gemm_mode != BUFFALO_GEMM_BF16) return BUFFALO_ERR_INVALID_ARG;
  if (m->gemm_mode == BUFFALO_GEMM_BF16)
    for (int l = 1; l <= m->num_layers; ++l)
      if (m->dim[l] > 256) {
        set_error("model: the bf16 tensor-core path supports dim[l] <= 256 for l >= 1");
        return BUFFALO_ERR_UNSUPPORTED;
      }
  if (m->aggregator < BUFFALO_AGG_MEAN || m->aggregator > BUFFALO_AGG_GAT) {
    set_error("model: unknown aggregator %d", m->aggregator);
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (m->aggregator != BUFFALO_AGG_MEAN && m->gemm_mode != BUFFALO_GEMM_FFMA) {
    set_error("model: the pool, LSTM and GAT models are built for gemm_mode FFMA (fp32) only");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (m->feat_pitch < round_up(m->dim[0], 8) || m->feat_pitch % 8) {
    set_error("model: feat_pitch must be a multiple of 8 and >= round_up(dim[0], 8)");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (const buffalo_feature_shards* sh = m->feat_shards) {
    if (sh->num_shards < 1 || sh->num_shards > BUFFALO_MAX_SHARDS || sh->rows_per_shard < 1 ||
        sh->rows_per_shard > INT32_MAX) {
      set_error("model: feat_shards needs 1..%d shards of 1..2^31-1 rows", BUFFALO_MAX_SHARDS);
      return BUFFALO_ERR_INVALID_ARG;
    }
    for (int k = 0; k < sh->num_shards; ++k)
      if (!sh->shard[k] || ((uintptr_t)sh->shard[k]) % 16) {
        set_error("model: feat_shards.shard[%d] is null or not 16-B aligned", k);
        return BUFFALO_ERR_INVALID_ARG;
      }
    if (m->feat_dtype != BUFFALO_BF16 || m->gemm_mode != BUFFALO_GEMM_BF16 || m->aggregator != BUFFALO_AGG_MEAN) {
      set_error("model: a sharded feature table is supported for the bf16 SAGE-mean path only");
      return BUFFALO_ERR_UNSUPPORTED;
    }
  }
  return BUFFALO_OK;
}

static buffalo_status validate_sampler(const buffalo_sampler* s, int L) {
  if (!s || s->num_layers != L) {
    set_error("sampler.num_layers must equal model.num_layers");
    return BUFFALO_ERR_INVALID_ARG;
  }
  for (int l = 0; l < L; ++l)
    if (s->fanout[l] > BUFFALO_MAX_FANOUT) {
      set_error("fanout %d > %d not supported", s->fanout[l], BUFFALO_MAX_FANOUT);
      return BUFFALO_ERR_UNSUPPORTED;
    }
  if (s->cutoff_F < 0 || s->cutoff_F > 254) {
    set_error("cutoff_F must be in [0, 254]");
    return BUFFALO_ERR_INVALID_ARG;
  }
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ scheduler (Alg. 3/4)
struct Item {
  int d, k;                  // bucket degree, micro-bucket index
  int64_t start, count;      // slice of the bucket-sorted seeds
  int64_t O, E, I, M, w;
};

constexpr int kStatsBatch = 256;       // items per statistics pass (mask_stats)

// Item statistics (R13, R15): exact layer sizes of up to 256 items per pass (mask_stats), then
// O = #seeds, E = e_L, I = n_{L-1} and M_est = hi of the memory model.
// cache_mode (the sampler's sample cache, when it has one): 1 = sample and store, 2 = read the
// rows stored by an earlier pass of the same call.
// sizes: one row [2L+1] per item: n_0..n_L, e_1..e_L.
static buffalo_status items_sizes(const buffalo_graph* g, const int32_t* sorted_ids, const std::vector<Item*>& items,
                                  const buffalo_sampler* sp, int L, char* ws, int64_t ws_bytes, bool& masks_clean,
                                  cudaStream_t s, int cache_mode, std::vector<int64_t>& sizes) {
  const int W = 2 * L + 1;
  sizes.assign(items.size() * W, 0);
  for (size_t b0 = 0; b0 < items.size(); b0 += kStatsBatch) {
    const int nit = (int)std::min<size_t>(kStatsBatch, items.size() - b0);
    int64_t starts[kStatsBatch], counts[kStatsBatch];
    for (int k = 0; k < nit; ++k) {
      starts[k] = items[b0 + k]->start;
      counts[k] = items[b0 + k]->count;
    }
    static thread_local int64_t nh[kStatsBatch][BUFFALO_MAX_LAYERS + 1], eh[kStatsBatch][BUFFALO_MAX_LAYERS];
    BF_CHECK(mask_stats(g, sorted_ids, starts, counts, nit, sp, L, ws, ws_bytes, masks_clean, nh, eh, s, cache_mode));
    masks_clean = true;
    for (int k = 0; k < nit; ++k) {
      int64_t* row = sizes.data() + (b0 + k) * W;
      for (int l = 0; l <= L; ++l) row[l] = nh[k][l];
      for (int l = 1; l <= L; ++l) row[L + l] = eh[k][l - 1];
    }
  }
  return BUFFALO_OK;
}

static void derive_item(Item& it, const int64_t* row, int L, const buffalo_model* m) {
  int64_t lo, hi;
  mem_model(L, row, row + L + 1, m, &lo, &hi);
  it.O = it.count;
  it.E = row[L + L];          // e_L
  it.I = row[L - 1];          // n_{L-1}
  it.M = hi;
}

static buffalo_status items_stats(const buffalo_graph* g, const int32_t* sorted_ids, std::vector<Item*>& items,
                                  const buffalo_sampler* sp, const buffalo_model* m, char* ws, int64_t ws_bytes,
                                  bool& masks_clean, cudaStream_t s, int cache_mode) {
  const int L = m->num_layers;
  std::vector<int64_t> sizes;
  BF_CHECK(items_sizes(g, sorted_ids, items, sp, L, ws, ws_bytes, masks_clean, s, cache_mode, sizes));
  for (size_t k = 0; k < items.size(); ++k) derive_item(*items[k], sizes.data() + k * (2 * L + 1), L, m);
  return BUFFALO_OK;
}

// The same statistics with the items shared out over the ranks (sched.allgather given, more
// than one GPU): rank r measures the items k = r, r + G, r + 2G, ... and one all-gather of their
// int64 size rows gives every rank the whole table (identical on every rank: the plan stays
// deterministic without a broadcast).  Used for every statistics pass of Alg. 3 (the degree
// buckets and the K loop's micro-bucket candidates); the group-size pass measures own groups.
static buffalo_status items_stats_shared(const buffalo_graph* g, const int32_t* sorted_ids, std::vector<Item*>& items,
                                         const buffalo_sampler* sp, const buffalo_model* m, const buffalo_sched* sc,
                                         char* ws, int64_t ws_bytes, bool& masks_clean, cudaStream_t s,
                                         int cache_mode) {
  const int G = sc->num_gpus;
  if (!sc->allgather || G <= 1)
    return items_stats(g, sorted_ids, items, sp, m, ws, ws_bytes, masks_clean, s, cache_mode);
  const int L = m->num_layers, W = 2 * L + 1;
  std::vector<Item*> mine;
  for (size_t k = sc->rank; k < items.size(); k += G) mine.push_back(items[k]);
  std::vector<int64_t> sizes;
  BF_CHECK(items_sizes(g, sorted_ids, mine, sp, L, ws, ws_bytes, masks_clean, s, cache_mode, sizes));
  const int64_t per = (int64_t)((items.size() + G - 1) / G);          // rows per rank (padded)
  std::vector<int64_t> send(per * W, -1), recv((size_t)G * per * W, -1);
  std::copy(sizes.begin(), sizes.end(), send.begin());
  if (sc->allgather(sc->allgather_ctx, send.data(), recv.data(), per * W * (int64_t)sizeof(int64_t)) != 0) {
    set_error("bucketize: the all-gather of the item statistics failed");
    return BUFFALO_ERR_CUDA;
  }
  for (size_t k = 0; k < items.size(); ++k) {
    const int r = (int)(k % G);
    const int64_t j = (int64_t)(k / G);
    derive_item(*items[k], recv.data() + ((int64_t)r * per + j) * W, L, m);
  }
  return BUFFALO_OK;
}

// SplitExplosionBucket (R8): K contiguous pieces of bucket F, the first (O mod K) one seed larger.
static std::vector<Item> split_pieces(const Item& itF, int F, int K) {
  std::vector<Item> pieces;
  const int64_t O = itF.count, base = O / K, extra = O % K;
  int64_t st0 = itF.start;
  for (int k = 0; k < K; ++k) {
    const int64_t len = base + (k < extra ? 1 : 0);
    if (len > 0) pieces.push_back(Item{F, k, st0, len, 0, 0, 0, 0, 0});
    st0 += len;
  }
  return pieces;
}

// Eq. 1-2, integer form (R14): floor(M * min(1, I*10^6 / (E*C_ppm))).
static int64_t grouping_weight(int64_t M, int64_t I, int64_t E, int64_t C_ppm) {
  if (E == 0 || C_ppm <= 0) return M;
  unsigned __int128 num = (unsigned __int128)M * (unsigned __int128)I * 1000000u;
  unsigned __int128 den = (unsigned __int128)E * (unsigned __int128)C_ppm;
  unsigned __int128 q = num / den;
  return q < (unsigned __int128)M ? (int64_t)q : M;
}

__global__ void k_scatter_segments(const int64_t* __restrict__ seg, const int32_t* __restrict__ order,
                                   const int32_t* __restrict__ sorted_ids, int32_t* __restrict__ group_seeds,
                                   int32_t* __restrict__ group_of_seed) {
  const int64_t start = seg[4 * blockIdx.x], len = seg[4 * blockIdx.x + 1];
  const int64_t grp = seg[4 * blockIdx.x + 2], off = seg[4 * blockIdx.x + 3];
  for (int64_t t = threadIdx.x; t < len; t += blockDim.x) {
    group_seeds[off + t] = sorted_ids[start + t];
    group_of_seed[order[start + t]] = (int32_t)grp;
  }
}

static int64_t bucketize_fixed_bytes(int64_t S, int F, int k_max) {
  const int64_t pc = part_count_elems(S);
  (void)F;
  return R(S) + 2 * R(4 * S) + R(4 * (pc + 1)) + R(4 * scan_ws_elems(pc + 1)) + R(4 * 258) +
         R(32 * (int64_t)(256 + k_max + 1));
}

}  // namespace buffalo

using namespace buffalo;

// ===================================================================== C ABI
extern "C" {

const char* buffalo_status_str(buffalo_status s) {
  switch (s) {
    case BUFFALO_OK: return "BUFFALO_OK";
    case BUFFALO_ERR_INVALID_ARG: return "BUFFALO_ERR_INVALID_ARG";
    case BUFFALO_ERR_BUDGET: return "BUFFALO_ERR_BUDGET";
    case BUFFALO_ERR_CAPACITY: return "BUFFALO_ERR_CAPACITY";
    case BUFFALO_ERR_CUDA: return "BUFFALO_ERR_CUDA";
    case BUFFALO_ERR_UNSUPPORTED: return "BUFFALO_ERR_UNSUPPORTED";
  }
  return "BUFFALO_ERR_UNKNOWN";
}

const char* buffalo_last_error(void) { return g_err.c_str(); }
int64_t buffalo_launch_count(void) { return g_launches.load(); }

buffalo_status buffalo_profile_begin(const char* family, void* counters, int64_t max_launches, void* stream) {
  const std::string fam = family ? family : "";
  if (!family || (fam != "gather" && fam != "pool_max" && fam != "lstm_gates" && fam != "gat_attn") || !counters ||
      max_launches <= 0) {
    set_error("profile_begin: unknown kernel family or no counter buffer");
    return BUFFALO_ERR_INVALID_ARG;
  }
  for (cudaEvent_t e : g_prof.ev) cudaEventDestroy(e);
  g_prof = Profiler();
  g_prof.on = true;
  g_prof.family = family;
  g_prof.counters = (unsigned long long*)counters;
  g_prof.max_launches = max_launches;
  // events are created here, outside the timed region (at most 16384 timed launches)
  g_prof.ev.resize(2 * std::min<int64_t>(max_launches, 16384));
  for (cudaEvent_t& e : g_prof.ev) BF_CUDA(cudaEventCreate(&e));
  BF_CUDA(cudaMemsetAsync(counters, 0, sizeof(unsigned long long) * max_launches, (cudaStream_t)stream));
  return BUFFALO_OK;
}

buffalo_status buffalo_profile_end(double* ms_total_h, int64_t* launches_h, double* algo_bytes_h) {
  if (!g_prof.on) return BUFFALO_ERR_INVALID_ARG;
  const int64_t n = (int64_t)g_prof.fixed.size();
  std::vector<unsigned long long> edges(n > 0 ? n : 1, 0);
  BF_CUDA(cudaDeviceSynchronize());
  if (n > 0) BF_CUDA(cudaMemcpy(edges.data(), g_prof.counters, sizeof(unsigned long long) * n, cudaMemcpyDeviceToHost));
  double ms = 0.0, bytes = 0.0;
  for (int64_t i = 0; i < n; ++i) {
    float t = 0.f;
    BF_CUDA(cudaEventElapsedTime(&t, g_prof.ev[2 * i], g_prof.ev[2 * i + 1]));
    ms += t;
    bytes += g_prof.fixed[i] + g_prof.per_edge[i] * (double)edges[i];
  }
  if (ms_total_h) *ms_total_h = ms;
  if (launches_h) *launches_h = n;
  if (algo_bytes_h) *algo_bytes_h = bytes;
  for (cudaEvent_t e : g_prof.ev) cudaEventDestroy(e);
  g_prof = Profiler();
  return BUFFALO_OK;
}

// The IPC handle covers a whole driver allocation (a caching allocator sub-allocates tensors
// inside larger ones), so the exported handle carries the pointer's offset from its allocation
// base after the 64-byte cudaIpcMemHandle_t.
typedef CUresult (*MemGetAddressRangeFn)(CUdeviceptr*, size_t*, CUdeviceptr);

buffalo_status buffalo_ipc_export(const void* dev_ptr, void* handle_h) {
  if (!dev_ptr || !handle_h) {
    set_error("ipc_export: null argument");
    return BUFFALO_ERR_INVALID_ARG;
  }
  static_assert(sizeof(cudaIpcMemHandle_t) + 8 == BUFFALO_IPC_HANDLE_BYTES, "IPC handle size");
  void* fn = nullptr;
  cudaDriverEntryPointQueryResult q;
  BF_CUDA(cudaGetDriverEntryPoint("cuMemGetAddressRange", &fn, cudaEnableDefault, &q));
  if (!fn || q != cudaDriverEntryPointSuccess) {
    set_error("ipc_export: cuMemGetAddressRange unavailable");
    return BUFFALO_ERR_CUDA;
  }
  CUdeviceptr base = 0;
  size_t size = 0;
  if (((MemGetAddressRangeFn)fn)(&base, &size, (CUdeviceptr)dev_ptr) != CUDA_SUCCESS) {
    set_error("ipc_export: the pointer is not inside a device allocation");
    return BUFFALO_ERR_INVALID_ARG;
  }
  cudaIpcMemHandle_t hd;
  BF_CUDA(cudaIpcGetMemHandle(&hd, (void*)base));
  const uint64_t off = (uint64_t)((CUdeviceptr)dev_ptr - base);
  memcpy(handle_h, &hd, sizeof(hd));
  memcpy((char*)handle_h + sizeof(hd), &off, 8);
  return BUFFALO_OK;
}

buffalo_status buffalo_ipc_open(const void* handle_h, void** dev_ptr_out_h) {
  if (!handle_h || !dev_ptr_out_h) {
    set_error("ipc_open: null argument");
    return BUFFALO_ERR_INVALID_ARG;
  }
  cudaIpcMemHandle_t hd;
  uint64_t off = 0;
  memcpy(&hd, handle_h, sizeof(hd));
  memcpy(&off, (const char*)handle_h + sizeof(hd), 8);
  void* p = nullptr;
  BF_CUDA(cudaIpcOpenMemHandle(&p, hd, cudaIpcMemLazyEnablePeerAccess));
  *dev_ptr_out_h = (char*)p + off;
  return BUFFALO_OK;
}

buffalo_status buffalo_ipc_close(const void* handle_h, void* dev_ptr) {
  if (!handle_h || !dev_ptr) return BUFFALO_ERR_INVALID_ARG;
  uint64_t off = 0;
  memcpy(&off, (const char*)handle_h + sizeof(cudaIpcMemHandle_t), 8);
  BF_CUDA(cudaIpcCloseMemHandle((char*)dev_ptr - off));
  return BUFFALO_OK;
}

size_t buffalo_graph_workspace_bytes(int64_t num_nodes) { return (size_t)graph_ws_bytes(num_nodes); }

buffalo_status buffalo_graph_prepare(buffalo_graph* g, void* workspace, size_t bytes, void* stream) {
  BF_CHECK(require_sm100());
  if (!g || !workspace || !g->row_ptr || (!g->col && g->nnz > 0) || g->nnz < 0 || g->num_nodes <= 0) {
    set_error("graph_prepare: null graph/workspace, empty graph or col NULL with nnz > 0");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (g->num_nodes >= INT32_MAX) {
    set_error("graph_prepare: node ids are int32: num_nodes must be < 2^31 - 1");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if ((int64_t)bytes < (int64_t)buffalo_graph_workspace_bytes(g->num_nodes)) {
    set_error("graph_prepare: workspace of %lld bytes, need %lld", (long long)bytes,
              (long long)buffalo_graph_workspace_bytes(g->num_nodes));
    return BUFFALO_ERR_CAPACITY;
  }
  g->node_map = (int32_t*)workspace;
  cudaStream_t s = (cudaStream_t)stream;
  k_fill_i32<<<grid_for(g->num_nodes, 256), 256, 0, s>>>(g->node_map, g->num_nodes, INT32_MAX);
  BF_LAUNCHED("k_fill_i32");
  const GraphWs gw = graph_ws(g);
  BF_CUDA(cudaMemsetAsync(gw.bits, 0, sizeof(uint32_t) * gw.words, s));
  return BUFFALO_OK;
}

buffalo_status buffalo_graph_validate(const buffalo_graph* g, int32_t check_symmetric, void* stream) {
  BF_CHECK(require_sm100());
  if (!g || !g->node_map || !g->row_ptr || (!g->col && g->nnz > 0) || g->num_nodes <= 0 || g->nnz < 0) {
    set_error("graph_validate: null or unprepared graph");
    return BUFFALO_ERR_INVALID_ARG;
  }
  return validate_graph(g, check_symmetric ? 1 : 0, (cudaStream_t)stream);
}

buffalo_status buffalo_estimate_mem(int32_t num_layers, const int64_t* n, const int64_t* e,
                                    const buffalo_model* m, int64_t* lo_bytes_h, int64_t* hi_bytes_h) {
  if (!n || !e || !m || !lo_bytes_h || !hi_bytes_h || num_layers != m->num_layers) return BUFFALO_ERR_INVALID_ARG;
  BF_CHECK(validate_model(m));
  mem_model(num_layers, n, e, m, lo_bytes_h, hi_bytes_h);
  return BUFFALO_OK;
}

size_t buffalo_bucketize_workspace_bytes(const buffalo_graph* g, int64_t n_seeds,
                                         const buffalo_sampler* s, const buffalo_model* m) {
  if (!g || !s || !m) return 0;
  return (size_t)(bucketize_fixed_bytes(n_seeds, s->cutoff_F, 4096) + mask_stats_bytes(g->num_nodes, m->num_layers));
}

buffalo_status buffalo_bucketize(const buffalo_graph* g, const int32_t* seeds, int64_t S,
                                 const buffalo_sampler* sp, const buffalo_model* m,
                                 const buffalo_sched* sc, buffalo_plan* plan, void* workspace,
                                 size_t workspace_bytes, void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  const int L = m->num_layers;
  BF_CHECK(validate_sampler(sp, L));
  if (!g || !g->node_map || !seeds || S <= 0 || !sc || !plan || !workspace) {
    set_error("bucketize: null argument or empty seed set");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (sc->mem_budget <= 0 || sc->k_max < 1 || sc->k_max > 4096 || sc->num_gpus < 1 || sc->k_multiple < 0 ||
      sc->rank < 0 || sc->rank >= sc->num_gpus) {
    set_error("bucketize: bad scheduler parameters");
    return BUFFALO_ERR_INVALID_ARG;
  }
  cudaStream_t s = (cudaStream_t)stream;
  const int F = sp->cutoff_F;
  const int fL = sp->fanout[L - 1];
  // carve the workspace
  char* q = (char*)workspace;
  const int64_t pc = part_count_elems(S);
  uint8_t* bucket = (uint8_t*)q; q += R(S);
  int32_t* order = (int32_t*)q; q += R(4 * S);
  int32_t* sorted_ids = (int32_t*)q; q += R(4 * S);
  int32_t* counts = (int32_t*)q; q += R(4 * (pc + 1));
  int32_t* ws = (int32_t*)q; q += R(4 * scan_ws_elems(pc + 1));
  int32_t* starts = (int32_t*)q; q += R(4 * 258);
  int64_t* segs = (int64_t*)q; q += R(32 * (int64_t)(256 + 4096 + 1));
  const int64_t used = q - (char*)workspace;
  if (used > (int64_t)workspace_bytes) {
    set_error("bucketize workspace too small");
    return BUFFALO_ERR_CAPACITY;
  }
  char* stats_ws = q;
  const int64_t stats_bytes = (int64_t)workspace_bytes - used;

  // shared statistics (include/buffalo.h buffalo_sched.allgather): no rank visits the whole
  // receptive field, so the per-rank sample cache cannot be filled; every pass samples
  const bool shared = sc->allgather && sc->num_gpus > 1;
  buffalo_sampler sp_local = *sp;
  if (shared)
    for (auto& c : sp_local.cache) c = nullptr;
  sp = &sp_local;
  // a1: DegreeBucketing (Alg. 3 l.1); validates the seed ids (in range, distinct).  The plan's
  // outputs are written only once a K succeeded (outputs untouched on error).
  std::vector<int64_t> hist(F + 1, 0);
  BF_CHECK(seed_bucketing(g, seeds, S, fL, F, bucket, order, sorted_ids, counts, ws, starts, hist.data(), s));
  std::vector<int64_t> bstart(F + 2, 0);
  for (int b = 0; b <= F; ++b) bstart[b + 1] = bstart[b] + hist[b];

  // a2: per-bucket statistics and estimates (K-independent); item k = degree bucket k
  bool masks_clean = false;
  std::vector<Item> bucket_item(F + 1);
  std::vector<Item*> todo;
  for (int d = 0; d <= F; ++d) {
    bucket_item[d] = Item{d, 0, bstart[d], hist[d], 0, 0, 0, 0, 0};
    if (hist[d] > 0) todo.push_back(&bucket_item[d]);
  }
  // the first statistics pass (every seed) fills the sample cache; later passes read it
  BF_CHECK(items_stats_shared(g, sorted_ids, todo, sp, m, sc, stats_ws, stats_bytes, masks_clean, s, 1));
  std::vector<int> non_split;
  int64_t sum_M_all = 0, sum_w = 0, max_w = 0;
  for (int d = 0; d <= F; ++d) {
    if (hist[d] == 0) continue;
    Item& it = bucket_item[d];
    it.w = grouping_weight(it.M, it.I, it.E, sc->C_ppm);
    sum_M_all += it.M;
    if (d != F) {
      non_split.push_back(d);
      sum_w += it.w;
      max_w = std::max(max_w, it.w);
    }
  }
  const bool hasF = hist[F] > 0;

  // a3: the K loop (Alg. 3) with MemBalancedGrouping (Alg. 4).  The micro-bucket statistics
  // of several consecutive K candidates are computed in one statistics pass (their pieces
  // overlap, each seed carries one bit per candidate); the loop itself stays sequential.
  const int k_lo = std::max(std::max(sc->k_min, sc->num_gpus), 1);
  // R31: with k_multiple > 1 only multiples of it are candidates (every rank gets K / #GPUs groups)
  auto candidate = [&](int K) { return sc->k_multiple <= 1 || K % sc->k_multiple == 0; };
  auto needs_split = [&](int K) {
    if (!candidate(K)) return false;
    if (max_w > sc->mem_budget) return false;
    if ((__int128)sum_w > (__int128)K * sc->mem_budget) return false;
    return hasF && K >= 2 && (__int128)bucket_item[F].M * K > (__int128)sum_M_all;
  };
  std::vector<std::vector<Item>> piece_cache(sc->k_max + 1);
  std::vector<char> have(sc->k_max + 1, 0);
  for (int K = k_lo; K <= sc->k_max; ++K) {
    if (!candidate(K)) continue;
    if (max_w > sc->mem_budget) break;                         // R25: fails for every K
    if ((__int128)sum_w > (__int128)K * sc->mem_budget) continue;  // R25: some group exceeds M_ctr
    std::vector<Item> items;
    for (int d : non_split) items.push_back(bucket_item[d]);
    bool exploded = false;
    if (hasF) {
      const Item& itF = bucket_item[F];
      exploded = K >= 2 && (__int128)itF.M * K > (__int128)sum_M_all;   // R7
      if (exploded) {
        if (!have[K]) {
          // batch this and the following candidates that will need a split (<= 256 pieces)
          std::vector<int> ks;
          int total = 0;
          for (int K2 = K; K2 <= sc->k_max && total < kStatsBatch; ++K2) {
            if (!needs_split(K2)) continue;
            const int np = (int)std::min<int64_t>(K2, itF.count);
            if (total + np > kStatsBatch && !ks.empty()) break;
            ks.push_back(K2);
            total += np;
          }
          std::vector<Item*> ptrs;
          for (int K2 : ks) {
            piece_cache[K2] = split_pieces(itF, F, K2);
            have[K2] = 1;
          }
          for (int K2 : ks)
            for (Item& it : piece_cache[K2]) ptrs.push_back(&it);
          BF_CHECK(items_stats_shared(g, sorted_ids, ptrs, sp, m, sc, stats_ws, stats_bytes, masks_clean, s, 2));
        }
        for (Item it : piece_cache[K]) {
          it.w = grouping_weight(it.M, it.I, it.E, sc->C_ppm);
          items.push_back(it);
        }
      } else {
        items.push_back(itF);
      }
    }
    // Alg. 4: sort by M_est descending (ties: degree asc, micro index asc), place each item
    // into the group with the lowest Eq. 2 estimate (ties: lowest index).
    std::vector<int> idx(items.size());
    for (size_t i = 0; i < idx.size(); ++i) idx[i] = (int)i;
    std::sort(idx.begin(), idx.end(), [&](int a, int b) {
      if (items[a].M != items[b].M) return items[a].M > items[b].M;
      if (items[a].d != items[b].d) return items[a].d < items[b].d;
      return items[a].k < items[b].k;
    });
    std::vector<int64_t> load(K, 0);
    std::vector<std::vector<int>> members(K);
    for (int i : idx) {
      int best = 0;
      for (int k = 1; k < K; ++k)
        if (load[k] < load[best]) best = k;
      members[best].push_back(i);
      load[best] += items[i].w;
    }
    int64_t mx = 0;
    for (int k = 0; k < K; ++k) mx = std::max(mx, load[k]);
    if (mx > sc->mem_budget) continue;

    // success: emit the plan (empty groups dropped, R17)
    std::vector<int64_t> seg;
    std::vector<int64_t> offs(1, 0), est;
    int gk = 0;
    for (int k = 0; k < K; ++k) {
      if (members[k].empty()) continue;
      std::vector<int> mem = members[k];
      std::sort(mem.begin(), mem.end(), [&](int a, int b) {
        if (items[a].d != items[b].d) return items[a].d < items[b].d;
        return items[a].k < items[b].k;
      });
      int64_t off = offs.back();
      for (int i : mem) {
        seg.push_back(items[i].start);
        seg.push_back(items[i].count);
        seg.push_back(gk);
        seg.push_back(off);
        off += items[i].count;
      }
      offs.push_back(off);
      est.push_back(load[k]);
      ++gk;
    }
    const int nseg = (int)(seg.size() / 4);
    BF_CUDA(cudaMemcpyAsync(segs, seg.data(), seg.size() * sizeof(int64_t), cudaMemcpyHostToDevice, s));
    k_scatter_segments<<<nseg, 256, 0, s>>>(segs, order, sorted_ids, plan->group_seeds, plan->group_of_seed);
    BF_LAUNCHED("k_scatter_segments");
    BF_CUDA(cudaMemcpyAsync(plan->group_offsets, offs.data(), offs.size() * sizeof(int64_t),
                            cudaMemcpyHostToDevice, s));
    for (int k = 0; k <= gk; ++k) plan->group_offsets_h[k] = offs[k];
    // LPT assignment of groups to ranks (R24)
    std::vector<int> gi(gk);
    for (int k = 0; k < gk; ++k) gi[k] = k;
    std::sort(gi.begin(), gi.end(), [&](int a, int b) { return est[a] != est[b] ? est[a] > est[b] : a < b; });
    std::vector<int64_t> rload(sc->num_gpus, 0);
    for (int k : gi) {
      int best = 0;
      for (int r = 1; r < sc->num_gpus; ++r)
        if (rload[r] < rload[best]) best = r;
      plan->rank_of_group_h[k] = best;
      rload[best] += est[k];
    }
    for (int k = 0; k < gk; ++k) plan->est_bytes_h[k] = est[k];
    if (plan->group_sizes_h) {
      // exact block sizes of this rank's groups (groups as items of the mask statistics), so
      // that buffalo_build_blocks can lay out the arena up front and run without host round
      // trips; the rows of other ranks' groups are set to -1 (each rank measures its own)
      const int W = 2 * L + 1;
      std::vector<Item> gitems;
      std::vector<int> gidx;
      for (int k = 0; k < gk; ++k) {
        int64_t* row = plan->group_sizes_h + (int64_t)k * W;
        if (sc->num_gpus > 1 && plan->rank_of_group_h[k] != sc->rank) {
          for (int c = 0; c < W; ++c) row[c] = -1;
          continue;
        }
        gitems.push_back(Item{0, k, offs[k], offs[k + 1] - offs[k], 0, 0, 0, 0, 0});
        gidx.push_back(k);
      }
      std::vector<Item*> gp;
      for (Item& it : gitems) gp.push_back(&it);
      std::vector<int64_t> sizes;
      BF_CHECK(items_sizes(g, plan->group_seeds, gp, sp, L, stats_ws, stats_bytes, masks_clean, s, 2, sizes));
      for (size_t j = 0; j < gidx.size(); ++j)
        std::copy(sizes.begin() + j * W, sizes.begin() + (j + 1) * W, plan->group_sizes_h + (int64_t)gidx[j] * W);
    }
    for (int d = 0; d <= F; ++d) plan->hist_h[d] = hist[d];
    plan->k_out = gk;
    plan->k_tried = K;
    plan->exploded = exploded ? 1 : 0;
    plan->num_items = (int)items.size();
    BF_CUDA(cudaStreamSynchronize(s));
    return BUFFALO_OK;
  }
  set_error("Buffalo scheduler: no K in [%d, %d] satisfies M_ctr = %lld", k_lo, sc->k_max,
            (long long)sc->mem_budget);
  return BUFFALO_ERR_BUDGET;
}

buffalo_status buffalo_build_blocks(const buffalo_graph* g, const int32_t* group_seeds, int64_t n,
                                    const buffalo_sampler* sp, const buffalo_model* m,
                                    buffalo_blocks* out, void* arena, size_t arena_bytes,
                                    int64_t* required_bytes_h, const int64_t* sizes_h, void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  const int L = m->num_layers;
  BF_CHECK(validate_sampler(sp, L));
  if (!g || !g->node_map || !group_seeds || n <= 0 || !out || !arena) {
    set_error("build_blocks: null argument or empty group");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (m->feat_shards) {
    if ((int64_t)m->feat_shards->num_shards * m->feat_shards->rows_per_shard < g->num_nodes) {
      set_error("build_blocks: the feature shards cover fewer rows than the graph has nodes");
      return BUFFALO_ERR_INVALID_ARG;
    }
    if (sp->fanout[0] <= 0) {
      set_error("build_blocks: a sharded feature table needs a sampled first block (fanout[0] > 0)");
      return BUFFALO_ERR_UNSUPPORTED;
    }
  }
  if (((uintptr_t)arena) % 256) {
    set_error("build_blocks: arena must be 256-B aligned");
    return BUFFALO_ERR_INVALID_ARG;
  }
  cudaStream_t s = (cudaStream_t)stream;
  if (sizes_h) {
    // sizes from the plan: validate, then check the whole arena need (R15: lo = exact) up front
    if (sizes_h[L] != n) {
      set_error("build_blocks: sizes_h[L] = %lld != n = %lld", (long long)sizes_h[L], (long long)n);
      return BUFFALO_ERR_INVALID_ARG;
    }
    for (int l = 0; l <= 2 * L; ++l)
      if (sizes_h[l] < 0 || sizes_h[l] > INT32_MAX) {
        set_error("build_blocks: bad sizes_h");
        return BUFFALO_ERR_INVALID_ARG;
      }
    int64_t lo, hi;
    mem_model(L, sizes_h, sizes_h + L + 1, m, &lo, &hi);
    if (lo > (int64_t)arena_bytes) {
      if (required_bytes_h) *required_bytes_h = lo;
      set_error("build_blocks: arena of %lld bytes too small (need %lld)", (long long)arena_bytes, (long long)lo);
      return BUFFALO_ERR_CAPACITY;
    }
  }
  if (!sizes_h) {
    // the read-back path synchronises anyway: validate the group's ids first (in range,
    // distinct); with sizes_h the group comes from a plan whose seeds buffalo_bucketize checked
    int32_t* err_dev = graph_ws(g).scan_ws;
    BF_CUDA(cudaMemsetAsync(err_dev, 0, sizeof(int32_t), s));
    BF_CHECK(check_ids(g, group_seeds, n, err_dev, s));
    int32_t err = 0;
    BF_CUDA(cudaMemcpyAsync(&err, err_dev, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    BF_CUDA(cudaStreamSynchronize(s));
    BF_CHECK(ids_error(err, "build_blocks"));
  }
  buffalo_blocks* const user_out = out;     // written only on success (outputs untouched on error)
  buffalo_blocks local;
  out = &local;
  memset(out, 0, sizeof(*out));
  out->num_layers = L;
  Arena A;
  A.base = (char*)arena;
  A.cap = (int64_t)arena_bytes;
  const int32_t* dst = group_seeds;
  int64_t nd = n;
  int64_t nn[BUFFALO_MAX_LAYERS + 1], ee[BUFFALO_MAX_LAYERS];
  for (int l = L; l >= 1; --l) {
    buffalo_block* b = &out->layer[l - 1];
    int64_t known[2];
    if (sizes_h) {
      known[0] = sizes_h[L + l];      // e_l
      known[1] = sizes_h[l - 1];      // n_{l-1}
    }
    buffalo_status st = build_layer(g, dst, nd, sp->fanout[l - 1], (uint32_t)(L - l + 1), sp->seed, l,
                                    false, A, b, s, sizes_h ? known : nullptr,
                                    m->aggregator == BUFFALO_AGG_POOL || m->aggregator == BUFFALO_AGG_GAT,
                                    sp->fanout[l - 1] > 0 ? sp->cache[l - 1] : nullptr,
                                    // the mean model walks sampled blocks in natural order: no
                                    // degree-class permutation (no row exceeds the fanout)
                                    !(m->aggregator == BUFFALO_AGG_MEAN && sp->fanout[l - 1] > 0));
    if (st == BUFFALO_ERR_CAPACITY || A.overflow) {
      if (required_bytes_h) *required_bytes_h = A.need;
      set_error("build_blocks: arena of %lld bytes too small (need >= %lld)", (long long)A.cap,
                (long long)A.need);
      cudaStreamSynchronize(s);
      return BUFFALO_ERR_CAPACITY;
    }
    BF_CHECK(st);
    nn[l] = nd;
    ee[l - 1] = b->n_edges;
    dst = b->src_global;
    nd = b->n_src;
  }
  nn[0] = nd;
  // activations (R20): saved h_agg per layer, H_l (l < L), logits
  const int64_t sa = m->gemm_mode == BUFFALO_GEMM_BF16 ? 2 : 4;
  for (int l = 1; l <= L; ++l) {
    buffalo_block* b = &out->layer[l - 1];
    b->ld_agg = pitch_of(m->dim[l - 1]);
    b->agg = m->aggregator == BUFFALO_AGG_GAT ? nullptr : A.take(b->n_dst * b->ld_agg * sa);
    b->ld_out = pitch_of(m->dim[l]);
    b->out = A.take(b->n_dst * b->ld_out * (l < L ? sa : 4));
  }
  if (m->feat_shards) {
    buffalo_block* b = &out->layer[0];
    b->ld_self = pitch_of(m->dim[0]);
    b->self_rows = A.take(b->n_dst * b->ld_self * 2);
  }
  if (m->aggregator == BUFFALO_AGG_POOL)
    for (int l = 1; l <= L; ++l) {
      buffalo_block* b = &out->layer[l - 1];
      b->ld_pool = pitch_of(m->dim[l - 1]);
      b->pool_P = (float*)A.take(b->n_src * b->ld_pool * 4);
      b->pool_arg = (int32_t*)A.take(b->n_dst * b->ld_pool * 4);
    }
  if (m->aggregator == BUFFALO_AGG_GAT)
    for (int l = 1; l <= L; ++l) {
      buffalo_block* b = &out->layer[l - 1];
      b->agg_saved_bytes = gat_saved_bytes(b->n_src, b->n_dst, b->n_edges, m->dim[l]);
      b->agg_saved = A.take(b->agg_saved_bytes);
    }
  if (m->aggregator == BUFFALO_AGG_LSTM)
    for (int l = 1; l <= L; ++l) {
      buffalo_block* b = &out->layer[l - 1];
      b->agg_saved_bytes = R(lstm_saved_bytes(b->n_dst, b->n_edges, m->dim[l - 1]));
      b->agg_saved = A.take(b->agg_saved_bytes);
    }
  // backward region: ping-pong dH buffers at the two ends, scratch in between
  int64_t B = 0;
  std::vector<int64_t> ah(L + 1, 0), tmp(L + 1, 0);
  for (int l = 1; l <= L; ++l) ah[l] = dh_slot_bytes(m, nn[l], l);
  for (int l = L; l >= 1; --l) {
    tmp[l] = bwd_scratch_for(m, nn[l], nn[l - 1], ee[l - 1], l);
    B = std::max(B, ah[l] + (l >= 2 ? ah[l - 1] : 0) + tmp[l]);
  }
  char* region = (char*)A.take(B);
  if (A.overflow) {
    if (required_bytes_h) *required_bytes_h = A.need;
    set_error("build_blocks: arena of %lld bytes too small (need %lld)", (long long)A.cap, (long long)A.need);
    return BUFFALO_ERR_CAPACITY;
  }
  for (int l = L; l >= 1; --l) {
    buffalo_block* b = &out->layer[l - 1];
    const bool low = ((L - l) % 2) == 0;        // dH_L at the low end, dH_{L-1} at the high end, ...
    b->dh = (float*)(low ? region : region + B - ah[l]);
    b->ld_dh = pitch_of(m->dim[l]);
    b->bwd_scratch = low ? region + ah[l] : region + (l >= 2 ? ah[l - 1] : 0);
    b->bwd_scratch_bytes = tmp[l];
  }
  out->arena_used = A.bottom;
  out->arena_peak = A.peak;
  mem_model(L, nn, ee, m, &out->est_lo, &out->est_hi);
  if (required_bytes_h) *required_bytes_h = A.peak;
  *user_out = local;
  return BUFFALO_OK;
}

size_t buffalo_packed_weight_bytes(const buffalo_model* m, int32_t layer) {
  if (!m || layer < 1 || layer > m->num_layers) return 0;
  const int64_t din = m->dim[layer - 1], dout = m->dim[layer];
  int64_t b = R(2 * din * dout * 4);
  if (m->gemm_mode == BUFFALO_GEMM_BF16) b += tc_packed_bytes(din, dout);
  return (size_t)b;
}

buffalo_status buffalo_pack_weights(const buffalo_model* m, int32_t layer, const float* W, void* packed,
                                    void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (layer < 1 || layer > m->num_layers || !W || !packed) return BUFFALO_ERR_INVALID_ARG;
  cudaStream_t s = (cudaStream_t)stream;
  const int din = m->dim[layer - 1], dout = m->dim[layer];
  BF_CHECK(launch_transpose_w(W, dout, 2 * din, (float*)packed, s));
  if (m->gemm_mode == BUFFALO_GEMM_BF16)
    BF_CHECK(tc_pack_weights(W, din, dout, (char*)packed + R((int64_t)2 * din * dout * 4), s));
  return BUFFALO_OK;
}

buffalo_status buffalo_sage_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                const void* h_src, int64_t ld_src, const float* W, const void* W_packed,
                                const float* b, void* out, int64_t ld_out, void* saved_agg,
                                int64_t ld_agg, void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (m->aggregator != BUFFALO_AGG_MEAN) {
    set_error("sage_fwd: model.aggregator is not MEAN (use buffalo_pool_fwd)");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (!blk || layer < 1 || layer > m->num_layers || !h_src || !W || !W_packed || !out || !saved_agg) {
    set_error("sage_fwd: null argument or bad layer");
    return BUFFALO_ERR_INVALID_ARG;
  }
  FwdArgs a{};
  a.blk = blk;
  a.layer1 = layer == 1;
  const bool act_bf16 = m->gemm_mode == BUFFALO_GEMM_BF16;
  a.in_bf16 = a.layer1 ? m->feat_dtype == BUFFALO_BF16 : act_bf16;
  a.act_bf16 = act_bf16;
  a.out_f32 = layer == m->num_layers;
  a.relu = layer < m->num_layers;
  a.d_in = m->dim[layer - 1];
  a.d_out = m->dim[layer];
  a.h_src = h_src;
  a.ld_src = a.layer1 ? m->feat_pitch : ld_src;
  a.W = W;
  a.W_packed = W_packed;
  a.b = b;
  a.out = out;
  a.ld_out = ld_out;
  a.agg = saved_agg;
  a.ld_agg = ld_agg;
  if (a.layer1 && !blk->col_global) return BUFFALO_ERR_INVALID_ARG;
  if (a.layer1 && m->feat_shards) {
    if (!blk->self_rows || blk->fanout <= 0 || blk->fanout > 128) {
      set_error("sage_fwd: sharded features need block 1 built with the sharded model and a sampled fanout");
      return BUFFALO_ERR_INVALID_ARG;
    }
    a.shards = m->feat_shards;
  }
  if (ld_out < pitch_of(a.d_out) || ld_agg < pitch_of(a.d_in) || a.ld_src < pitch_of(a.d_in) ||
      ld_out % 8 || ld_agg % 8 || a.ld_src % 8) {
    set_error("sage_fwd: leading dimensions must be multiples of 8 and >= the padded widths");
    return BUFFALO_ERR_INVALID_ARG;
  }
  cudaStream_t s = (cudaStream_t)stream;
  if (m->gemm_mode == BUFFALO_GEMM_BF16 && tc_fwd_supported(a)) return tc_sage_fwd(a, s);
  return sage_fwd_ffma(a, s);
}

size_t buffalo_sage_bwd_scratch_bytes(const buffalo_block* blk, int32_t layer, const buffalo_model* m) {
  if (!blk || !m || layer < 1 || layer > m->num_layers) return 0;
  return (size_t)bwd_scratch_for(m, blk->n_dst, blk->n_src, blk->n_edges, layer);
}

buffalo_status buffalo_sage_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                float* dh_dst, int64_t ld_dh, const void* h_src, int64_t ld_src,
                                const void* saved_agg, int64_t ld_agg, const void* h_dst,
                                int64_t ld_hdst, const float* W, const void* W_packed, float* dW_accum,
                                float* db_accum, float* dh_src, int64_t ld_dh_src,
                                void* scratch, size_t scratch_bytes, void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (m->aggregator != BUFFALO_AGG_MEAN) {
    set_error("sage_bwd: model.aggregator is not MEAN (use buffalo_pool_bwd)");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (!blk || layer < 1 || layer > m->num_layers || !dh_dst || !h_src || !saved_agg || !W ||
      !dW_accum || !db_accum || !scratch) {
    set_error("sage_bwd: null argument or bad layer");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (layer < m->num_layers && !h_dst) return BUFFALO_ERR_INVALID_ARG;
  if (dh_src && (layer == 1 || !blk->t_row_ptr)) {
    set_error("sage_bwd: dh_src needs a transposed block (layer >= 2)");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if ((int64_t)scratch_bytes < (int64_t)buffalo_sage_bwd_scratch_bytes(blk, layer, m)) return BUFFALO_ERR_CAPACITY;
  BwdArgs a{};
  a.blk = blk;
  a.layer1 = layer == 1;
  const bool act_bf16 = m->gemm_mode == BUFFALO_GEMM_BF16;
  a.in_bf16 = a.layer1 ? m->feat_dtype == BUFFALO_BF16 : act_bf16;
  a.act_bf16 = act_bf16;
  a.last = layer == m->num_layers;
  a.d_in = m->dim[layer - 1];
  a.d_out = m->dim[layer];
  a.dh = dh_dst;
  a.ld_dh = ld_dh;
  a.h_src = h_src;
  a.ld_src = a.layer1 ? m->feat_pitch : ld_src;
  a.agg = saved_agg;
  a.ld_agg = ld_agg;
  a.h_dst = h_dst;
  a.ld_hdst = ld_hdst;
  a.W = W;
  a.W_packed = W_packed;
  a.dW = dW_accum;
  a.db = db_accum;
  a.dh_src = dh_src;
  a.ld_dh_src = ld_dh_src;
  a.scratch = scratch;
  a.scratch_bytes = (int64_t)scratch_bytes;
  if (a.layer1 && m->feat_shards) {
    if (!blk->self_rows) {
      set_error("sage_bwd: sharded features need block 1 built with the sharded model");
      return BUFFALO_ERR_INVALID_ARG;
    }
    a.shards = m->feat_shards;
  }
  cudaStream_t s = (cudaStream_t)stream;
  if (m->gemm_mode == BUFFALO_GEMM_BF16) {
    if (!tc_bwd_supported(a)) return BUFFALO_ERR_UNSUPPORTED;
    return tc_sage_bwd(a, s);
  }
  return sage_bwd_ffma(a, s);
}

static buffalo_status pool_args(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                 const void* h_src, int64_t ld_src, PoolArgs& a, const char* who) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (m->aggregator != BUFFALO_AGG_POOL) {
    set_error("%s: model.aggregator is not BUFFALO_AGG_POOL", who);
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (!blk || layer < 1 || layer > m->num_layers || !h_src) {
    set_error("%s: null argument or bad layer", who);
    return BUFFALO_ERR_INVALID_ARG;
  }
  a = PoolArgs{};
  a.blk = blk;
  a.layer1 = layer == 1;
  a.in_bf16 = a.layer1 && m->feat_dtype == BUFFALO_BF16;
  a.last = layer == m->num_layers;
  a.d_in = m->dim[layer - 1];
  a.d_out = m->dim[layer];
  a.h_src = h_src;
  a.ld_src = a.layer1 ? m->feat_pitch : ld_src;
  if (a.ld_src < pitch_of(a.d_in) || a.ld_src % 8) {
    set_error("%s: ld_src must be a multiple of 8 and >= pitch(d_in)", who);
    return BUFFALO_ERR_INVALID_ARG;
  }
  return BUFFALO_OK;
}

buffalo_status buffalo_pool_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                const void* h_src, int64_t ld_src, const float* W_pool, const float* b_pool,
                                const float* W, const void* W_packed, const float* b, void* out, int64_t ld_out,
                                void* saved_agg, int64_t ld_agg, float* P, int32_t* arg, int64_t ld_pool,
                                void* stream) {
  PoolArgs a;
  BF_CHECK(pool_args(blk, layer, m, h_src, ld_src, a, "pool_fwd"));
  if (!W_pool || !b_pool || !W || !W_packed || !b || !out || !saved_agg || !P || !arg) {
    set_error("pool_fwd: null argument");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (ld_out < pitch_of(a.d_out) || ld_agg < pitch_of(a.d_in) || ld_pool < pitch_of(a.d_in) || ld_out % 8 ||
      ld_agg % 8 || ld_pool % 8) {
    set_error("pool_fwd: leading dimensions must be multiples of 8 and >= the padded widths");
    return BUFFALO_ERR_INVALID_ARG;
  }
  a.W_pool = W_pool;
  a.b_pool = b_pool;
  a.W = W;
  a.W_packed = (const float*)W_packed;
  a.b = b;
  a.out = (float*)out;
  a.ld_out = ld_out;
  a.agg = (float*)saved_agg;
  a.ld_agg = ld_agg;
  a.P = P;
  a.arg = arg;
  a.ld_pool = ld_pool;
  return pool_fwd_ffma(a, (cudaStream_t)stream);
}

buffalo_status buffalo_pool_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                float* dh_dst, int64_t ld_dh, const void* h_src, int64_t ld_src,
                                const void* saved_agg, int64_t ld_agg, const void* h_dst, int64_t ld_hdst,
                                const float* P, const int32_t* arg, int64_t ld_pool, const float* W_pool,
                                const float* W, float* dW_pool_accum, float* db_pool_accum, float* dW_accum,
                                float* db_accum, float* dh_src, int64_t ld_dh_src, void* scratch,
                                size_t scratch_bytes, void* stream) {
  PoolArgs a;
  BF_CHECK(pool_args(blk, layer, m, h_src, ld_src, a, "pool_bwd"));
  if (!dh_dst || !saved_agg || !P || !arg || !W_pool || !W || !dW_pool_accum || !db_pool_accum || !dW_accum ||
      !db_accum || !scratch || (!a.last && !h_dst)) {
    set_error("pool_bwd: null argument");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (!blk->t_row_ptr || !blk->t_col) {
    set_error("pool_bwd: the block has no transpose (build it with model.aggregator = POOL)");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (dh_src && layer == 1) {
    set_error("pool_bwd: no dh_src at layer 1 (features are not trained)");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if ((int64_t)scratch_bytes < pool_bwd_scratch_bytes(blk->n_dst, blk->n_src, a.d_in, a.d_out)) {
    set_error("pool_bwd: scratch too small");
    return BUFFALO_ERR_CAPACITY;
  }
  a.dh = dh_dst;
  a.ld_dh = ld_dh;
  a.agg = (float*)saved_agg;
  a.ld_agg = ld_agg;
  a.h_dst = (const float*)h_dst;
  a.ld_hdst = ld_hdst;
  a.P = (float*)P;
  a.arg = (int32_t*)arg;
  a.ld_pool = ld_pool;
  a.W_pool = W_pool;
  a.W = W;
  a.dW_pool = dW_pool_accum;
  a.db_pool = db_pool_accum;
  a.dW = dW_accum;
  a.db = db_accum;
  a.dh_src = dh_src;
  a.ld_dh_src = ld_dh_src;
  a.scratch = scratch;
  a.scratch_bytes = (int64_t)scratch_bytes;
  return pool_bwd_ffma(a, (cudaStream_t)stream);
}

static buffalo_status lstm_args(const buffalo_block* blk, int32_t layer, const buffalo_model* m,
                                 const void* h_src, int64_t ld_src, void* saved, size_t saved_bytes, LstmArgs& a,
                                 const char* who) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (m->aggregator != BUFFALO_AGG_LSTM) {
    set_error("%s: model.aggregator is not BUFFALO_AGG_LSTM", who);
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (!blk || layer < 1 || layer > m->num_layers || !h_src || !saved || !blk->cls_perm) {
    set_error("%s: null argument or bad layer", who);
    return BUFFALO_ERR_INVALID_ARG;
  }
  if ((int64_t)saved_bytes < lstm_saved_bytes(blk->n_dst, blk->n_edges, m->dim[layer - 1])) {
    set_error("%s: lstm_saved too small", who);
    return BUFFALO_ERR_CAPACITY;
  }
  a = LstmArgs{};
  a.blk = blk;
  a.layer1 = layer == 1;
  a.in_bf16 = a.layer1 && m->feat_dtype == BUFFALO_BF16;
  a.last = layer == m->num_layers;
  a.d_in = m->dim[layer - 1];
  a.d_out = m->dim[layer];
  a.h_src = h_src;
  a.ld_src = a.layer1 ? m->feat_pitch : ld_src;
  a.saved = saved;
  if (a.ld_src < pitch_of(a.d_in) || a.ld_src % 8) {
    set_error("%s: ld_src must be a multiple of 8 and >= pitch(d_in)", who);
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (a.layer1 && !blk->col_global) return BUFFALO_ERR_INVALID_ARG;
  return BUFFALO_OK;
}

buffalo_status buffalo_lstm_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m, const void* h_src,
                                int64_t ld_src, const float* W_ih, const float* W_hh, const float* b_lstm,
                                const float* W, const void* W_packed, const float* b, void* out, int64_t ld_out,
                                void* saved_agg, int64_t ld_agg, void* lstm_saved, size_t lstm_saved_bytes,
                                void* stream) {
  LstmArgs a;
  BF_CHECK(lstm_args(blk, layer, m, h_src, ld_src, lstm_saved, lstm_saved_bytes, a, "lstm_fwd"));
  if (!W_ih || !W_hh || !b_lstm || !W || !W_packed || !b || !out || !saved_agg) {
    set_error("lstm_fwd: null argument");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (ld_out < pitch_of(a.d_out) || ld_agg < pitch_of(a.d_in) || ld_out % 8 || ld_agg % 8) {
    set_error("lstm_fwd: leading dimensions must be multiples of 8 and >= the padded widths");
    return BUFFALO_ERR_INVALID_ARG;
  }
  a.W_ih = W_ih;
  a.W_hh = W_hh;
  a.b_lstm = b_lstm;
  a.W = W;
  a.W_packed = (const float*)W_packed;
  a.b = b;
  a.out = (float*)out;
  a.ld_out = ld_out;
  a.agg = (float*)saved_agg;
  a.ld_agg = ld_agg;
  return lstm_fwd_ffma(a, (cudaStream_t)stream);
}

buffalo_status buffalo_lstm_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m, float* dh_dst,
                                int64_t ld_dh, const void* h_src, int64_t ld_src, const void* saved_agg,
                                int64_t ld_agg, const void* h_dst, int64_t ld_hdst, void* lstm_saved,
                                size_t lstm_saved_bytes, const float* W_ih, const float* W_hh, const float* W,
                                float* dW_ih_accum, float* dW_hh_accum, float* db_lstm_accum, float* dW_accum,
                                float* db_accum, float* dh_src, int64_t ld_dh_src, void* scratch,
                                size_t scratch_bytes, void* stream) {
  LstmArgs a;
  BF_CHECK(lstm_args(blk, layer, m, h_src, ld_src, lstm_saved, lstm_saved_bytes, a, "lstm_bwd"));
  if (!dh_dst || !saved_agg || !W_ih || !W_hh || !W || !dW_ih_accum || !dW_hh_accum || !db_lstm_accum ||
      !dW_accum || !db_accum || !scratch || (!a.last && !h_dst)) {
    set_error("lstm_bwd: null argument");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if (dh_src && (layer == 1 || !blk->t_row_ptr)) {
    set_error("lstm_bwd: dh_src needs a transposed block (layer >= 2)");
    return BUFFALO_ERR_INVALID_ARG;
  }
  if ((int64_t)scratch_bytes < lstm_bwd_scratch_bytes(blk->n_dst, blk->n_edges, layer, a.d_in, a.d_out)) {
    set_error("lstm_bwd: scratch too small");
    return BUFFALO_ERR_CAPACITY;
  }
  a.dh = dh_dst;
  a.ld_dh = ld_dh;
  a.agg = (float*)saved_agg;
  a.ld_agg = ld_agg;
  a.h_dst = (const float*)h_dst;
  a.ld_hdst = ld_hdst;
  a.W_ih = W_ih;
  a.W_hh = W_hh;
  a.W = W;
  a.dW_ih = dW_ih_accum;
  a.dW_hh = dW_hh_accum;
  a.db_lstm = db_lstm_accum;
  a.dW = dW_accum;
  a.db = db_accum;
  a.dh_src = dh_src;
  a.ld_dh_src = ld_dh_src;
  a.scratch = scratch;
  return lstm_bwd_ffma(a, (cudaStream_t)stream);
}

buffalo_status buffalo_gat_fwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m, const void* h_src,
                               int64_t ld_src, const float* W, const float* a_l, const float* a_r, const float* b,
                               void* out, int64_t ld_out, void* gat_saved, size_t gat_saved_bytes, void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (m->aggregator != BUFFALO_AGG_GAT) {
    set_error("gat_fwd: model.aggregator is not BUFFALO_AGG_GAT");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (!blk || layer < 1 || layer > m->num_layers || !h_src || !W || !a_l || !a_r || !b || !out || !gat_saved ||
      !blk->cls_perm) {
    set_error("gat_fwd: null argument or bad layer");
    return BUFFALO_ERR_INVALID_ARG;
  }
  GatArgs a{};
  a.blk = blk;
  a.layer1 = layer == 1;
  a.in_bf16 = a.layer1 && m->feat_dtype == BUFFALO_BF16;
  a.last = layer == m->num_layers;
  a.d_in = m->dim[layer - 1];
  a.d_out = m->dim[layer];
  a.h_src = h_src;
  a.ld_src = a.layer1 ? m->feat_pitch : ld_src;
  if ((int64_t)gat_saved_bytes < buffalo::gat_saved_bytes(blk->n_src, blk->n_dst, blk->n_edges, a.d_out) ||
      ld_out < pitch_of(a.d_out) || ld_out % 8 || a.ld_src < pitch_of(a.d_in) || a.ld_src % 8) {
    set_error("gat_fwd: saved region too small or bad leading dimensions");
    return BUFFALO_ERR_INVALID_ARG;
  }
  a.W = W;
  a.a_l = a_l;
  a.a_r = a_r;
  a.b = b;
  a.out = (float*)out;
  a.ld_out = ld_out;
  a.saved = gat_saved;
  return gat_fwd_ffma(a, (cudaStream_t)stream);
}

buffalo_status buffalo_gat_bwd(const buffalo_block* blk, int32_t layer, const buffalo_model* m, float* dh_dst,
                               int64_t ld_dh, const void* h_src, int64_t ld_src, const void* h_dst, int64_t ld_hdst,
                               void* gat_saved, size_t gat_saved_bytes, const float* W, const float* a_l,
                               const float* a_r, float* dW_accum, float* db_accum, float* da_l_accum,
                               float* da_r_accum, float* dh_src, int64_t ld_dh_src, void* scratch,
                               size_t scratch_bytes, void* stream) {
  BF_CHECK(require_sm100());
  BF_CHECK(validate_model(m));
  if (m->aggregator != BUFFALO_AGG_GAT) {
    set_error("gat_bwd: model.aggregator is not BUFFALO_AGG_GAT");
    return BUFFALO_ERR_UNSUPPORTED;
  }
  if (!blk || layer < 1 || layer > m->num_layers || !dh_dst || !h_src || !gat_saved || !W || !a_l || !a_r ||
      !dW_accum || !db_accum || !da_l_accum || !da_r_accum || !scratch || (layer < m->num_layers && !h_dst) ||
      !blk->t_row_ptr || (dh_src && layer == 1)) {
    set_error("gat_bwd: null argument, bad layer or no transposed block");
    return BUFFALO_ERR_INVALID_ARG;
  }
  GatArgs a{};
  a.blk = blk;
  a.layer1 = layer == 1;
  a.in_bf16 = a.layer1 && m->feat_dtype == BUFFALO_BF16;
  a.last = layer == m->num_layers;
  a.d_in = m->dim[layer - 1];
  a.d_out = m->dim[layer];
  a.h_src = h_src;
  a.ld_src = a.layer1 ? m->feat_pitch : ld_src;
  if ((int64_t)gat_saved_bytes < buffalo::gat_saved_bytes(blk->n_src, blk->n_dst, blk->n_edges, a.d_out) ||
      (int64_t)scratch_bytes < gat_bwd_scratch_bytes(blk->n_src, blk->n_dst, blk->n_edges, a.d_in, a.d_out)) {
    set_error("gat_bwd: saved region or scratch too small");
    return BUFFALO_ERR_CAPACITY;
  }
  a.dh = dh_dst;
  a.ld_dh = ld_dh;
  a.h_dst = (const float*)h_dst;
  a.ld_hdst = ld_hdst;
  a.saved = gat_saved;
  a.W = W;
  a.a_l = a_l;
  a.a_r = a_r;
  a.dW = dW_accum;
  a.db = db_accum;
  a.da_l = da_l_accum;
  a.da_r = da_r_accum;
  a.dh_src = dh_src;
  a.ld_dh_src = ld_dh_src;
  a.scratch = scratch;
  return gat_bwd_ffma(a, (cudaStream_t)stream);
}

buffalo_status buffalo_softmax_ce(const float* logits, int64_t ld, int64_t n, int32_t classes,
                                  const int32_t* labels, const int32_t* row_ids, int64_t batch_size,
                                  float* loss_accum, float* dlogits, int64_t ld_d, void* stream) {
  BF_CHECK(require_sm100());
  if (!logits || !labels || !row_ids || !loss_accum || !dlogits || batch_size <= 0 || classes < 1 ||
      ld < classes || ld_d < classes)
    return BUFFALO_ERR_INVALID_ARG;
  return launch_softmax_ce(logits, ld, n, classes, labels, row_ids, batch_size, loss_accum, dlogits, ld_d,
                           (cudaStream_t)stream);
}

buffalo_status buffalo_sgd_step(float* param, float* grad, int64_t n, float lr, void* stream) {
  BF_CHECK(require_sm100());
  if (!param || !grad || n < 0) return BUFFALO_ERR_INVALID_ARG;
  return launch_sgd(param, grad, n, lr, (cudaStream_t)stream);
}

}  // extern "C"
