// common.cuh — shared helpers of libbuffalo (CUDA side only; nothing here is shared with oracle/).
#pragma once
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <stdint.h>
#include <stdio.h>
#include <atomic>
#include <string>

#include "../../include/buffalo.h"

namespace buffalo {

constexpr int64_t kAlign = 256;
constexpr int kHeavyT = 128;          // rows with D > kHeavyT take the cooperative long-tail path
constexpr int kScanTile = 4096;       // elements per scan tile (512 threads x 8)

__host__ __device__ inline int64_t round_up(int64_t x, int64_t a) { return (x + a - 1) / a * a; }
__host__ __device__ inline int64_t R(int64_t bytes) { return round_up(bytes, kAlign); }
__host__ __device__ inline int64_t pitch_of(int64_t d) { return round_up(d, 8); }

void set_error(const char* fmt, ...);
void count_launch(int n = 1);

// Live timing of one kernel family (buffalo_profile_begin/end): the launch site asks for a
// slot; with one, it records CUDA events around the launch on its stream, passes the slot's
// device counter (edges actually aggregated) and notes the launch's fixed and per-edge bytes.
struct ProfSlot {
  unsigned long long* edges_dev;   // null: not profiled
  int index;
};
ProfSlot prof_begin_launch(const char* family, cudaStream_t s);
void prof_end_launch(const ProfSlot& slot, cudaStream_t s, double fixed_bytes, double bytes_per_edge);

// Returns BUFFALO_ERR_CUDA with the message if the last launch failed.
buffalo_status check_cuda(const char* what);

#define BF_CHECK(...)                                                \
  do {                                                               \
    buffalo_status _s = (__VA_ARGS__);                                      \
    if (_s != BUFFALO_OK) return _s;                                 \
  } while (0)

#define BF_CUDA(...)                                                 \
  do {                                                               \
    cudaError_t _e = (__VA_ARGS__);                                  \
    if (_e != cudaSuccess) {                                         \
      buffalo::set_error("%s: %s", #__VA_ARGS__, cudaGetErrorString(_e)); \
      return BUFFALO_ERR_CUDA;                                       \
    }                                                                \
  } while (0)

#define BF_LAUNCHED(name)                                            \
  do {                                                               \
    buffalo::count_launch();                                         \
    buffalo_status _s = buffalo::check_cuda(name);                   \
    if (_s != BUFFALO_OK) return _s;                                 \
  } while (0)

inline int64_t ceil_div(int64_t a, int64_t b) { return (a + b - 1) / b; }

// Grid size for grid-stride kernels: a multiple of the 148 SMs, capped by the work.
inline int grid_for(int64_t work_items, int per_block, int blocks_per_sm = 8) {
  int64_t g = ceil_div(work_items > 0 ? work_items : 1, per_block);
  int64_t cap = 148LL * blocks_per_sm;
  return (int)(g < cap ? g : cap);
}

// A library-owned non-blocking side stream per device, for fork / join overlap of independent
// launches inside one call (events order it against the caller's stream).  Created once per
// device; a thread that loses the creation race destroys its duplicate.  nullptr on failure
// (callers then stay on their stream).
inline cudaStream_t side_stream(int k = 0) {
  static std::atomic<cudaStream_t> streams[64][2];
  int dev = 0;
  if (k < 0 || k > 1 || cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return nullptr;
  cudaStream_t st = streams[dev][k].load(std::memory_order_acquire);
  if (st) return st;
  cudaStream_t mine = nullptr;
  if (cudaStreamCreateWithFlags(&mine, cudaStreamNonBlocking) != cudaSuccess) return nullptr;
  cudaStream_t expected = nullptr;
  if (!streams[dev][k].compare_exchange_strong(expected, mine, std::memory_order_acq_rel)) {
    cudaStreamDestroy(mine);
    return expected;
  }
  return mine;
}

// Fork of side stream k off the caller's stream (work enqueued on stream() after the fork point
// runs concurrently with later work on the caller's stream); join() — or the destructor, on
// early error returns — makes the caller's stream wait for it.  Without a side stream (on==false
// or creation failure) stream() is the caller's stream and join() is a no-op.
struct SideFork {
  cudaStream_t main, side = nullptr;
  cudaEvent_t ev = nullptr;
  SideFork(cudaStream_t s, int k, bool on) : main(s) {
    if (!on || !(side = side_stream(k))) return;
    if (cudaEventCreateWithFlags(&ev, cudaEventDisableTiming) != cudaSuccess || cudaEventRecord(ev, main) != cudaSuccess ||
        cudaStreamWaitEvent(side, ev, 0) != cudaSuccess) {
      if (ev) cudaEventDestroy(ev);
      ev = nullptr;
      side = nullptr;
    }
  }
  cudaStream_t stream() const { return side ? side : main; }
  bool join() {
    if (!side) return true;
    bool ok = cudaEventRecord(ev, side) == cudaSuccess && cudaStreamWaitEvent(main, ev, 0) == cudaSuccess;
    cudaEventDestroy(ev);
    ev = nullptr;
    side = nullptr;
    return ok;
  }
  ~SideFork() { join(); }
  SideFork(const SideFork&) = delete;
  SideFork& operator=(const SideFork&) = delete;
};

// Programmatic dependent launch for the block build's chains of small kernels: a kernel launched
// with launch_pdl may be scheduled while its predecessor on the stream drains, and waits at its
// top (pdl_wait: griddepcontrol.wait, a no-op for a normal launch) until that grid has completed
// and its memory is visible — semantics of a plain launch, minus the launch gap.  Every kernel
// passed to launch_pdl must call pdl_wait() before touching global memory.
constexpr bool kPdl = true;
__device__ __forceinline__ void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
template <typename... KArgs, typename... Args>
inline void launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
  cudaLaunchConfig_t cfg{};
  cfg.gridDim = grid;
  cfg.blockDim = block;
  cfg.dynamicSmemBytes = smem;
  cfg.stream = s;
  cudaLaunchAttribute at[1];
  at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  at[0].val.programmaticStreamSerializationAllowed = kPdl ? 1 : 0;
  cfg.attrs = at;
  cfg.numAttrs = 1;
  cudaLaunchKernelEx(&cfg, k, args...);
}

// sm_100a check of the current device.
buffalo_status require_sm100();

// cudaFuncSetAttribute(MaxDynamicSharedMemorySize) once per (kernel, device): the kernel is a
// template argument, so every kernel has its own done-mask (one bit per device ordinal: the
// attribute is per device).  The mask is an idempotent cache (two threads racing both set the
// same attribute), not state that changes results.
template <auto Kern>
inline buffalo_status set_max_smem_once(int bytes) {
  static std::atomic<uint64_t> done{0};
  int dev = 0;
  BF_CUDA(cudaGetDevice(&dev));
  const uint64_t bit = dev < 64 ? (1ull << dev) : 0ull;
  if (bit && (done.load(std::memory_order_acquire) & bit)) return BUFFALO_OK;
  BF_CUDA(cudaFuncSetAttribute(Kern, cudaFuncAttributeMaxDynamicSharedMemorySize, bytes));
  done.fetch_or(bit, std::memory_order_release);
  return BUFFALO_OK;
}

// Simple bump allocator over the caller's arena: bottom grows up (persistent), frames are
// placed at the top (temporary).  Tracks the high-water mark bottom + frame.
struct Arena {
  char* base = nullptr;
  int64_t cap = 0, bottom = 0, frame = 0, peak = 0;
  bool overflow = false;
  int64_t need = 0;
  void* take(int64_t bytes) {
    int64_t b = R(bytes);
    void* p = base + bottom;
    bottom += b;
    touch();
    return p;
  }
  // Reserve a temporary frame of `bytes` at the top; returns its base.
  char* push_frame(int64_t bytes) {
    frame = R(bytes);
    touch();
    return base + (cap - frame);
  }
  void pop_frame() { frame = 0; }
  void touch() {
    if (bottom + frame > peak) peak = bottom + frame;
    if (bottom + frame > cap) { overflow = true; if (bottom + frame > need) need = bottom + frame; }
  }
};

// ---------------------------------------------------------------- device helpers
__device__ __forceinline__ float bf2f(__nv_bfloat16 v) { return __bfloat162float(v); }
__device__ __forceinline__ int lane_id() { return threadIdx.x & 31; }

// a0 += low bf16 of w, a1 += high bf16 of w: one mixed-precision add per element
// (add.rn.f32.bf16: exact widening of the bf16 half-register, one fp32 rounding), the same
// result as widening then adding, at half the instructions.
__device__ __forceinline__ void add_bf16x2(float& a0, float& a1, uint32_t w) {
  asm("{\n\t.reg .b16 lo, hi;\n\tmov.b32 {lo, hi}, %2;\n\t"
      "add.rn.f32.bf16 %0, lo, %0;\n\tadd.rn.f32.bf16 %1, hi, %1;\n\t}"
      : "+f"(a0), "+f"(a1)
      : "r"(w));
}

// Rows with more than kHeavyT entries sit at the tail of a degree-class permutation (stable
// partition by min(D, kHeavyT + 1)).  Kernels over them walk the permutation from its end and
// stop at the first light row, so they need no host-side count: the grid is the count when the
// host knows it (>= 0), else a bound from the entry total (at most e / (kHeavyT + 1) heavy rows).
inline int heavy_tail_grid(int64_t n_heavy_known, int64_t entries) {
  if (n_heavy_known >= 0) return (int)std::min<int64_t>(n_heavy_known, 148 * 8);
  return (int)std::min<int64_t>(entries / (kHeavyT + 1), 148 * 8);
}

}  // namespace buffalo
