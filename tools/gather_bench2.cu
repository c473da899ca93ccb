// Microbenchmark (diagnostic, not part of the library): neighbour-row gather strategies on B200.
//   ldg   : lanes load 16-B pieces of the neighbour rows into registers (U rows in flight per lane)
//   bulk  : per batch of dst rows one lane per neighbour row issues a 1D cp.async.bulk of the whole
//           row into a shared-memory slot (mbarrier tx count), double-buffered; lanes sum from smem
//   ldgsts: each lane copies its 16-B pieces of the batch's neighbour rows with cp.async (no
//           register destination), double-buffered; lanes sum from smem
// Rows: W bytes (bf16), D neighbours per dst row, random neighbour ids over N table rows.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

__device__ __forceinline__ void acc8(float* a, uint4 u) {
  const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) { a[2*i] += __uint_as_float(w[i] << 16); a[2*i+1] += __uint_as_float(w[i] & 0xffff0000u); }
}
__device__ __forceinline__ uint4 pack8(const float* a) {
  uint4 o; __nv_bfloat162 t;
  t = __floats2bfloat162_rn(a[0], a[1]); o.x = *(uint32_t*)&t; t = __floats2bfloat162_rn(a[2], a[3]); o.y = *(uint32_t*)&t;
  t = __floats2bfloat162_rn(a[4], a[5]); o.z = *(uint32_t*)&t; t = __floats2bfloat162_rn(a[6], a[7]); o.w = *(uint32_t*)&t;
  return o;
}
__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

template <int LPR, int U>
__global__ void __launch_bounds__(256) k_ldg(const int32_t* __restrict__ col, int D, int64_t n,
                                             const uint4* __restrict__ h, int ld16, uint4* __restrict__ out) {
  const int lane = threadIdx.x & 31, g = lane / LPR, pc = lane % LPR;
  constexpr int G = 32 / LPR;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * G < n; w += warps) {
    const int64_t row = w * G + g;
    float a[8] = {};
    if (row < n && pc < ld16) {
      const int32_t* c = col + row * D;
      for (int e = 0; e < D; e += U) {
        uint4 r[U];
#pragma unroll
        for (int u = 0; u < U; ++u) r[u] = (e + u < D) ? __ldg(h + (int64_t)__ldg(c + e + u) * ld16 + pc) : make_uint4(0,0,0,0);
#pragma unroll
        for (int u = 0; u < U; ++u) acc8(a, r[u]);
      }
      out[row * ld16 + pc] = pack8(a);
    }
  }
}

// A warp handles batches of B = 32 / D dst rows (B*D <= 32 neighbour rows, one slot each).
template <int WARPS, bool BULK>
__global__ void __launch_bounds__(WARPS * 32) k_staged(const int32_t* __restrict__ col, int D, int64_t n,
                                                      const uint4* __restrict__ h, int ld16, uint4* __restrict__ out) {
  extern __shared__ __align__(128) uint8_t smem[];
  const int lane = threadIdx.x & 31, wl = threadIdx.x >> 5;
  const int W = ld16 * 16;
  uint8_t* buf = smem + (size_t)wl * 2 * 32 * W;                 // 2 stages x 32 slots x W
  __shared__ uint64_t bar[WARPS][2];
  if (BULK && lane == 0) {
    for (int s = 0; s < 2; ++s) asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(su32(&bar[wl][s])));
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();
  const int B = 32 / D;
  const int64_t nb = (n + B - 1) / B;
  const int64_t warps = (int64_t)gridDim.x * WARPS;
  int64_t bi = blockIdx.x * (int64_t)WARPS + wl;
  uint32_t phase[2] = {0, 0};
  auto issue = [&](int64_t b, int st) {
    const int64_t r0 = b * B;
    const int nr = (int)(n - r0 < B ? n - r0 : B);
    const int ne = nr * D;
    uint8_t* sb = buf + (size_t)st * 32 * W;
    if (BULK) {
      if (lane == 0)
        asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(&bar[wl][st])), "r"(ne * W) : "memory");
      __syncwarp();
      if (lane < ne) {
        const int32_t j = __ldg(col + r0 * D + lane);
        asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                         su32(sb + lane * W)), "l"(h + (int64_t)j * ld16), "r"(W), "r"(su32(&bar[wl][st])) : "memory");
      }
    } else {
      const int32_t j = lane < ne ? __ldg(col + r0 * D + lane) : 0;
      for (int s = 0; s < ne; ++s) {
        const int32_t js = __shfl_sync(0xffffffffu, j, s);
        for (int p = lane; p < ld16; p += 32)
          asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(su32(sb + s * W + p * 16)), "l"(h + (int64_t)js * ld16 + p) : "memory");
      }
      asm volatile("cp.async.commit_group;" ::: "memory");
    }
  };
  if (bi < nb) issue(bi, 0);
  int st = 0;
  for (; bi < nb; bi += warps, st ^= 1) {
    if (bi + warps < nb) issue(bi + warps, st ^ 1);
    if (BULK) {
      asm volatile("{\n\t.reg .pred P1;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@!P1 bra W_%=;\n\t}" ::"r"(
                       su32(&bar[wl][st])), "r"(phase[st]) : "memory");
      phase[st] ^= 1;
    } else {
      if (bi + warps < nb) asm volatile("cp.async.wait_group 1;" ::: "memory");
      else asm volatile("cp.async.wait_group 0;" ::: "memory");
      __syncwarp();
    }
    const int64_t r0 = bi * B;
    const int nr = (int)(n - r0 < B ? n - r0 : B);
    const uint8_t* sb = buf + (size_t)st * 32 * W;
    // lanes: row piece p = lane % ld16 (ld16 <= 32), rows of the batch round-robin over lane groups
    const int lpr = ld16 <= 16 ? 16 : 32;
    const int grp = lane / lpr, pc = lane % lpr;
    for (int r = grp; r < nr; r += 32 / lpr) {
      float a[8] = {};
      if (pc < ld16)
        for (int e = 0; e < D; ++e) acc8(a, *reinterpret_cast<const uint4*>(sb + (r * D + e) * W + pc * 16));
      if (pc < ld16) out[(r0 + r) * ld16 + pc] = pack8(a);
    }
    __syncwarp();
  }
}

static void report(const char* name, float ms, int64_t n, int D, int W) {
  double bytes = (double)n * D * (W + 4) + (double)n * W;
  printf("%-34s W=%3d D=%2d: %.3f ms  %.0f GB/s\n", name, W, D, ms, bytes / ms / 1e6);
}

template <class F>
float timeit(F f) {
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int it = 0; it < 2; ++it) f();
  cudaEventRecord(a);
  for (int it = 0; it < 5; ++it) f();
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b);
  return ms / 5;
}

int main() {
  const int64_t N = 2449029;
  struct Cfg { int W, D; int64_t n; } cfgs[] = {{512, 25, 1500000}, {256, 10, 1800000}, {512, 2, 8000000}, {512, 10, 3000000}};
  for (auto c : cfgs) {
    const int ld16 = c.W / 16;
    uint4* h; cudaMalloc(&h, (size_t)N * c.W); cudaMemset(h, 0, (size_t)N * c.W);
    int32_t* col; cudaMalloc(&col, (size_t)c.n * c.D * 4);
    int32_t* hc = (int32_t*)malloc((size_t)c.n * c.D * 4);
    uint64_t x = 88172645463325252ull;
    for (int64_t i = 0; i < c.n * c.D; ++i) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; hc[i] = (int32_t)(x % N); }
    cudaMemcpy(col, hc, (size_t)c.n * c.D * 4, cudaMemcpyHostToDevice);
    uint4* out; cudaMalloc(&out, (size_t)c.n * c.W);
    char nm[64];
    if (c.W == 512) {
      report("ldg LPR32 U2 6cta", timeit([&] { k_ldg<32, 2><<<148 * 6 * 4, 256>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
      report("ldg LPR32 U4 6cta", timeit([&] { k_ldg<32, 4><<<148 * 6 * 4, 256>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
    } else {
      report("ldg LPR16 U2 6cta", timeit([&] { k_ldg<16, 2><<<148 * 6 * 4, 256>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
      report("ldg LPR16 U4 6cta", timeit([&] { k_ldg<16, 4><<<148 * 6 * 4, 256>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
    }
    for (int warps : {4, 8}) {
      const size_t sm = (size_t)warps * 2 * 32 * c.W;
      if (sm > 227 * 1024) continue;
      int ctas = (int)((227 * 1024) / (sm + 1024));
      if (ctas > 16) ctas = 16;
      if (warps == 4) {
        cudaFuncSetAttribute(k_staged<4, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        cudaFuncSetAttribute(k_staged<4, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        snprintf(nm, sizeof nm, "bulk 4w x%d cta/SM", ctas);
        report(nm, timeit([&] { k_staged<4, true><<<148 * ctas, 128, sm>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
        snprintf(nm, sizeof nm, "ldgsts 4w x%d cta/SM", ctas);
        report(nm, timeit([&] { k_staged<4, false><<<148 * ctas, 128, sm>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
      } else {
        cudaFuncSetAttribute(k_staged<8, true>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        cudaFuncSetAttribute(k_staged<8, false>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
        snprintf(nm, sizeof nm, "bulk 8w x%d cta/SM", ctas);
        report(nm, timeit([&] { k_staged<8, true><<<148 * ctas, 256, sm>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
        snprintf(nm, sizeof nm, "ldgsts 8w x%d cta/SM", ctas);
        report(nm, timeit([&] { k_staged<8, false><<<148 * ctas, 256, sm>>>(col, c.D, c.n, h, ld16, out); }), c.n, c.D, c.W);
      }
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("  (%s)\n", cudaGetErrorString(e));
    cudaFree(h); cudaFree(col); cudaFree(out); free(hc);
  }
  return 0;
}
