// Microbenchmark (diagnostic, not part of the library): TMA load throughput into shared memory
// on B200 as a function of pipeline depth, for 2D boxes (64 bf16 x 128 rows, SW128) and for
// tile::gather4 of random rows.  Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3
// -std=c++17 tools/tma_bench.cu -lcuda -o tools/tma_bench
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>
#include <algorithm>

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, uint32_t c) { asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c)); }
__device__ __forceinline__ void mb_arrive(uint64_t* b) { asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory"); }
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t bytes) { asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory"); }
__device__ __forceinline__ void mb_wait(uint64_t* b, uint32_t parity) {
  asm volatile("{\n\t.reg .pred P1;\n\tW_%=:\n\tmbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t@P1 bra D_%=;\n\tbra W_%=;\n\tD_%=:\n\t}" ::"r"(su32(b)), "r"(parity) : "memory");
}
__device__ __forceinline__ void tma_2d(void* dst, const CUtensorMap* map, int c0, int c1, uint64_t* bar) {
  asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::"r"(su32(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(su32(bar)) : "memory");
}
__device__ __forceinline__ void bulk_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(su32(dst)), "l"(src), "r"(bytes), "r"(su32(bar)) : "memory");
}
__device__ __forceinline__ void tma_gather4(void* dst, const CUtensorMap* map, int c0, int r0, int r1, int r2, int r3, uint64_t* bar) {
  asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];" ::"r"(su32(dst)), "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(bar)) : "memory");
}

constexpr int kBox = 16384;   // 128 rows x 128 B
// mode 0: 2D boxes over rows [0, nrows) x chunk columns; mode 1: gather4 of rows idx[]
__global__ void __launch_bounds__(64, 1) k_bench(const __grid_constant__ CUtensorMap map, const __grid_constant__ CUtensorMap gmap,
                                                 int mode, int NS, int64_t ntiles, int nchunks, const int32_t* idx,
                                                 const __grid_constant__ CUtensorMap smap, int split, const uint8_t* raw) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = (uint64_t*)(smem + NS * kBox);
  uint64_t* empty = full + NS;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { for (int i = 0; i < NS; ++i) { mb_init(&full[i], 1); mb_init(&empty[i], 1); } asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  __syncthreads();
  if (warp == 0) {
    int64_t g = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x) {
      int32_t r[4];
      if (mode == 1) for (int k = 0; k < 4; ++k) r[k] = __ldg(idx + t * 128 + lane * 4 + k);
      for (int c = 0; c < nchunks; ++c, ++g) {
        const int st = (int)(g % NS);
        if (lane == 0) { if (g >= NS) mb_wait(&empty[st], (uint32_t)(((g / NS) - 1) & 1)); mb_expect(&full[st], kBox); }
        __syncwarp();
        if (mode == 1) tma_gather4(smem + st * kBox + lane * 512, &gmap, c * 64, r[0], r[1], r[2], r[3], &full[st]);
        else if (mode == 2) { if (lane < split) tma_2d(smem + st * kBox + lane * (kBox / split), &smap, c * 64, (int)(t * 128 + lane * (128 / split)), &full[st]); }
        else if (mode == 3) { if (lane < split) bulk_1d(smem + st * kBox + lane * (kBox / split), raw + (t * nchunks + c) * (int64_t)kBox + lane * (kBox / split), kBox / split, &full[st]); }
        else if (lane == 0) tma_2d(smem + st * kBox, &map, c * 64, (int)(t * 128), &full[st]);
        __syncwarp();
      }
    }
  } else if (lane == 0) {
    int64_t g = 0;
    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x)
      for (int c = 0; c < nchunks; ++c, ++g) {
        const int st = (int)(g % NS);
        mb_wait(&full[st], (uint32_t)((g / NS) & 1));
        mb_arrive(&empty[st]);
      }
  }
}


// P producer warps in one CTA, each with its own ring of NS stages over every P-th tile of the
// CTA; warp P's lane 0 consumes the rings in turn.  gather: tile::gather4 rows, else 2D boxes.
__global__ void __launch_bounds__(288, 1) k_multi(const __grid_constant__ CUtensorMap map, const __grid_constant__ CUtensorMap gmap,
                                                  int gather, int P, int NS, int64_t ntiles, int nchunks, const int32_t* idx) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = (uint64_t*)(smem + P * NS * kBox);
  uint64_t* empty = full + P * NS;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  if (threadIdx.x == 0) { for (int i = 0; i < P * NS; ++i) { mb_init(&full[i], 1); mb_init(&empty[i], 1); } asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory"); }
  __syncthreads();
  const int64_t my = (ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x;   // tiles of this CTA
  if (warp < P) {
    uint8_t* ring = smem + warp * NS * kBox;
    int64_t g = 0;
    for (int64_t k = warp; k < my; k += P) {
      const int64_t t = blockIdx.x + k * gridDim.x;
      int32_t r[4];
      if (gather) for (int q = 0; q < 4; ++q) r[q] = __ldg(idx + t * 128 + lane * 4 + q);
      for (int c = 0; c < nchunks; ++c, ++g) {
        const int st = (int)(g % NS);
        if (lane == 0) { if (g >= NS) mb_wait(&empty[warp * NS + st], (uint32_t)(((g / NS) - 1) & 1)); mb_expect(&full[warp * NS + st], kBox); }
        __syncwarp();
        if (gather) tma_gather4(ring + st * kBox + lane * 512, &gmap, c * 64, r[0], r[1], r[2], r[3], &full[warp * NS + st]);
        else if (lane == 0) tma_2d(ring + st * kBox, &map, c * 64, (int)(t * 128), &full[warp * NS + st]);
        __syncwarp();
      }
    }
  } else if (warp == P && lane == 0) {
    int64_t gs[8] = {0, 0, 0, 0, 0, 0, 0, 0};
    for (int64_t k = 0; k < my; ++k) {
      const int w = (int)(k % P);
      for (int c = 0; c < nchunks; ++c, ++gs[w]) {
        const int st = (int)(gs[w] % NS);
        mb_wait(&full[w * NS + st], (uint32_t)((gs[w] / NS) & 1));
        mb_arrive(&empty[w * NS + st]);
      }
    }
  }
}

typedef CUresult (*EncFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                          const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                          CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

int main() {
  const int64_t rows = 4 << 20, cols = 128;   // 4M rows x 256 B = 1 GiB bf16
  void* buf; cudaMalloc(&buf, rows * cols * 2); cudaMemset(buf, 1, rows * cols * 2);
  void* flush; cudaMalloc(&flush, 512 << 20);
  std::vector<int32_t> hidx(rows);
  uint64_t x = 88172645463325252ull;
  for (auto& v : hidx) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; v = (int32_t)(x % rows); }
  int32_t* didx; cudaMalloc(&didx, rows * 4); cudaMemcpy(didx, hidx.data(), rows * 4, cudaMemcpyHostToDevice);
  void* f = nullptr; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  EncFn enc = (EncFn)f;
  CUtensorMap m2, mg;
  cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)rows}; cuuint64_t str[1] = {(cuuint64_t)cols * 2};
  cuuint32_t box[2] = {64, 128}, boxg[2] = {64, 1}, es[2] = {1, 1};
  enc(&m2, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  enc(&mg, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, boxg, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  cudaFuncSetAttribute(k_bench, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  const int64_t ntiles = rows / 128;
  auto run = [&](const char* name, int mode, int NS, int cps, int split) {
    CUtensorMap ms;
    cuuint32_t sbox[2] = {64, (cuuint32_t)(128 / split)};
    enc(&ms, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, buf, dims, str, sbox, es, CU_TENSOR_MAP_INTERLEAVE_NONE, CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
    const int smem = NS * kBox + 16 * NS + 2048;
    float best = 1e9f;
    for (int rep = 0; rep < 3; ++rep) {
      cudaMemset(flush, rep, 512 << 20);
      cudaEventRecord(a);
      k_bench<<<148 * cps, 64, smem>>>(m2, mg, mode, NS, ntiles, 2, didx, ms, split, (const uint8_t*)buf);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms_; cudaEventElapsedTime(&ms_, a, b); best = std::min(best, ms_);
    }
    cudaError_t e = cudaGetLastError();
    printf("%-8s NS=%2d ctas/SM=%d split=%d  %.3f ms  %.0f GB/s %s\n", name, NS, cps, split, best, rows * 256.0 / best / 1e6, e ? cudaGetErrorString(e) : "");
  };
  auto runm = [&](int gather, int P, int NS) {
    cudaFuncSetAttribute(k_multi, cudaFuncAttributeMaxDynamicSharedMemorySize, 227 * 1024);
    const int smem = P * NS * kBox + 16 * P * NS + 2048;
    float best = 1e9f;
    for (int rep = 0; rep < 3; ++rep) {
      cudaMemset(flush, rep, 512 << 20);
      cudaEventRecord(a);
      k_multi<<<148, 32 * (P + 1), smem>>>(m2, mg, gather, P, NS, ntiles, 2, didx);
      cudaEventRecord(b); cudaEventSynchronize(b);
      float ms_; cudaEventElapsedTime(&ms_, a, b); best = std::min(best, ms_);
    }
    cudaError_t e = cudaGetLastError();
    printf("multi %s P=%d NS=%d  %.3f ms  %.0f GB/s %s\n", gather ? "gather4" : "2d", P, NS, best, rows * 256.0 / best / 1e6, e ? cudaGetErrorString(e) : "");
  };
  for (int rep = 0; rep < 2; ++rep) { run("2d", 0, 4, 1, 1); run("2d", 0, 12, 1, 1); }
  runm(0, 1, 8); runm(0, 2, 4); runm(0, 4, 3); runm(0, 8, 1);
  runm(1, 1, 8); runm(1, 2, 4); runm(1, 4, 3); runm(1, 8, 1);
  run("2d", 0, 4, 2, 1); run("2d", 0, 4, 3, 1); run("2d", 0, 3, 4, 1);
  run("2dsplit", 2, 4, 1, 2); run("2dsplit", 2, 4, 1, 4); run("2dsplit", 2, 8, 1, 4); run("2dsplit", 2, 8, 1, 8); run("2dsplit", 2, 12, 1, 16);
  run("bulk1d", 3, 4, 1, 1); run("bulk1d", 3, 8, 1, 4); run("bulk1d", 3, 12, 1, 8);
  run("gather4", 1, 4, 1, 1); run("gather4", 1, 4, 2, 1); run("gather4", 1, 3, 4, 1);
  return 0;
}
