// Probe: TMA tile::gather4 of fp32 rows with a {32, 1} box and SWIZZLE_128B (two gather4 into one
// 1024-B atom, the second at +512 B); checks the smem image.  height: real rows, then INT32_MAX.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cstdio>
#include <cstdint>
#include <vector>

__global__ void k(const __grid_constant__ CUtensorMap map, const int* rows, int c0, float* out) {
  __shared__ __align__(1024) uint8_t sm[8 * 128];
  __shared__ __align__(8) uint64_t bar;
  uint32_t sb = (uint32_t)__cvta_generic_to_shared(&bar), sd = (uint32_t)__cvta_generic_to_shared(sm);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sb));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sb), "r"(8 * 128));
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(sd), "l"((uint64_t)&map), "r"(c0), "r"(rows[0]), "r"(rows[1]), "r"(rows[2]), "r"(rows[3]), "r"(sb) : "memory");
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(sd + 512), "l"((uint64_t)&map), "r"(c0), "r"(rows[4]), "r"(rows[5]), "r"(rows[6]), "r"(rows[7]), "r"(sb) : "memory");
    asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(sb));
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 8 * 32; i += blockDim.x) out[i] = ((float*)sm)[i];
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main() {
  const int R = 1000, C = 104, P = 104;
  std::vector<float> h((size_t)R * P);
  for (int r = 0; r < R; ++r) for (int c = 0; c < P; ++c) h[(size_t)r * P + c] = (float)(r * 1000 + c);
  float* d; cudaMalloc(&d, h.size() * 4); cudaMemcpy(d, h.data(), h.size() * 4, cudaMemcpyHostToDevice);
  void* f; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  int hr[8] = {5, 17, 900, 3, 42, 7, 999, 100};
  int* dr; cudaMalloc(&dr, 32); cudaMemcpy(dr, hr, 32, cudaMemcpyHostToDevice);
  float* dout; cudaMalloc(&dout, 8 * 32 * 4);
  for (long long height : {(long long)R, (long long)0x7fffffff}) {
    for (int c0 : {0, 32, 96}) {
      CUtensorMap map;
      cuuint64_t dims[2] = {(cuuint64_t)C, (cuuint64_t)height}, str[1] = {(cuuint64_t)P * 4};
      cuuint32_t box[2] = {32, 1}, es[2] = {1, 1};
      CUresult rc = ((Enc)f)(&map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                             CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
      cudaMemset(dout, 0xff, 8 * 32 * 4);
      k<<<1, 128>>>(map, dr, c0, dout);
      cudaError_t e = cudaDeviceSynchronize();
      std::vector<float> o(8 * 32); cudaMemcpy(o.data(), dout, o.size() * 4, cudaMemcpyDeviceToHost);
      int bad = 0;
      for (int r = 0; r < 8; ++r)
        for (int c = 0; c < 32; ++c) {
          int piece = c / 4, phys = piece ^ (r & 7);
          float got = o[r * 32 + phys * 4 + (c % 4)];
          float exp = c0 + c < C ? (float)(hr[r] * 1000 + c0 + c) : 0.f;
          if (got != exp) { if (bad < 3) printf("  r%d c%d got %g exp %g\n", r, c, got, exp); ++bad; }
        }
      printf("height %lld c0 %d: encode rc=%d kernel %s -> %s (%d bad)\n", height, c0, (int)rc, cudaGetErrorString(e),
             bad ? "MISMATCH" : "OK", bad);
    }
  }
}
