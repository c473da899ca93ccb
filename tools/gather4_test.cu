// Probe: TMA tile::gather4 with a {64, 1} box and SWIZZLE_128B; checks the smem image.
#include <cuda.h>
#include <cuda_runtime.h>
#include <cuda_bf16.h>
#include <cstdio>
#include <cstdint>
#include <vector>

__global__ void k(const __grid_constant__ CUtensorMap map, const int* rows, uint16_t* out) {
  __shared__ __align__(1024) uint8_t sm[8 * 128];
  __shared__ __align__(8) uint64_t bar;
  uint32_t sb = (uint32_t)__cvta_generic_to_shared(&bar), sd = (uint32_t)__cvta_generic_to_shared(sm);
  if (threadIdx.x == 0) {
    asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" ::"r"(sb));
    asm volatile("fence.mbarrier_init.release.cluster;");
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(sb), "r"(8 * 128));
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(sd), "l"((uint64_t)&map), "r"(0), "r"(rows[0]), "r"(rows[1]), "r"(rows[2]), "r"(rows[3]), "r"(sb) : "memory");
    asm volatile("cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, %4, %5, %6}], [%7];"
                 ::"r"(sd + 512), "l"((uint64_t)&map), "r"(0), "r"(rows[4]), "r"(rows[5]), "r"(rows[6]), "r"(rows[7]), "r"(sb) : "memory");
    asm volatile("{\n.reg .pred P;\nW: mbarrier.try_wait.parity.shared::cta.b64 P, [%0], 0;\n@!P bra W;\n}" ::"r"(sb));
  }
  __syncthreads();
  for (int i = threadIdx.x; i < 8 * 64; i += blockDim.x) out[i] = ((uint16_t*)sm)[i];
}

typedef CUresult (*Enc)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*, const cuuint64_t*,
                        const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave, CUtensorMapSwizzle,
                        CUtensorMapL2promotion, CUtensorMapFloatOOBfill);
int main() {
  const int R = 1000, C = 104;   // rows of 104 bf16 (pitch 104 -> 208 B)
  std::vector<uint16_t> h(R * C);
  for (int r = 0; r < R; ++r) for (int c = 0; c < C; ++c) h[r * C + c] = (uint16_t)(r * 100 + c);
  uint16_t* d; cudaMalloc(&d, h.size() * 2); cudaMemcpy(d, h.data(), h.size() * 2, cudaMemcpyHostToDevice);
  void* f; cudaDriverEntryPointQueryResult q;
  cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q);
  CUtensorMap map;
  cuuint64_t dims[2] = {C, R}, str[1] = {C * 2};
  cuuint32_t box[2] = {64, 1}, es[2] = {1, 1};
  CUresult rc = ((Enc)f)(&map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, d, dims, str, box, es, CU_TENSOR_MAP_INTERLEAVE_NONE,
                         CU_TENSOR_MAP_SWIZZLE_128B, CU_TENSOR_MAP_L2_PROMOTION_L2_256B, CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  printf("encode rc=%d\n", (int)rc);
  int hr[8] = {5, 17, 900, 3, 42, 7, 999, 100};
  int* dr; cudaMalloc(&dr, 32); cudaMemcpy(dr, hr, 32, cudaMemcpyHostToDevice);
  uint16_t* dout; cudaMalloc(&dout, 8 * 64 * 2);
  k<<<1, 128>>>(map, dr, dout);
  printf("kernel: %s\n", cudaGetErrorString(cudaDeviceSynchronize()));
  std::vector<uint16_t> o(8 * 64); cudaMemcpy(o.data(), dout, o.size() * 2, cudaMemcpyDeviceToHost);
  int bad = 0;
  for (int r = 0; r < 8; ++r)
    for (int c = 0; c < 64; ++c) {
      int piece = c / 8, phys = piece ^ (r & 7);
      uint16_t got = o[r * 64 + phys * 8 + (c % 8)];
      uint16_t exp = (uint16_t)(hr[r] * 100 + c);
      if (got != exp) { if (bad < 5) printf("r%d c%d got %d exp %d\n", r, c, got, exp); ++bad; }
    }
  printf("gather4 swizzled image %s (%d bad)\n", bad ? "MISMATCH" : "OK", bad);
}
