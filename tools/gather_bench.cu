// Microbenchmark (diagnostic, not part of the library): achievable bandwidth of the
// neighbour-row gather of SAGE-mean on B200 for random rows of W bytes, D neighbours per row.
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>
#include <cuda_bf16.h>

__device__ __forceinline__ void acc8(float* a, uint4 u) {
  const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) { a[2*i] += __uint_as_float(w[i] << 16); a[2*i+1] += __uint_as_float(w[i] & 0xffff0000u); }
}

// lanes per row = LPR (16 B per lane), rows per warp = 32/LPR; U neighbours in flight per lane
template <int LPR, int U>
__global__ void __launch_bounds__(256) k_gather(const int32_t* __restrict__ col, int D, int64_t n,
                                                const uint4* __restrict__ h, int ld16, uint4* __restrict__ out,
                                                int pieces) {
  const int lane = threadIdx.x & 31, g = lane / LPR, pc = lane % LPR;
  constexpr int G = 32 / LPR;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w * G < n; w += warps) {
    const int64_t row = w * G + g;
    float a[8] = {};
    if (row < n && pc < pieces) {
      const int32_t* c = col + row * D;
      for (int e = 0; e < D; e += U) {
        uint4 r[U];
#pragma unroll
        for (int u = 0; u < U; ++u) r[u] = (e + u < D) ? __ldg(h + (int64_t)__ldg(c + e + u) * ld16 + pc) : make_uint4(0,0,0,0);
#pragma unroll
        for (int u = 0; u < U; ++u) acc8(a, r[u]);
      }
      uint4 o; __nv_bfloat162 t;
      t = __floats2bfloat162_rn(a[0], a[1]); o.x = *(uint32_t*)&t; t = __floats2bfloat162_rn(a[2], a[3]); o.y = *(uint32_t*)&t;
      t = __floats2bfloat162_rn(a[4], a[5]); o.z = *(uint32_t*)&t; t = __floats2bfloat162_rn(a[6], a[7]); o.w = *(uint32_t*)&t;
      out[row * ld16 + pc] = o;
    }
  }
}

template <int LPR, int U>
void run(const char* name, const int32_t* col, int D, int64_t n, const uint4* h, int ld16, uint4* out, int bps,
         int pieces = 32) {
  int grid = 148 * bps;
  cudaEvent_t a, b; cudaEventCreate(&a); cudaEventCreate(&b);
  for (int it = 0; it < 3; ++it) k_gather<LPR, U><<<grid, 256>>>(col, D, n, h, ld16, out, pieces);
  cudaEventRecord(a);
  for (int it = 0; it < 5; ++it) k_gather<LPR, U><<<grid, 256>>>(col, D, n, h, ld16, out, pieces);
  cudaEventRecord(b); cudaEventSynchronize(b);
  float ms; cudaEventElapsedTime(&ms, a, b); ms /= 5;
  const int useful = (pieces < LPR ? pieces : LPR) * 16;
  double bytes = (double)n * D * (useful + 4) + (double)n * useful;
  printf("%-28s LPR=%2d U=%2d blocks/SM=%d useful=%d pitch=%d: %.3f ms  %.0f GB/s\n", name, LPR, U, bps, useful,
         ld16 * 16, ms, bytes / ms / 1e6);
}

int main() {
  const int64_t N = 2449029;          // products-shaped feature table, d = 100 bf16 -> 13 pieces of 16 B
  const int D = 10;
  const int64_t n = 1700000;
  int32_t* col; cudaMalloc(&col, (size_t)n * D * 4);
  int32_t* hc = (int32_t*)malloc((size_t)n * D * 4);
  uint64_t x = 88172645463325252ull;
  for (int64_t i = 0; i < n * D; ++i) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; hc[i] = (int32_t)(x % N); }
  cudaMemcpy(col, hc, (size_t)n * D * 4, cudaMemcpyHostToDevice);
  for (int W : {208, 224, 256}) {
    const int ld16 = W / 16;
    uint4* h; cudaMalloc(&h, (size_t)N * W);
    cudaMemset(h, 0, (size_t)N * W);
    uint4* out; cudaMalloc(&out, (size_t)n * 256);
    for (int bps : {8}) {
      run<16, 4>("feat rows", col, D, n, h, ld16, out, bps, 13);
      run<16, 8>("feat rows", col, D, n, h, ld16, out, bps, 13);
    }
    cudaFree(h); cudaFree(out);
  }
  cudaError_t e = cudaGetLastError();
  printf("%s\n", cudaGetErrorString(e));
  return 0;
}

int main_old() {
  const int64_t N = 2449029;          // products-shaped table
  const int D = 25;
  for (int W : {512, 256}) {
    const int ld16 = W / 16;
    uint4* h; cudaMalloc(&h, (size_t)N * W);
    cudaMemset(h, 0, (size_t)N * W);
    const int64_t n = 2000000;
    int32_t* col; cudaMalloc(&col, (size_t)n * D * 4);
    int32_t* hc = (int32_t*)malloc((size_t)n * D * 4);
    uint64_t x = 88172645463325252ull;
    for (int64_t i = 0; i < n * D; ++i) { x ^= x << 13; x ^= x >> 7; x ^= x << 17; hc[i] = (int32_t)(x % N); }
    cudaMemcpy(col, hc, (size_t)n * D * 4, cudaMemcpyHostToDevice);
    uint4* out; cudaMalloc(&out, (size_t)n * W);
    printf("row bytes %d, table %.2f GB, %lld rows x %d nbrs\n", W, N * (double)W / 1e9, (long long)n, D);
    if (W == 512) {
      run<32, 4>("warp/row", col, D, n, h, ld16, out, 8);
      run<32, 8>("warp/row", col, D, n, h, ld16, out, 8);
      run<32, 16>("warp/row", col, D, n, h, ld16, out, 4);
      run<32, 8>("warp/row", col, D, n, h, ld16, out, 4);
      run<32, 8>("warp/row", col, D, n, h, ld16, out, 2);
    } else {
      run<16, 4>("half-warp/row", col, D, n, h, ld16, out, 8);
      run<16, 8>("half-warp/row", col, D, n, h, ld16, out, 8);
      run<16, 8>("half-warp/row", col, D, n, h, ld16, out, 4);
      run<16, 16>("half-warp/row", col, D, n, h, ld16, out, 4);
    }
    cudaFree(h); cudaFree(col); cudaFree(out); free(hc);
  }
  cudaError_t e = cudaGetLastError();
  printf("%s\n", cudaGetErrorString(e));
}
