// sage.cu — GraphSAGE-mean layer kernels, CUDA-core path.
//
// Aggregate (Alg. 2 l.8): warp per destination row, 16-byte vector loads of the
// neighbour rows, fp32 accumulation in CSR order, one IEEE division by D (R21).  Rows with
// D > kHeavyT (the long tail of full-neighbour blocks) go to a CTA-cooperative kernel whose
// per-warp partial sums are combined in warp order (deterministic, depends only on D).
// Update (Alg. 2 l.9): fp32 SIMT GEMM over [h_self || h_agg] (gemm_mode FFMA, the parity
// path); the tensor-core path is in tc_sage.cu.
#include "common.cuh"
#include <type_traits>

#include <vector>

#include "sage.cuh"
#include "tc_f32.cuh"

namespace buffalo {

// ------------------------------------------------------------------ vector loads
template <class T, int C> struct VecIO;
template <> struct VecIO<float, 4> {
  static __device__ __forceinline__ void load(const float* p, float* v) {
    float4 a = __ldg(reinterpret_cast<const float4*>(p));
    v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
  }
  static __device__ __forceinline__ void store(float* p, const float* v) {
    *reinterpret_cast<float4*>(p) = make_float4(v[0], v[1], v[2], v[3]);
  }
};
template <> struct VecIO<float, 8> {
  static __device__ __forceinline__ void load(const float* p, float* v) {
    VecIO<float, 4>::load(p, v);
    VecIO<float, 4>::load(p + 4, v + 4);
  }
  static __device__ __forceinline__ void store(float* p, const float* v) {
    VecIO<float, 4>::store(p, v);
    VecIO<float, 4>::store(p + 4, v + 4);
  }
};
__device__ __forceinline__ void unpack_bf2(uint32_t w, float& a, float& b) {
  a = __uint_as_float(w << 16);
  b = __uint_as_float(w & 0xffff0000u);
}
__device__ __forceinline__ uint32_t pack_bf2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}
template <> struct VecIO<__nv_bfloat16, 4> {
  static __device__ __forceinline__ void load(const __nv_bfloat16* p, float* v) {
    uint2 a = __ldg(reinterpret_cast<const uint2*>(p));
    unpack_bf2(a.x, v[0], v[1]); unpack_bf2(a.y, v[2], v[3]);
  }
  static __device__ __forceinline__ void store(__nv_bfloat16* p, const float* v) {
    *reinterpret_cast<uint2*>(p) = make_uint2(pack_bf2(v[0], v[1]), pack_bf2(v[2], v[3]));
  }
};
template <> struct VecIO<__nv_bfloat16, 8> {
  static __device__ __forceinline__ void load(const __nv_bfloat16* p, float* v) {
    uint4 a = __ldg(reinterpret_cast<const uint4*>(p));
    unpack_bf2(a.x, v[0], v[1]); unpack_bf2(a.y, v[2], v[3]);
    unpack_bf2(a.z, v[4], v[5]); unpack_bf2(a.w, v[6], v[7]);
  }
  static __device__ __forceinline__ void store(__nv_bfloat16* p, const float* v) {
    *reinterpret_cast<uint4*>(p) = make_uint4(pack_bf2(v[0], v[1]), pack_bf2(v[2], v[3]),
                                              pack_bf2(v[4], v[5]), pack_bf2(v[6], v[7]));
  }
};

template <class T> __device__ __forceinline__ float ld1(const T* p);
template <> __device__ __forceinline__ float ld1<float>(const float* p) { return __ldg(p); }
template <> __device__ __forceinline__ float ld1<__nv_bfloat16>(const __nv_bfloat16* p) {
  return __bfloat162float(*p);
}
template <class T> __device__ __forceinline__ void st1(T* p, float v);
template <> __device__ __forceinline__ void st1<float>(float* p, float v) { *p = v; }
template <> __device__ __forceinline__ void st1<__nv_bfloat16>(__nv_bfloat16* p, float v) {
  *p = __float2bfloat16_rn(v);
}

// ------------------------------------------------------------------ aggregate (regular rows)
template <class TI, class TO, int C>
__global__ void __launch_bounds__(256) k_agg_rows(const int32_t* __restrict__ rp,
                                                  const int32_t* __restrict__ col, int64_t n,
                                                  const TI* __restrict__ h, int64_t ldh, int d,
                                                  TO* __restrict__ agg, int64_t lda) {
  const int lane = threadIdx.x & 31;
  const int nch = (d + C - 1) / C;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
    const int32_t b = rp[i], e_end = rp[i + 1];
    const int32_t D = e_end - b;
    if (D > kHeavyT) continue;
    for (int c = lane; c < nch; c += 32) {
      float acc[C];
#pragma unroll
      for (int k = 0; k < C; ++k) acc[k] = 0.f;
      int32_t e = b;
      for (; e + 4 <= e_end; e += 4) {
        const int64_t j0 = col[e], j1 = col[e + 1], j2 = col[e + 2], j3 = col[e + 3];
        float v0[C], v1[C], v2[C], v3[C];
        VecIO<TI, C>::load(h + j0 * ldh + c * C, v0);
        VecIO<TI, C>::load(h + j1 * ldh + c * C, v1);
        VecIO<TI, C>::load(h + j2 * ldh + c * C, v2);
        VecIO<TI, C>::load(h + j3 * ldh + c * C, v3);
#pragma unroll
        for (int k = 0; k < C; ++k) { acc[k] += v0[k]; acc[k] += v1[k]; acc[k] += v2[k]; acc[k] += v3[k]; }
      }
      for (; e < e_end; ++e) {
        float v0[C];
        VecIO<TI, C>::load(h + (int64_t)col[e] * ldh + c * C, v0);
#pragma unroll
        for (int k = 0; k < C; ++k) acc[k] += v0[k];
      }
      const float fd = (float)D;
#pragma unroll
      for (int k = 0; k < C; ++k) acc[k] = D > 0 ? acc[k] / fd : 0.f;
      VecIO<TO, C>::store(agg + i * lda + c * C, acc);
    }
  }
}

// ------------------------------------------------------------------ aggregate (long tail)
template <class TI, class TO, int C>
__global__ void __launch_bounds__(256) k_agg_heavy(const int32_t* __restrict__ perm, int64_t n,
                                                   const int32_t* __restrict__ rp,
                                                   const int32_t* __restrict__ col,
                                                   const TI* __restrict__ h, int64_t ldh, int d,
                                                   TO* __restrict__ agg, int64_t lda) {
  __shared__ float part[8][32][C];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  for (int64_t hh = blockIdx.x; hh < n; hh += gridDim.x) {
  const int64_t i = perm[n - 1 - hh];        // heavy rows: the tail of the degree-class perm
  const int32_t b = rp[i], e_end = rp[i + 1];
  if (e_end - b <= kHeavyT) break;
  const float fd = (float)(e_end - b);
  const int nch = (d + C - 1) / C;
  for (int c0 = 0; c0 < nch; c0 += 32) {
    const int c = c0 + lane;
    float acc[C];
#pragma unroll
    for (int k = 0; k < C; ++k) acc[k] = 0.f;
    if (c < nch) {
      int32_t e = b + w;
      if constexpr (std::is_same<TI, __nv_bfloat16>::value && C == 8) {
        for (; e + 24 < e_end; e += 32) {                // four rows in flight per lane
          uint4 r[4];
#pragma unroll
          for (int u = 0; u < 4; ++u) r[u] = __ldg(reinterpret_cast<const uint4*>(h + (int64_t)col[e + 8 * u] * ldh + c * C));
#pragma unroll
          for (int u = 0; u < 4; ++u) {
            add_bf16x2(acc[0], acc[1], r[u].x); add_bf16x2(acc[2], acc[3], r[u].y);
            add_bf16x2(acc[4], acc[5], r[u].z); add_bf16x2(acc[6], acc[7], r[u].w);
          }
        }
      } else {
        for (; e + 24 < e_end; e += 32) {
          float v[4][C];
#pragma unroll
          for (int u = 0; u < 4; ++u) VecIO<TI, C>::load(h + (int64_t)col[e + 8 * u] * ldh + c * C, v[u]);
#pragma unroll
          for (int u = 0; u < 4; ++u)
#pragma unroll
            for (int k = 0; k < C; ++k) acc[k] += v[u][k];
        }
      }
      for (; e < e_end; e += 8) {
        float v[C];
        VecIO<TI, C>::load(h + (int64_t)col[e] * ldh + c * C, v);
#pragma unroll
        for (int k = 0; k < C; ++k) acc[k] += v[k];
      }
    }
#pragma unroll
    for (int k = 0; k < C; ++k) part[w][lane][k] = acc[k];
    __syncthreads();
    if (w == 0 && c < nch) {
      float s[C];
#pragma unroll
      for (int k = 0; k < C; ++k) s[k] = part[0][lane][k];
      for (int ww = 1; ww < 8; ++ww)
#pragma unroll
        for (int k = 0; k < C; ++k) s[k] += part[ww][lane][k];
#pragma unroll
      for (int k = 0; k < C; ++k) s[k] = s[k] / fd;
      VecIO<TO, C>::store(agg + i * lda + c * C, s);
    }
    __syncthreads();
  }
  }
}

template <class TI, class TO>
static buffalo_status launch_agg(const buffalo_block* blk, const int32_t* col, const TI* h,
                                 int64_t ldh, int d, TO* agg, int64_t lda, cudaStream_t s) {
  const int64_t n = blk->n_dst;
  if (n <= 0) return BUFFALO_OK;
  const bool wide = d > 128;
  const ProfSlot ps = prof_begin_launch("gather", s);
  if (wide) {
    k_agg_rows<TI, TO, 8><<<grid_for(n * 32, 256, 16), 256, 0, s>>>(blk->row_ptr, col, n, h, ldh, d, agg, lda);
  } else {
    k_agg_rows<TI, TO, 4><<<grid_for(n * 32, 256, 16), 256, 0, s>>>(blk->row_ptr, col, n, h, ldh, d, agg, lda);
  }
  BF_LAUNCHED("k_agg_rows");
  // algorithmic bytes: per row the row_ptr pair + the output row; per edge index + source row
  prof_end_launch(ps, s, (double)n * (8.0 + (double)pitch_of(d) * sizeof(TO)) +
                             (double)blk->n_edges * (4.0 + (double)pitch_of(d) * sizeof(TI)), 0.0);
  const int hg = heavy_tail_grid(blk->n_heavy, blk->n_edges);
  if (hg > 0) {
    if (wide)
      k_agg_heavy<TI, TO, 8><<<hg, 256, 0, s>>>(blk->cls_perm, n, blk->row_ptr, col, h, ldh, d, agg, lda);
    else
      k_agg_heavy<TI, TO, 4><<<hg, 256, 0, s>>>(blk->cls_perm, n, blk->row_ptr, col, h, ldh, d, agg, lda);
    BF_LAUNCHED("k_agg_heavy");
  }
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ SIMT GEMM
// C[M][Np] = A1[M][K1] B1[K1][N] + A2[M][K2] B2[K2][N] (+ bias) (ReLU); columns N..Np-1 = 0.
// A1 row r is A1[gidx ? gidx[r] : r] and is zero for r >= m1.
// CTA tile 128 x 128, K step 8, 256 threads with an 8 x 8 register tile each (rows
// 8 ty .. 8 ty + 7, columns in two 4-wide runs tx * 4 and 64 + tx * 4, so that both fragments
// are two float4 shared loads per k); the next K step's operands are prefetched into registers while the
// current one is multiplied.  The K loop order is fixed, so results are deterministic.
constexpr int GB_M = 128, GB_N = 128, GB_K = 8;

// TB: B1 and B2 are read transposed (B[k][n] = Bt[n][k], ldb = row pitch of Bt).
template <class TA1, class TA2, class TO, bool TB = false>
__global__ void __launch_bounds__(256, 2) k_gemm2(int64_t M, int N, int Np, int K1, int K2,
                                                  const TA1* __restrict__ A1, int64_t lda1,
                                                  const int32_t* __restrict__ gidx, int64_t m1,
                                                  const TA2* __restrict__ A2, int64_t lda2,
                                                  const float* __restrict__ B1, int64_t ldb1,
                                                  const float* __restrict__ B2, int64_t ldb2,
                                                  const float* __restrict__ bias, int relu,
                                                  TO* __restrict__ Cm, int64_t ldc) {
  __shared__ __align__(16) float As[GB_K][GB_M + 4];
  __shared__ __align__(16) float Bs[GB_K][GB_N + 4];
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int64_t m0 = (int64_t)blockIdx.x * GB_M;
  const int n0 = blockIdx.y * GB_N;
  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  const int nk1 = (K1 + GB_K - 1) / GB_K, nk2 = (K2 + GB_K - 1) / GB_K;
  // A loads: row ar = tid / 2, k ak .. ak + 3 (ak = 0 or 4); gathered row index read once
  const int ar = tid >> 1, ak = (tid & 1) * 4;
  const int64_t r = m0 + ar;
  int64_t rr1 = -1;
  if (r < M && r < m1) rr1 = gidx ? (int64_t)gidx[r] : r;
  // B loads: plain: k bk = tid / 32, n bn .. bn + 3; transposed: n tn = tid / 2, k tk .. tk + 3
  const int bk = tid >> 5, bn = (tid & 31) * 4;
  float ra[4], rb[4];
  auto load = [&](int kt) {
    const bool first = kt < nk1;
    const int k0 = first ? kt * GB_K : (kt - nk1) * GB_K;
    const int K = first ? K1 : K2;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int k = k0 + ak + q;
      float v = 0.f;
      if (k < K) {
        if (first) {
          if (rr1 >= 0) v = ld1<TA1>(A1 + rr1 * lda1 + k);
        } else if (r < M) {
          v = ld1<TA2>(A2 + r * lda2 + k);
        }
      }
      ra[q] = v;
    }
    const float* B = first ? B1 : B2;
    const int64_t ldb = first ? ldb1 : ldb2;
    if (TB) {
      const int nn = n0 + ar;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int k = k0 + ak + q;
        rb[q] = (k < K && nn < N) ? __ldg(B + (int64_t)nn * ldb + k) : 0.f;
      }
    } else {
      const int k = k0 + bk;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int nn = n0 + bn + q;
        rb[q] = (k < K && nn < N) ? __ldg(B + (int64_t)k * ldb + nn) : 0.f;
      }
    }
  };
  const int nkt = nk1 + nk2;
  if (nkt > 0) load(0);
  for (int kt = 0; kt < nkt; ++kt) {
#pragma unroll
    for (int q = 0; q < 4; ++q) As[ak + q][ar] = ra[q];
    if (TB) {
#pragma unroll
      for (int q = 0; q < 4; ++q) Bs[ak + q][ar] = rb[q];
    } else {
      *reinterpret_cast<float4*>(&Bs[bk][bn]) = make_float4(rb[0], rb[1], rb[2], rb[3]);
    }
    __syncthreads();
    if (kt + 1 < nkt) load(kt + 1);              // global loads in flight during the math
#pragma unroll
    for (int kk = 0; kk < GB_K; ++kk) {
      float a[8], b[8];
      const float4 a0 = *reinterpret_cast<const float4*>(&As[kk][ty * 8]);
      const float4 a1 = *reinterpret_cast<const float4*>(&As[kk][ty * 8 + 4]);
      a[0] = a0.x; a[1] = a0.y; a[2] = a0.z; a[3] = a0.w;
      a[4] = a1.x; a[5] = a1.y; a[6] = a1.z; a[7] = a1.w;
      const float4 b0 = *reinterpret_cast<const float4*>(&Bs[kk][tx * 4]);
      const float4 b1 = *reinterpret_cast<const float4*>(&Bs[kk][64 + tx * 4]);
      b[0] = b0.x; b[1] = b0.y; b[2] = b0.z; b[3] = b0.w;
      b[4] = b1.x; b[5] = b1.y; b[6] = b1.z; b[7] = b1.w;
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(a[i], b[j], acc[i][j]);
    }
    __syncthreads();
  }
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int64_t row = m0 + ty * 8 + i;
    if (row >= M) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int nn = n0 + (j < 4 ? tx * 4 + j : 64 + tx * 4 + (j - 4));
      if (nn >= Np) continue;
      float v = 0.f;
      if (nn < N) {
        v = acc[i][j] + (bias ? bias[nn] : 0.f);
        if (relu) v = fmaxf(v, 0.f);
      }
      st1<TO>(Cm + row * ldc + nn, v);
    }
  }
}

// ------------------------------------------------------------------ fp32 GEMM on tensor pipes (3xTF32)
// Same contract as k_gemm2 (used by the pool / LSTM / GAT paths, whose GEMMs have K <= 2 d <= 512):
// each operand is split x = hi + lo into two TF32 values and the product summed as
// hi*hi + hi*lo + lo*hi (mma.sync m16n8k8, fp32 accumulate), fp32-level accuracy for these short
// K.  The long split-K reductions (k_dw_partial) and the mean model's FFMA parity path stay on
// the CUDA-core kernels: their K runs over thousands of rows with heavy cancellation, where the
// tensor pipe's accumulation measured outside the fp32 parity tolerance (Cora dW_1).
// CTA tile 128 x 128, K step 8, 8 warps as 4 (M) x 2 (N), each 32 x 64 = 2 x 8 MMA tiles;
// operands staged fp32 in shared memory (pitch 136), next K step prefetched into registers.
constexpr int GB_P = 136;   // shared pitch of the 3xTF32 kernel (conflict-free fragment reads)

__device__ __forceinline__ uint32_t tf32_hi(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return r;
}
__device__ __forceinline__ void split_tf32(float x, uint32_t& hi, uint32_t& lo) {
  hi = tf32_hi(x);
  lo = tf32_hi(x - __uint_as_float(hi));
}
__device__ __forceinline__ void mma_tf32(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1) {
  asm volatile("mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0,%1,%2,%3}, {%4,%5,%6,%7}, {%8,%9}, "
               "{%0,%1,%2,%3};"
               : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
               : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}
// One K step of 8 on the warp's 32 x 64 tile: A element (m, k) = As[k][m], B element (k, n) =
// Bs[k][n]; wm0 / wn0: the warp's first row / column inside the CTA tile.
__device__ __forceinline__ void warp_mma_k8(const float (*As)[GB_P], const float (*Bs)[GB_P], int wm0, int wn0,
                                            float (&acc)[2][8][4]) {
  const int lane = threadIdx.x & 31, g = lane >> 2, t = lane & 3;
  uint32_t ah[2][4], al[2][4];
#pragma unroll
  for (int mt = 0; mt < 2; ++mt) {
    const int m = wm0 + mt * 16 + g;
    split_tf32(As[t][m], ah[mt][0], al[mt][0]);
    split_tf32(As[t][m + 8], ah[mt][1], al[mt][1]);
    split_tf32(As[t + 4][m], ah[mt][2], al[mt][2]);
    split_tf32(As[t + 4][m + 8], ah[mt][3], al[mt][3]);
  }
#pragma unroll
  for (int nt = 0; nt < 8; ++nt) {
    const int n = wn0 + nt * 8 + g;
    uint32_t bh0, bl0, bh1, bl1;
    split_tf32(Bs[t][n], bh0, bl0);
    split_tf32(Bs[t + 4][n], bh1, bl1);
#pragma unroll
    for (int mt = 0; mt < 2; ++mt) {
      mma_tf32(acc[mt][nt], al[mt], bh0, bh1);
      mma_tf32(acc[mt][nt], ah[mt], bl0, bl1);
      mma_tf32(acc[mt][nt], ah[mt], bh0, bh1);
    }
  }
}

// TB: B1 and B2 are read transposed (B[k][n] = Bt[n][k], ldb = row pitch of Bt).
template <class TA1, class TA2, class TO, bool TB = false>
__global__ void __launch_bounds__(256, 2) k_gemm2_tc(int64_t M, int N, int Np, int K1, int K2,
                                                  const TA1* __restrict__ A1, int64_t lda1,
                                                  const int32_t* __restrict__ gidx, int64_t m1,
                                                  const TA2* __restrict__ A2, int64_t lda2,
                                                  const float* __restrict__ B1, int64_t ldb1,
                                                  const float* __restrict__ B2, int64_t ldb2,
                                                  const float* __restrict__ bias, int relu,
                                                  TO* __restrict__ Cm, int64_t ldc) {
  __shared__ __align__(16) float As[GB_K][GB_P];
  __shared__ __align__(16) float Bs[GB_K][GB_P];
  const int tid = threadIdx.x, warp = tid >> 5;
  const int wm0 = (warp >> 1) * 32, wn0 = (warp & 1) * 64;
  const int64_t m0 = (int64_t)blockIdx.x * GB_M;
  const int n0 = blockIdx.y * GB_N;
  float acc[2][8][4];
#pragma unroll
  for (int i = 0; i < 2; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j)
#pragma unroll
      for (int c = 0; c < 4; ++c) acc[i][j][c] = 0.f;
  const int nk1 = (K1 + GB_K - 1) / GB_K, nk2 = (K2 + GB_K - 1) / GB_K;
  // A loads: row ar = tid / 2, k ak .. ak + 3 (ak = 0 or 4); gathered row index read once
  const int ar = tid >> 1, ak = (tid & 1) * 4;
  const int64_t r = m0 + ar;
  int64_t rr1 = -1;
  if (r < M && r < m1) rr1 = gidx ? (int64_t)gidx[r] : r;
  // B loads: plain: k bk = tid / 32, n bn .. bn + 3; transposed: n = tid / 2, k ak .. ak + 3
  const int bk = tid >> 5, bn = (tid & 31) * 4;
  float ra[4], rb[4];
  auto load = [&](int kt) {
    const bool first = kt < nk1;
    const int k0 = first ? kt * GB_K : (kt - nk1) * GB_K;
    const int K = first ? K1 : K2;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int k = k0 + ak + q;
      float v = 0.f;
      if (k < K) {
        if (first) {
          if (rr1 >= 0) v = ld1<TA1>(A1 + rr1 * lda1 + k);
        } else if (r < M) {
          v = ld1<TA2>(A2 + r * lda2 + k);
        }
      }
      ra[q] = v;
    }
    const float* B = first ? B1 : B2;
    const int64_t ldb = first ? ldb1 : ldb2;
    if (TB) {
      const int nn = n0 + ar;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int k = k0 + ak + q;
        rb[q] = (k < K && nn < N) ? __ldg(B + (int64_t)nn * ldb + k) : 0.f;
      }
    } else {
      const int k = k0 + bk;
#pragma unroll
      for (int q = 0; q < 4; ++q) {
        const int nn = n0 + bn + q;
        rb[q] = (k < K && nn < N) ? __ldg(B + (int64_t)k * ldb + nn) : 0.f;
      }
    }
  };
  const int nkt = nk1 + nk2;
  if (nkt > 0) load(0);
  for (int kt = 0; kt < nkt; ++kt) {
#pragma unroll
    for (int q = 0; q < 4; ++q) As[ak + q][ar] = ra[q];
    if (TB) {
#pragma unroll
      for (int q = 0; q < 4; ++q) Bs[ak + q][ar] = rb[q];
    } else {
      *reinterpret_cast<float4*>(&Bs[bk][bn]) = make_float4(rb[0], rb[1], rb[2], rb[3]);
    }
    __syncthreads();
    if (kt + 1 < nkt) load(kt + 1);              // global loads in flight during the MMAs
    warp_mma_k8(As, Bs, wm0, wn0, acc);
    __syncthreads();
  }
  const int lane = tid & 31, g = lane >> 2, t = lane & 3;
#pragma unroll
  for (int mt = 0; mt < 2; ++mt)
#pragma unroll
    for (int hh = 0; hh < 2; ++hh) {
      const int64_t row = m0 + wm0 + mt * 16 + g + 8 * hh;
      if (row >= M) continue;
#pragma unroll
      for (int nt = 0; nt < 8; ++nt)
#pragma unroll
        for (int cc = 0; cc < 2; ++cc) {
          const int nn = n0 + wn0 + nt * 8 + 2 * t + cc;
          if (nn >= Np) continue;
          float v = 0.f;
          if (nn < N) {
            v = acc[mt][nt][2 * hh + cc] + (bias ? bias[nn] : 0.f);
            if (relu) v = fmaxf(v, 0.f);
          }
          st1<TO>(Cm + row * ldc + nn, v);
        }
    }
}

// The dense GEMMs of every fp32-output path: tcgen05 kind::tf32 (tc_f32.cu) when the operands
// meet its 16-B row alignment, else the fallback kernel (SIMT k_gemm2 or the mma.sync
// k_gemm2_tc) on the same contract.  SIMT (the mean model's FFMA parity path) asks tcf_gemm for
// the exact 3-term split.
template <class TA1, class TA2, class TO, bool TB = false, bool SIMT = false>
static buffalo_status gemm2(dim3 grid, cudaStream_t s, int64_t M, int N, int Np, int K1, int K2, const TA1* A1,
                            int64_t lda1, const int32_t* gidx, int64_t m1, const TA2* A2, int64_t lda2,
                            const float* B1, int64_t ldb1, const float* B2, int64_t ldb2, const float* bias, int relu,
                            TO* C, int64_t ldc) {
  if (std::is_same<TA2, float>::value && std::is_same<TO, float>::value && K1 + K2 <= kTcfMaxK &&
      tcf_aligned(A1, lda1, sizeof(TA1)) &&
      tcf_aligned(A2, lda2, 4) && tcf_aligned(B1, ldb1, 4) && tcf_aligned(B2, ldb2, 4) && tcf_aligned(C, ldc, 4)) {
    TcfGemm p{};
    p.M = M; p.N = N; p.Np = Np; p.K1 = K1; p.K2 = K2;
    p.A1 = A1; p.lda1 = lda1; p.gidx = gidx; p.m1 = m1;
    p.A2 = (const float*)A2; p.lda2 = lda2;
    p.B1 = B1; p.ldb1 = ldb1; p.B2 = B2; p.ldb2 = ldb2;
    p.bias = bias; p.relu = relu; p.C = (float*)C; p.ldc = ldc;
    return tcf_gemm(p, std::is_same<TA1, __nv_bfloat16>::value, TB, SIMT, s);
  }
  if (SIMT) {
    k_gemm2<TA1, TA2, TO, TB><<<grid, 256, 0, s>>>(M, N, Np, K1, K2, A1, lda1, gidx, m1, A2, lda2, B1, ldb1, B2, ldb2,
                                                   bias, relu, C, ldc);
  } else {
    k_gemm2_tc<TA1, TA2, TO, TB><<<grid, 256, 0, s>>>(M, N, Np, K1, K2, A1, lda1, gidx, m1, A2, lda2, B1, ldb1, B2,
                                                      ldb2, bias, relu, C, ldc);
  }
  BF_LAUNCHED("k_gemm2");
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ backward pieces
template <class TH>
__global__ void k_dz_mask(float* __restrict__ dz, int64_t ldz, const TH* __restrict__ h, int64_t ldh,
                          int64_t n, int d) {
  const int64_t total = n * d;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = t / d;
    const int c = (int)(t - i * d);
    if (!(ld1<TH>(h + i * ldh + c) > 0.f)) dz[i * ldz + c] = 0.f;
  }
}

// Transposed aggregate: out[j] = sum_{t in T(j)} dZ[i_t] / D(i_t), ascending i_t.
__global__ void __launch_bounds__(256) k_aggT(const int32_t* __restrict__ trp, const int32_t* __restrict__ tcol,
                                              const int32_t* __restrict__ rp, int64_t n_src,
                                              const float* __restrict__ dz, int64_t ldz, int d,
                                              float* __restrict__ out, int64_t ldo, int dp) {
  const int lane = threadIdx.x & 31;
  const int nch = (dp + 3) / 4;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_src; j += warps) {
    const int32_t b = trp[j], e_end = trp[j + 1];
    for (int c = lane; c < nch; c += 32) {
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      for (int32_t t = b; t < e_end; ++t) {
        const int64_t i = tcol[t];
        const float fd = (float)(rp[i + 1] - rp[i]);
        float v[4];
        VecIO<float, 4>::load(dz + i * ldz + c * 4, v);
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[k] += v[k] / fd;
      }
#pragma unroll
      for (int k = 0; k < 4; ++k)
        if (c * 4 + k >= d) acc[k] = 0.f;
      VecIO<float, 4>::store(out + j * ldo + c * 4, acc);
    }
  }
}

// dW partial of split s: part[s][n][k] = sum_{r in split s} dZ[r][n] * Afwd[r][k],
// Afwd[r] = [self(r) || agg(r)].
// K = 2 d_in (Update weight: [self || agg]) or d_in (pool weight: self rows only).
// CTA tile 128 (n) x 128 (k) over one row split, 8 rows per step, 8 x 8 register tile per
// thread, next step prefetched into registers; db partial (column sums of dZ, fixed row order)
// by the CTAs of k-tile 0.
constexpr int DW_T = 128, DW_R = 8;
template <class TS, class TG>
__global__ void __launch_bounds__(256, 2) k_dw_partial(int64_t nrows, int d_out, int d_in, int K,
                                                       const float* __restrict__ dz, int64_t ldz,
                                                       const TS* __restrict__ self, int64_t lds,
                                                       const int32_t* __restrict__ gidx,
                                                       const TG* __restrict__ agg, int64_t ldg,
                                                       int64_t rows_per_split, float* __restrict__ part,
                                                       float* __restrict__ db_part) {
  __shared__ __align__(16) float Zs[DW_R][DW_T + 4];
  __shared__ __align__(16) float As[DW_R][DW_T + 4];
  const int tid = threadIdx.x, tx = tid & 15, ty = tid >> 4;
  const int k0 = blockIdx.x * DW_T, n0 = blockIdx.y * DW_T;
  const int64_t r_beg = (int64_t)blockIdx.z * rows_per_split;
  const int64_t r_end = min(nrows, r_beg + rows_per_split);
  float acc[8][8];
#pragma unroll
  for (int i = 0; i < 8; ++i)
#pragma unroll
    for (int j = 0; j < 8; ++j) acc[i][j] = 0.f;
  const bool do_db = blockIdx.x == 0 && tid < DW_T;
  float dbs = 0.f;
  // loads: row lr = tid / 32 of the step, 4 consecutive columns lc .. lc + 3
  const int lr = tid >> 5, lc = (tid & 31) * 4;
  float rz[4], ra[4];
  auto load = [&](int64_t r0) {
    const int64_t rw = r0 + lr;
    const bool in = rw < r_end;
    const int64_t rs = (in && gidx) ? (int64_t)gidx[rw] : rw;
#pragma unroll
    for (int q = 0; q < 4; ++q) {
      const int nn = n0 + lc + q, k = k0 + lc + q;
      rz[q] = (in && nn < d_out) ? dz[rw * ldz + nn] : 0.f;
      float a = 0.f;
      if (in) {
        if (k < d_in) a = ld1<TS>(self + rs * lds + k);
        else if (k < K) a = ld1<TG>(agg + rw * ldg + (k - d_in));
      }
      ra[q] = a;
    }
  };
  if (r_beg < r_end) load(r_beg);
  for (int64_t r0 = r_beg; r0 < r_end; r0 += DW_R) {
    *reinterpret_cast<float4*>(&Zs[lr][lc]) = make_float4(rz[0], rz[1], rz[2], rz[3]);
    *reinterpret_cast<float4*>(&As[lr][lc]) = make_float4(ra[0], ra[1], ra[2], ra[3]);
    __syncthreads();
    if (r0 + DW_R < r_end) load(r0 + DW_R);
    if (do_db)
#pragma unroll
      for (int rr = 0; rr < DW_R; ++rr) dbs += Zs[rr][tid];
#pragma unroll
    for (int rr = 0; rr < DW_R; ++rr) {
      float z[8], a[8];
      const float4 z0 = *reinterpret_cast<const float4*>(&Zs[rr][ty * 8]);
      const float4 z1 = *reinterpret_cast<const float4*>(&Zs[rr][ty * 8 + 4]);
      z[0] = z0.x; z[1] = z0.y; z[2] = z0.z; z[3] = z0.w;
      z[4] = z1.x; z[5] = z1.y; z[6] = z1.z; z[7] = z1.w;
      const float4 a0 = *reinterpret_cast<const float4*>(&As[rr][tx * 4]);
      const float4 a1 = *reinterpret_cast<const float4*>(&As[rr][64 + tx * 4]);
      a[0] = a0.x; a[1] = a0.y; a[2] = a0.z; a[3] = a0.w;
      a[4] = a1.x; a[5] = a1.y; a[6] = a1.z; a[7] = a1.w;
#pragma unroll
      for (int i = 0; i < 8; ++i)
#pragma unroll
        for (int j = 0; j < 8; ++j) acc[i][j] = fmaf(z[i], a[j], acc[i][j]);
    }
    __syncthreads();
  }
  if (do_db && n0 + tid < d_out) db_part[(int64_t)blockIdx.z * d_out + n0 + tid] = dbs;
  float* P = part + (int64_t)blockIdx.z * d_out * K;
#pragma unroll
  for (int i = 0; i < 8; ++i) {
    const int nn = n0 + ty * 8 + i;
    if (nn >= d_out) continue;
#pragma unroll
    for (int j = 0; j < 8; ++j) {
      const int k = k0 + (j < 4 ? tx * 4 + j : 64 + tx * 4 + (j - 4));
      if (k < K) P[(int64_t)nn * K + k] = acc[i][j];
    }
  }
}

__global__ void k_reduce_partials(const float* __restrict__ part, int S, int64_t count, float* __restrict__ out) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < count; j += (int64_t)gridDim.x * blockDim.x) {
    float s = 0.f;
    for (int q = 0; q < S; ++q) s += part[(int64_t)q * count + j];
    out[j] += s;
  }
}

// Column sums of x [n][d] over row splits of rps rows: part[s][c] (fixed order: deterministic);
// wt (nullable): weighted sums, row i scaled by wt[i] (GAT's da_l = d_el^T Z, da_r = d_er^T Z).
__global__ void __launch_bounds__(256) k_colsum_partial(const float* __restrict__ x, int64_t ldx, int64_t n, int d,
                                                        int64_t rps, float* __restrict__ part,
                                                        const float* __restrict__ wt = nullptr) {
  __shared__ float sh[8][33];
  const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + lane;
  const int64_t r0 = (int64_t)blockIdx.y * rps, r1 = min(n, r0 + rps);
  float s = 0.f;
  if (c < d) {
    if (wt) {
      for (int64_t i = r0 + warp; i < r1; i += 8) s = fmaf(__ldg(wt + i), __ldg(x + i * ldx + c), s);
    } else {
      for (int64_t i = r0 + warp; i < r1; i += 8) s += x[i * ldx + c];
    }
  }
  sh[warp][lane] = s;
  __syncthreads();
  if (warp == 0 && c < d) {
    float t = 0.f;
    for (int w = 0; w < 8; ++w) t += sh[w][lane];
    part[(int64_t)blockIdx.y * d + c] = t;
  }
}

// dW partials part[s][n][k] and db partials db_part[s][n] (the k_dw_partial contract): on the
// tensor cores (tc_f32.cu: 6xTF32 with per-chunk fp32 accumulation) plus a fixed-order column sum
// for db when the operand rows are 16-B aligned; otherwise (e.g. GAT's d_el vectors, ld = 1) on
// the CUDA-core kernel above.
template <class TS, class TG>
static buffalo_status dw_partial(dim3 grid, cudaStream_t s, int64_t nrows, int d_out, int d_in, int K, const float* dz,
                                 int64_t ldz, const TS* self, int64_t lds, const int32_t* gidx, const TG* agg,
                                 int64_t ldg, int64_t rows_per_split, float* part, float* db_part) {
  const bool halves = K == 2 * d_in && agg;
  if (std::is_same<TG, float>::value && (halves || (K == d_in && !agg)) && tcf_aligned(dz, ldz, 4) &&
      tcf_aligned(self, lds, sizeof(TS)) && tcf_aligned(agg, ldg, 4)) {
    const int S = (int)grid.z;
    TcfDw p{};
    p.n = nrows; p.d_out = d_out; p.d_in = d_in;
    p.Z = dz; p.ldz = ldz; p.self = self; p.lds = lds; p.gidx = gidx;
    p.agg = (const float*)agg; p.lda = ldg; p.part = part;
    if (std::is_same<TS, float>::value) BF_CHECK(tcf_dw_tma(p, S, s));
    else BF_CHECK(tcf_dw(p, S, true, s));
    if (db_part) {
      k_colsum_partial<<<dim3((unsigned)ceil_div(d_out, 32), (unsigned)S), 256, 0, s>>>(dz, ldz, nrows, d_out,
                                                                                         rows_per_split, db_part);
      BF_LAUNCHED("k_colsum_partial");
    }
    return BUFFALO_OK;
  }
  k_dw_partial<TS, TG><<<grid, 256, 0, s>>>(nrows, d_out, d_in, K, dz, ldz, self, lds, gidx, agg, ldg, rows_per_split,
                                            part, db_part);
  BF_LAUNCHED("k_dw_partial");
  return BUFFALO_OK;
}

// ------------------------------------------------------------------ loss, optimizer, packing
__global__ void __launch_bounds__(256) k_softmax_ce(const float* __restrict__ z, int64_t ld, int64_t n, int classes,
                                                    const int32_t* __restrict__ labels,
                                                    const int32_t* __restrict__ ids, float invS,
                                                    float* __restrict__ loss, float* __restrict__ dl,
                                                    int64_t ldd) {
  __shared__ float sw[8];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int64_t warps = (int64_t)gridDim.x * 8;
  float blk_loss = 0.f;
  for (int64_t i = blockIdx.x * 8LL + w; i < n; i += warps) {
    const float* zi = z + i * ld;
    const int y = labels[ids[i]];
    float m = -INFINITY;
    for (int c = lane; c < classes; c += 32) m = fmaxf(m, zi[c]);
#pragma unroll
    for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float s = 0.f;
    for (int c = lane; c < classes; c += 32) s += expf(zi[c] - m);
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    const float lse = m + logf(s);
    for (int c = lane; c < (int)ldd; c += 32) {
      float g = 0.f;
      if (c < classes) g = (expf(zi[c] - m) / s - (c == y ? 1.f : 0.f)) * invS;
      dl[i * ldd + c] = g;
    }
    if (lane == 0) blk_loss += (lse - zi[y]) * invS;
  }
  if (lane == 0) sw[w] = blk_loss;
  __syncthreads();
  if (threadIdx.x == 0) {
    float t = 0.f;
    for (int k = 0; k < 8; ++k) t += sw[k];
    atomicAdd(loss, t);
  }
}

__global__ void k_sgd(float* __restrict__ p, float* __restrict__ g, int64_t n, float lr) {
  for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
    p[j] -= lr * g[j];
    g[j] = 0.f;
  }
}

__global__ void k_transpose_w(const float* __restrict__ W, int rows, int cols, float* __restrict__ Wt) {
  const int64_t total = (int64_t)rows * cols;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int r = (int)(t / cols), c = (int)(t % cols);
    Wt[(int64_t)c * rows + r] = W[t];
  }
}

// ================================================================== host launchers
// Long-tail rows of the tensor-core path: mean written (bf16) into the saved h_agg, which the
// fused kernel then reads instead of gathering.
buffalo_status launch_agg_heavy_bf16(const FwdArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  const int32_t* col = a.layer1 ? blk->col_global : blk->col_local;
  const bool wide = a.d_in > 128;
  __nv_bfloat16* agg = (__nv_bfloat16*)a.agg;
  const int g = heavy_tail_grid(blk->n_heavy, blk->n_edges);
  if (g <= 0) return BUFFALO_OK;
  const int32_t* perm = blk->cls_perm;
  const int64_t n = blk->n_dst;
  if (a.in_bf16) {
    const __nv_bfloat16* h = (const __nv_bfloat16*)a.h_src;
    if (wide) k_agg_heavy<__nv_bfloat16, __nv_bfloat16, 8><<<g, 256, 0, s>>>(perm, n, blk->row_ptr, col, h, a.ld_src, a.d_in, agg, a.ld_agg);
    else k_agg_heavy<__nv_bfloat16, __nv_bfloat16, 4><<<g, 256, 0, s>>>(perm, n, blk->row_ptr, col, h, a.ld_src, a.d_in, agg, a.ld_agg);
  } else {
    const float* h = (const float*)a.h_src;
    if (wide) k_agg_heavy<float, __nv_bfloat16, 8><<<g, 256, 0, s>>>(perm, n, blk->row_ptr, col, h, a.ld_src, a.d_in, agg, a.ld_agg);
    else k_agg_heavy<float, __nv_bfloat16, 4><<<g, 256, 0, s>>>(perm, n, blk->row_ptr, col, h, a.ld_src, a.d_in, agg, a.ld_agg);
  }
  BF_LAUNCHED("k_agg_heavy");
  return BUFFALO_OK;
}

buffalo_status launch_softmax_ce(const float* logits, int64_t ld, int64_t n, int classes,
                                 const int32_t* labels, const int32_t* ids, int64_t S,
                                 float* loss, float* dl, int64_t ldd, cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  k_softmax_ce<<<grid_for(n, 8, 16), 256, 0, s>>>(logits, ld, n, classes, labels, ids, 1.0f / (float)S,
                                                  loss, dl, ldd);
  BF_LAUNCHED("k_softmax_ce");
  return BUFFALO_OK;
}

buffalo_status launch_sgd(float* p, float* g, int64_t n, float lr, cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  k_sgd<<<grid_for(n, 256), 256, 0, s>>>(p, g, n, lr);
  BF_LAUNCHED("k_sgd");
  return BUFFALO_OK;
}

buffalo_status launch_transpose_w(const float* W, int rows, int cols, float* Wt, cudaStream_t s) {
  k_transpose_w<<<grid_for((int64_t)rows * cols, 256), 256, 0, s>>>(W, rows, cols, Wt);
  BF_LAUNCHED("k_transpose_w");
  return BUFFALO_OK;
}

template <class TI, class TA>
static buffalo_status fwd_ffma_t(const FwdArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  const int32_t* col = a.layer1 ? blk->col_global : blk->col_local;
  BF_CHECK(launch_agg<TI, TA>(blk, col, (const TI*)a.h_src, a.ld_src, a.d_in, (TA*)a.agg, a.ld_agg, s));
  const int64_t M = blk->n_dst;
  if (M <= 0) return BUFFALO_OK;
  const int Np = (int)pitch_of(a.d_out);
  dim3 grid((unsigned)ceil_div(M, GB_M), (unsigned)ceil_div(Np, GB_N));
  const float* Wt = (const float*)a.W_packed;   // [2 d_in][d_out]
  if (a.out_f32) {
    BF_CHECK((gemm2<TI, TA, float, false, true>(grid, s, M, a.d_out, Np, a.d_in, a.d_in, (const TI*)a.h_src, a.ld_src,
                                               a.layer1 ? blk->src_global : nullptr, M, (const TA*)a.agg,
                                               a.ld_agg, Wt, a.d_out, Wt + (int64_t)a.d_in * a.d_out,
                                               a.d_out, a.b, a.relu, (float*)a.out, a.ld_out)));
  } else {
    BF_CHECK((gemm2<TI, TA, TA, false, true>(grid, s, M, a.d_out, Np, a.d_in, a.d_in, (const TI*)a.h_src, a.ld_src,
                                            a.layer1 ? blk->src_global : nullptr, M, (const TA*)a.agg,
                                            a.ld_agg, Wt, a.d_out, Wt + (int64_t)a.d_in * a.d_out,
                                            a.d_out, a.b, a.relu, (TA*)a.out, a.ld_out)));
  }
  return BUFFALO_OK;
}

buffalo_status sage_fwd_ffma(const FwdArgs& a, cudaStream_t s) {
  if (a.in_bf16 && a.act_bf16) return fwd_ffma_t<__nv_bfloat16, __nv_bfloat16>(a, s);
  if (a.in_bf16 && !a.act_bf16) return fwd_ffma_t<__nv_bfloat16, float>(a, s);
  if (!a.in_bf16 && a.act_bf16) return fwd_ffma_t<float, __nv_bfloat16>(a, s);
  return fwd_ffma_t<float, float>(a, s);
}

int dw_splits(int64_t n_l, int d_out, int d_in) {
  int64_t tiles = ceil_div(d_out, 64) * ceil_div(2 * d_in, 64);
  int64_t a = ceil_div(592, tiles), b = ceil_div(n_l, 512);
  int64_t sp = a < b ? a : b;
  return (int)(sp < 1 ? 1 : sp);
}

int64_t bwd_scratch_bytes(int64_t n_dst, int64_t n_src, int layer, int d_in, int d_out) {
  int S = dw_splits(n_dst, d_out, d_in);
  int64_t b = R((int64_t)S * d_out * 2 * d_in * 4) + R((int64_t)S * pitch_of(d_out) * 4);
  if (layer >= 2) b += R(n_src * pitch_of(d_out) * 4);
  return b;
}

template <class TS, class TG, class TH>
static buffalo_status bwd_ffma_t(const BwdArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  const int64_t n = blk->n_dst;
  const int d_in = a.d_in, d_out = a.d_out;
  if (!a.last && n > 0) {
    k_dz_mask<TH><<<grid_for(n * d_out, 256), 256, 0, s>>>(a.dh, a.ld_dh, (const TH*)a.h_dst, a.ld_hdst, n, d_out);
    BF_LAUNCHED("k_dz_mask");
  }
  const int S = dw_splits(n, d_out, d_in);
  char* q = (char*)a.scratch;
  float* dw_part = (float*)q; q += R((int64_t)S * d_out * 2 * d_in * 4);
  float* db_part = (float*)q; q += R((int64_t)S * pitch_of(d_out) * 4);
  float* aggT = (float*)q;
  const int64_t rps = ceil_div(n > 0 ? n : 1, S);
  if (n > 0) {
    dim3 g((unsigned)ceil_div(2 * d_in, DW_T), (unsigned)ceil_div(d_out, DW_T), (unsigned)S);
    BF_CHECK((dw_partial<TS, TG>(g, s, n, d_out, d_in, 2 * d_in, a.dh, a.ld_dh, (const TS*)a.h_src, a.ld_src,
                                           a.layer1 ? blk->src_global : nullptr, (const TG*)a.agg,
                                           a.ld_agg, rps, dw_part, db_part)));
    k_reduce_partials<<<grid_for((int64_t)d_out * 2 * d_in, 256), 256, 0, s>>>(dw_part, S, (int64_t)d_out * 2 * d_in, a.dW);
    BF_LAUNCHED("k_reduce_partials");
    k_reduce_partials<<<1, 256, 0, s>>>(db_part, S, d_out, a.db);
    BF_LAUNCHED("k_reduce_partials");
  }
  if (a.dh_src) {
    const int64_t ns = blk->n_src;
    if (ns <= 0) return BUFFALO_OK;
    const int dp = (int)pitch_of(d_out);
    const ProfSlot ps = prof_begin_launch("gather", s);
    k_aggT<<<grid_for(ns * 32, 256, 16), 256, 0, s>>>(blk->t_row_ptr, blk->t_col, blk->row_ptr, ns, a.dh,
                                                     a.ld_dh, d_out, aggT, dp, dp);
    BF_LAUNCHED("k_aggT");
    // algorithmic bytes: per src row the t_row_ptr pair + the fp32 output row; per entry the dst
    // index, its row_ptr pair (1/D) and the dZ row
    prof_end_launch(ps, s, (double)ns * (8.0 + 4.0 * dp) + (double)blk->n_edges * (12.0 + 4.0 * dp), 0.0);
    const int Np = (int)pitch_of(d_in);
    dim3 grid((unsigned)ceil_div(ns, GB_M), (unsigned)ceil_div(Np, GB_N));
    BF_CHECK((gemm2<float, float, float, false, true>(grid, s, ns, d_in, Np, d_out, d_out, a.dh, a.ld_dh, nullptr, n,
                                                      aggT, dp, a.W, 2 * d_in, a.W + d_in, 2 * d_in,
                                                      nullptr, 0, a.dh_src, a.ld_dh_src)));
  }
  return BUFFALO_OK;
}

buffalo_status sage_bwd_ffma(const BwdArgs& a, cudaStream_t s) {
  // TS: dtype of the layer input rows (features at layer 1), TG/TH: activation dtype
  if (a.in_bf16 && a.act_bf16) return bwd_ffma_t<__nv_bfloat16, __nv_bfloat16, __nv_bfloat16>(a, s);
  if (a.in_bf16 && !a.act_bf16) return bwd_ffma_t<__nv_bfloat16, float, float>(a, s);
  if (!a.in_bf16 && a.act_bf16) return bwd_ffma_t<float, __nv_bfloat16, __nv_bfloat16>(a, s);
  return bwd_ffma_t<float, float, float>(a, s);
}

// ================================================================== GraphSAGE-pool (R28)
// Neighbour max of the pooled rows: warp per dst row (degree-class order), each lane owns
// 4-column chunks; strict '>' keeps the first neighbour (CSR order) attaining the max; the
// running max starts at 0 (P >= 0), so arg = -1 exactly where the max is 0 (or D = 0).
__global__ void __launch_bounds__(256) k_pool_max(const int32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                  const int32_t* __restrict__ perm, int64_t n,
                                                  const float* __restrict__ P, int64_t ldp, int d,
                                                  float* __restrict__ agg, int64_t ld_agg,
                                                  int32_t* __restrict__ arg, int64_t ld_arg) {
  const int lane = threadIdx.x & 31;
  const int nch = (int)(pitch_of(d) / 4);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w < n; w += warps) {
    const int64_t i = perm ? perm[w] : w;
    const int32_t e0 = rp[i], e1 = rp[i + 1];
    for (int c = lane; c < nch; c += 32) {
      float best[4] = {0.f, 0.f, 0.f, 0.f};
      int32_t am[4] = {-1, -1, -1, -1};
      for (int32_t e = e0; e < e1; ++e) {
        const int32_t j = col[e];
        float v[4];
        VecIO<float, 4>::load(P + (int64_t)j * ldp + c * 4, v);
#pragma unroll
        for (int q = 0; q < 4; ++q)
          if (v[q] > best[q]) { best[q] = v[q]; am[q] = j; }
      }
      VecIO<float, 4>::store(agg + i * ld_agg + c * 4, best);
      *reinterpret_cast<int4*>(arg + i * ld_arg + c * 4) = make_int4(am[0], am[1], am[2], am[3]);
    }
  }
}

// dQ[j] = 1[P[j] > 0] * sum over the dst i of src j (transposed block, ascending i) of
// dh_agg[i] restricted to the columns whose argmax is j.  Warp per src row.
__global__ void __launch_bounds__(256) k_pool_scatterT(const int32_t* __restrict__ trp, const int32_t* __restrict__ tcol,
                                                       int64_t n_src, const int32_t* __restrict__ arg, int64_t ld_arg,
                                                       const float* __restrict__ dagg, int64_t ld_dagg,
                                                       const float* __restrict__ P, int64_t ldp, int d,
                                                       float* __restrict__ dq, int64_t ldq) {
  const int lane = threadIdx.x & 31;
  const int nch = (int)(pitch_of(d) / 4);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_src; j += warps) {
    const int32_t t0 = trp[j], t1 = trp[j + 1];
    for (int c = lane; c < nch; c += 32) {
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      for (int32_t t = t0; t < t1; ++t) {
        const int64_t i = tcol[t];
        const int4 a4 = __ldg(reinterpret_cast<const int4*>(arg + i * ld_arg + c * 4));
        float g[4];
        VecIO<float, 4>::load(dagg + i * ld_dagg + c * 4, g);
        acc[0] += a4.x == (int32_t)j ? g[0] : 0.f;
        acc[1] += a4.y == (int32_t)j ? g[1] : 0.f;
        acc[2] += a4.z == (int32_t)j ? g[2] : 0.f;
        acc[3] += a4.w == (int32_t)j ? g[3] : 0.f;
      }
      float p[4];
      VecIO<float, 4>::load(P + j * ldp + c * 4, p);
#pragma unroll
      for (int q = 0; q < 4; ++q)
        if (!(p[q] > 0.f) || c * 4 + q >= d) acc[q] = 0.f;
      VecIO<float, 4>::store(dq + j * ldq + c * 4, acc);
    }
  }
}

int pool_dw_splits(int64_t n_rows, int d) {
  const int64_t tiles = ceil_div(d, 64) * ceil_div(d, 64);
  const int64_t a = ceil_div(592, tiles), b = ceil_div(n_rows, 512);
  const int64_t sp = a < b ? a : b;
  return (int)(sp < 1 ? 1 : sp);
}

// Layout of the pool backward scratch (R15 restated in DESIGN.md §5): dW/db partials of the
// Update weight, dh_agg, dQ, dW_pool/db_pool partials.
int64_t pool_bwd_scratch_bytes(int64_t n_dst, int64_t n_src, int d_in, int d_out) {
  const int S = dw_splits(n_dst, d_out, d_in), S2 = pool_dw_splits(n_src, d_in);
  return R((int64_t)S * d_out * 2 * d_in * 4) + R((int64_t)S * pitch_of(d_out) * 4) +
         R(n_dst * pitch_of(d_in) * 4) + R(n_src * pitch_of(d_in) * 4) +
         R((int64_t)S2 * d_in * d_in * 4) + R((int64_t)S2 * pitch_of(d_in) * 4);
}

template <class TI>
static buffalo_status pool_fwd_t(const PoolArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  const int64_t ns = blk->n_src, nd = blk->n_dst;
  const int dp = (int)pitch_of(a.d_in);
  const int32_t* gidx = a.layer1 ? blk->src_global : nullptr;
  if (ns > 0) {   // P = ReLU(H W_pool^T + b_pool)
    dim3 grid((unsigned)ceil_div(ns, GB_M), (unsigned)ceil_div(dp, GB_N));
    BF_CHECK((gemm2<TI, float, float, true, false>(grid, s, ns, a.d_in, dp, a.d_in, 0, (const TI*)a.h_src, a.ld_src,
                                                        gidx, ns, nullptr, 0, a.W_pool, a.d_in, nullptr, 0,
                                                        a.b_pool, 1, a.P, a.ld_pool)));
  }
  if (nd <= 0) return BUFFALO_OK;
  const ProfSlot ps = prof_begin_launch("pool_max", s);
  k_pool_max<<<grid_for(nd * 32, 256, 16), 256, 0, s>>>(blk->row_ptr, blk->col_local, blk->cls_perm, nd, a.P,
                                                        a.ld_pool, a.d_in, a.agg, a.ld_agg, a.arg, a.ld_pool);
  BF_LAUNCHED("k_pool_max");
  // algorithmic bytes: per row perm + row_ptr pair + the max and argmax rows written; per edge
  // the index and the pooled source row (the edge count is known on the host: no counter)
  prof_end_launch(ps, s, (double)nd * (12.0 + 8.0 * dp) + (double)blk->n_edges * (4.0 + 4.0 * dp), 0.0);
  const int Np = (int)pitch_of(a.d_out);
  dim3 grid((unsigned)ceil_div(nd, GB_M), (unsigned)ceil_div(Np, GB_N));
  const float* Wt = a.W_packed;   // [2 d_in][d_out]
  BF_CHECK((gemm2<TI, float, float, false, false>(grid, s, nd, a.d_out, Np, a.d_in, a.d_in, (const TI*)a.h_src, a.ld_src,
                                                gidx, nd, a.agg, a.ld_agg, Wt, a.d_out,
                                                Wt + (int64_t)a.d_in * a.d_out, a.d_out, a.b, !a.last, a.out,
                                                a.ld_out)));
  return BUFFALO_OK;
}

buffalo_status pool_fwd_ffma(const PoolArgs& a, cudaStream_t s) {
  return a.in_bf16 ? pool_fwd_t<__nv_bfloat16>(a, s) : pool_fwd_t<float>(a, s);
}

template <class TI>
static buffalo_status pool_bwd_t(const PoolArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  const int64_t n = blk->n_dst, ns = blk->n_src;
  const int d_in = a.d_in, d_out = a.d_out, dp = (int)pitch_of(d_in);
  const int32_t* gidx = a.layer1 ? blk->src_global : nullptr;
  if (!a.last && n > 0) {
    k_dz_mask<float><<<grid_for(n * d_out, 256), 256, 0, s>>>(a.dh, a.ld_dh, a.h_dst, a.ld_hdst, n, d_out);
    BF_LAUNCHED("k_dz_mask");
  }
  const int S = dw_splits(n, d_out, d_in), S2 = pool_dw_splits(ns, d_in);
  char* q = (char*)a.scratch;
  float* dw_part = (float*)q; q += R((int64_t)S * d_out * 2 * d_in * 4);
  float* db_part = (float*)q; q += R((int64_t)S * pitch_of(d_out) * 4);
  float* dagg = (float*)q; q += R(n * dp * 4);
  float* dq = (float*)q; q += R(ns * dp * 4);
  float* dwp_part = (float*)q; q += R((int64_t)S2 * d_in * d_in * 4);
  float* dbp_part = (float*)q;
  if (n > 0) {
    // dW, db of the Update weight (as the mean path)
    dim3 g((unsigned)ceil_div(2 * d_in, DW_T), (unsigned)ceil_div(d_out, DW_T), (unsigned)S);
    BF_CHECK((dw_partial<TI, float>(g, s, n, d_out, d_in, 2 * d_in, a.dh, a.ld_dh, (const TI*)a.h_src,
                                              a.ld_src, gidx, a.agg, a.ld_agg, ceil_div(n, S), dw_part, db_part)));
    k_reduce_partials<<<grid_for((int64_t)d_out * 2 * d_in, 256), 256, 0, s>>>(dw_part, S, (int64_t)d_out * 2 * d_in, a.dW);
    BF_LAUNCHED("k_reduce_partials");
    k_reduce_partials<<<1, 256, 0, s>>>(db_part, S, d_out, a.db);
    BF_LAUNCHED("k_reduce_partials");
    // dh_agg = dZ W_neigh  (B[k][n] = W[k][d_in + n])
    dim3 gg((unsigned)ceil_div(n, GB_M), (unsigned)ceil_div(dp, GB_N));
    BF_CHECK((gemm2<float, float, float, false, false>(gg, s, n, d_in, dp, d_out, 0, a.dh, a.ld_dh, nullptr, n, nullptr, 0,
                                                   a.W + d_in, 2 * d_in, nullptr, 0, nullptr, 0, dagg, dp)));
  }
  if (ns <= 0) return BUFFALO_OK;
  if (n > 0) {
    k_pool_scatterT<<<grid_for(ns * 32, 256, 16), 256, 0, s>>>(blk->t_row_ptr, blk->t_col, ns, a.arg, a.ld_pool,
                                                               dagg, dp, a.P, a.ld_pool, d_in, dq, dp);
    BF_LAUNCHED("k_pool_scatterT");
  } else {
    BF_CUDA(cudaMemsetAsync(dq, 0, sizeof(float) * ns * dp, s));
  }
  // dW_pool, db_pool over the src rows
  dim3 g2((unsigned)ceil_div(d_in, DW_T), (unsigned)ceil_div(d_in, DW_T), (unsigned)S2);
  BF_CHECK((dw_partial<TI, float>(g2, s, ns, d_in, d_in, d_in, dq, dp, (const TI*)a.h_src, a.ld_src, gidx,
                                             nullptr, 0, ceil_div(ns, S2), dwp_part, dbp_part)));
  k_reduce_partials<<<grid_for((int64_t)d_in * d_in, 256), 256, 0, s>>>(dwp_part, S2, (int64_t)d_in * d_in, a.dW_pool);
  BF_LAUNCHED("k_reduce_partials");
  k_reduce_partials<<<1, 256, 0, s>>>(dbp_part, S2, d_in, a.db_pool);
  BF_LAUNCHED("k_reduce_partials");
  if (a.dh_src) {   // dH_{l-1} = pad(dZ W_self) + dQ W_pool
    dim3 gg((unsigned)ceil_div(ns, GB_M), (unsigned)ceil_div(dp, GB_N));
    BF_CHECK((gemm2<float, float, float, false, false>(gg, s, ns, d_in, dp, d_out, d_in, a.dh, a.ld_dh, nullptr, n, dq, dp,
                                                   a.W, 2 * d_in, a.W_pool, d_in, nullptr, 0, a.dh_src,
                                                   a.ld_dh_src)));
  }
  return BUFFALO_OK;
}

buffalo_status pool_bwd_ffma(const PoolArgs& a, cudaStream_t s) {
  return a.in_bf16 ? pool_bwd_t<__nv_bfloat16>(a, s) : pool_bwd_t<float>(a, s);
}

// ================================================================== GraphSAGE-LSTM (R29)
// An LSTM (hidden size d = d_{l-1}, gate order i, f, u, o) over each dst row's sampled
// neighbours in CSR order.  The rows are walked in degree-class order (cls_perm, ascending D),
// so the rows still running at step t are a suffix [s_t, n) of the permutation (the packed-
// sequence layout): step t is one gate GEMM over c_t = n - s_t rows plus one cell kernel, and
// the per-step tensors are stored packed, step after step (off_t = sum of earlier c_t'), e rows
// in all.  Rows with D > kHeavyT are not supported here (sampled fanouts are <= 32).
__device__ __forceinline__ float sigm(float x) { return 1.f / (1.f + expf(-x)); }

// counts of rows per degree class min(D, kHeavyT + 1) and the maximum degree (cnt[kHeavyT + 2])
__global__ void __launch_bounds__(256) k_lstm_hist(const int32_t* __restrict__ rp, int64_t n, int32_t* __restrict__ cnt) {
  __shared__ int32_t sh[kHeavyT + 3];
  for (int i = threadIdx.x; i < kHeavyT + 3; i += blockDim.x) sh[i] = 0;
  __syncthreads();
  for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
    const int32_t D = rp[i + 1] - rp[i];
    atomicAdd(&sh[D > kHeavyT ? kHeavyT + 1 : D], 1);
    atomicMax(&sh[kHeavyT + 2], D);
  }
  __syncthreads();
  for (int i = threadIdx.x; i < kHeavyT + 2; i += blockDim.x)
    if (sh[i]) atomicAdd(&cnt[i], sh[i]);
  if (threadIdx.x == 0) atomicMax(&cnt[kHeavyT + 2], sh[kHeavyT + 2]);
}

// step t: source row (gix) of each running row's t-th neighbour, packed position of the edge
__global__ void k_lstm_gix(const int32_t* __restrict__ perm, const int32_t* __restrict__ rp,
                           const int32_t* __restrict__ colsrc, int64_t s_t, int64_t c_t, int t, int64_t off_t,
                           int32_t* __restrict__ gix, int32_t* __restrict__ ppos) {
  for (int64_t q = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; q < c_t; q += (int64_t)gridDim.x * blockDim.x) {
    const int64_t e = rp[perm[s_t + q]] + t;
    gix[off_t + q] = colsrc[e];
    ppos[e] = (int32_t)(off_t + q);
  }
}

// step t cell: gates (pre-activation, from the GEMM) -> i, f, u, o saved in place; c_t saved
// packed; running state (h, c) of row r = s_t + q updated.
__global__ void k_lstm_cell(float* __restrict__ G, int64_t ldg, float* __restrict__ Cs, float* __restrict__ Hs,
                            float* __restrict__ Cst, int64_t s_t, int64_t c_t, int t, int d, int64_t dp) {
  const int64_t total = c_t * d;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = x / d;
    const int k = (int)(x - q * d);
    const int64_t r = s_t + q;
    float* g = G + q * ldg;
    const float gi = sigm(g[k]), gf = sigm(g[d + k]), gu = tanhf(g[2 * d + k]), go = sigm(g[3 * d + k]);
    const float cp = t ? Cst[r * dp + k] : 0.f;
    const float c = gf * cp + gi * gu;
    g[k] = gi;
    g[d + k] = gf;
    g[2 * d + k] = gu;
    g[3 * d + k] = go;
    Cs[q * dp + k] = c;
    Cst[r * dp + k] = c;
    Hs[r * dp + k] = go * tanhf(c);
  }
}

// h_agg[perm[r]] = last hidden state (0 for D = 0), padding columns 0
__global__ void k_lstm_final(const int32_t* __restrict__ perm, const int32_t* __restrict__ rp,
                             const float* __restrict__ Hs, int64_t n, int d, int64_t dp, float* __restrict__ agg,
                             int64_t ld_agg) {
  const int64_t total = n * dp;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = x / dp;
    const int k = (int)(x - r * dp);
    const int32_t i = perm[r];
    agg[(int64_t)i * ld_agg + k] = (k < d && rp[i + 1] > rp[i]) ? Hs[r * dp + k] : 0.f;
  }
}

// backward state: dh = dh_agg of the row, dc = 0
__global__ void k_lstm_bwd_init(const int32_t* __restrict__ perm, const float* __restrict__ dagg, int64_t n,
                                int64_t dp, float* __restrict__ dhs, float* __restrict__ dcs) {
  const int64_t total = n * dp;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t r = x / dp;
    const int64_t k = x - r * dp;
    dhs[x] = dagg[(int64_t)perm[r] * dp + k];
    dcs[x] = 0.f;
  }
}

// step t of the backward: gate pre-activation gradients (written over the saved gates), h_{t-1}
// (recomputed from step t-1's o and c) for dW_hh, dc carried to t-1.
__global__ void k_lstm_cell_bwd(float* __restrict__ G, int64_t ldg, const float* __restrict__ Cs, int64_t dp,
                                int64_t off_t, int64_t s_t, int64_t c_t, int64_t off_p, int64_t s_p, int t, int d,
                                const float* __restrict__ dhs, float* __restrict__ dcs, float* __restrict__ Hprev) {
  const int64_t total = c_t * d;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t q = x / d;
    const int k = (int)(x - q * d);
    const int64_t r = s_t + q, p = off_t + q;
    float* g = G + p * ldg;
    const float gi = g[k], gf = g[d + k], gu = g[2 * d + k], go = g[3 * d + k];
    const float c = Cs[p * dp + k];
    float cp = 0.f, hp = 0.f;
    if (t) {
      const int64_t pp = off_p + (r - s_p);
      cp = Cs[pp * dp + k];
      hp = G[pp * ldg + 3 * d + k] * tanhf(cp);
    }
    Hprev[p * dp + k] = hp;
    const float dh = dhs[r * dp + k];
    const float tc = tanhf(c);
    const float dc = dcs[r * dp + k] + dh * go * (1.f - tc * tc);
    g[k] = dc * gu * gi * (1.f - gi);
    g[d + k] = dc * cp * gf * (1.f - gf);
    g[2 * d + k] = dc * gi * (1.f - gu * gu);
    g[3 * d + k] = dh * tc * go * (1.f - go);
    dcs[r * dp + k] = dc * gf;
  }
}

// dh_src[j] += sum over the dst i of src j (ascending i) of dx at the packed position of edge
// (i, j); warp per src row, the edge found by a ballot over row i.
__global__ void __launch_bounds__(256) k_lstm_scatterT(const int32_t* __restrict__ trp, const int32_t* __restrict__ tcol,
                                                       const int32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                       const int32_t* __restrict__ ppos, int64_t n_src,
                                                       const float* __restrict__ dx, int64_t dp, int d,
                                                       float* __restrict__ out, int64_t ldo) {
  const int lane = threadIdx.x & 31;
  const int nch = (int)(dp / 4);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_src; j += warps) {
    const int32_t t0 = trp[j], t1 = trp[j + 1];
    for (int c0 = 0; c0 < nch; c0 += 32) {
      const int c = c0 + lane;
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      for (int32_t t = t0; t < t1; ++t) {
        const int32_t i = tcol[t];
        int32_t e = -1;
        for (int32_t e0 = rp[i]; e0 < rp[i + 1] && e < 0; e0 += 32) {
          const bool hit = e0 + lane < rp[i + 1] && col[e0 + lane] == (int32_t)j;
          const unsigned m = __ballot_sync(0xffffffffu, hit);
          if (m) e = e0 + __ffs(m) - 1;
        }
        if (c < nch) {
          float v[4];
          VecIO<float, 4>::load(dx + (int64_t)ppos[e] * dp + c * 4, v);
#pragma unroll
          for (int k = 0; k < 4; ++k) acc[k] += v[k];
        }
      }
      if (c < nch) {
        float o[4];
        VecIO<float, 4>::load(out + j * ldo + c * 4, o);
#pragma unroll
        for (int k = 0; k < 4; ++k) o[k] = (c * 4 + k < d) ? o[k] + acc[k] : o[k];
        VecIO<float, 4>::store(out + j * ldo + c * 4, o);
      }
    }
  }
}

int lstm_dw_splits(int64_t n_rows, int d) {
  const int64_t tiles = ceil_div(4 * d, 64) * ceil_div(d, 64);
  const int64_t a = ceil_div(592, tiles), b = ceil_div(n_rows > 0 ? n_rows : 1, 512);
  const int64_t sp = a < b ? a : b;
  return (int)(sp < 1 ? 1 : sp);
}

int64_t lstm_saved_bytes(int64_t n, int64_t e, int d) {
  const int64_t dp = pitch_of(d), ldg = pitch_of(4 * d);
  return R(e * ldg * 4) + R(e * dp * 4) + 2 * R(e * 4) + 2 * R(n * dp * 4) + R(4 * 256);
}

struct LstmSaved {
  float *G, *Cs;
  int32_t *gix, *ppos;
  float *Hs, *Cst;
  int32_t* cnt;
};
static LstmSaved lstm_saved_view(void* base, int64_t n, int64_t e, int d) {
  const int64_t dp = pitch_of(d), ldg = pitch_of(4 * d);
  char* q = (char*)base;
  LstmSaved v;
  v.G = (float*)q; q += R(e * ldg * 4);
  v.Cs = (float*)q; q += R(e * dp * 4);
  v.gix = (int32_t*)q; q += R(e * 4);
  v.ppos = (int32_t*)q; q += R(e * 4);
  v.Hs = (float*)q; q += R(n * dp * 4);
  v.Cst = (float*)q; q += R(n * dp * 4);
  v.cnt = (int32_t*)q;
  return v;
}

int64_t lstm_bwd_scratch_bytes(int64_t n_dst, int64_t e, int layer, int d_in, int d_out) {
  const int S = dw_splits(n_dst, d_out, d_in), S3 = lstm_dw_splits(e, d_in);
  const int64_t dp = pitch_of(d_in);
  int64_t b = R((int64_t)S * d_out * 2 * d_in * 4) + R((int64_t)S * pitch_of(d_out) * 4);
  b += R(n_dst * dp * 4) + R(e * dp * 4);
  if (layer >= 2) b += R(e * dp * 4);
  b += R((int64_t)S3 * 4 * d_in * d_in * 4) + R((int64_t)S3 * pitch_of(4 * d_in) * 4);
  return b;
}

// Step table from the degree-class counts (one 520-byte read-back: the GEMM sizes are
// data dependent).  s[t] = first running row at step t, off[t] = packed offset, T = max D.
static buffalo_status lstm_steps(const buffalo_block* blk, int32_t* cnt_dev, std::vector<int64_t>& s,
                                 std::vector<int64_t>& off, int& T, cudaStream_t st) {
  const int64_t n = blk->n_dst;
  int32_t h[kHeavyT + 3] = {0};
  if (n > 0) {
    BF_CUDA(cudaMemcpyAsync(h, cnt_dev, sizeof(h), cudaMemcpyDeviceToHost, st));
    BF_CUDA(cudaStreamSynchronize(st));
  }
  if (h[kHeavyT + 1] > 0) {
    set_error("lstm: rows with more than %d neighbours are not supported (max degree %d)", kHeavyT, h[kHeavyT + 2]);
    return BUFFALO_ERR_UNSUPPORTED;
  }
  T = h[kHeavyT + 2];
  s.assign(T + 1, n);
  off.assign(T + 1, 0);
  int64_t run = n - h[0];            // rows with D > 0
  int64_t o = 0;
  for (int t = 0; t < T; ++t) {
    s[t] = n - run;
    off[t] = o;
    o += run;
    run -= h[t + 1];                 // rows with D = t + 1 stop after step t
  }
  off[T] = o;
  if (o != blk->n_edges) {
    set_error("lstm: packed steps %lld != edges %lld", (long long)o, (long long)blk->n_edges);
    return BUFFALO_ERR_INVALID_ARG;
  }
  return BUFFALO_OK;
}

template <class TI>
static buffalo_status lstm_fwd_t(const LstmArgs& a, cudaStream_t st) {
  const buffalo_block* blk = a.blk;
  const int64_t n = blk->n_dst, e = blk->n_edges;
  const int d = a.d_in;
  const int64_t dp = pitch_of(d), ldg = pitch_of(4 * d);
  LstmSaved v = lstm_saved_view(a.saved, n, e, d);
  BF_CUDA(cudaMemsetAsync(v.cnt, 0, 4 * (kHeavyT + 3), st));
  if (n > 0) {
    k_lstm_hist<<<grid_for(n, 256, 4), 256, 0, st>>>(blk->row_ptr, n, v.cnt);
    BF_LAUNCHED("k_lstm_hist");
  }
  std::vector<int64_t> s, off;
  int T = 0;
  BF_CHECK(lstm_steps(blk, v.cnt, s, off, T, st));
  const int32_t* colsrc = a.layer1 ? blk->col_global : blk->col_local;
  for (int t = 0; t < T; ++t) {
    const int64_t c_t = n - s[t];
    k_lstm_gix<<<grid_for(c_t, 256), 256, 0, st>>>(blk->cls_perm, blk->row_ptr, colsrc, s[t], c_t, t, off[t], v.gix,
                                                   v.ppos);
    BF_LAUNCHED("k_lstm_gix");
    dim3 grid((unsigned)ceil_div(c_t, GB_M), (unsigned)ceil_div(ldg, GB_N));
    const ProfSlot ps = prof_begin_launch("lstm_gates", st);
    BF_CHECK((gemm2<TI, float, float, true, false>(grid, st, c_t, 4 * d, (int)ldg, d, t ? d : 0, (const TI*)a.h_src,
                                                         a.ld_src, v.gix + off[t], c_t, v.Hs + s[t] * dp, dp,
                                                         a.W_ih, d, a.W_hh, d, a.b_lstm, 0, v.G + off[t] * ldg, ldg)));
    // "algorithmic bytes" of this family are FLOPs: 2 * rows * 4d * (d [x_t] + d [h_{t-1}, t > 0])
    prof_end_launch(ps, st, 2.0 * (double)c_t * 4.0 * d * (double)(t ? 2 * d : d), 0.0);
    k_lstm_cell<<<grid_for(c_t * d, 256), 256, 0, st>>>(v.G + off[t] * ldg, ldg, v.Cs + off[t] * dp, v.Hs, v.Cst,
                                                        s[t], c_t, t, d, dp);
    BF_LAUNCHED("k_lstm_cell");
  }
  if (n <= 0) return BUFFALO_OK;
  k_lstm_final<<<grid_for(n * dp, 256), 256, 0, st>>>(blk->cls_perm, blk->row_ptr, v.Hs, n, d, dp, a.agg, a.ld_agg);
  BF_LAUNCHED("k_lstm_final");
  const int Np = (int)pitch_of(a.d_out);
  dim3 grid((unsigned)ceil_div(n, GB_M), (unsigned)ceil_div(Np, GB_N));
  const float* Wt = a.W_packed;   // [2 d_in][d_out]
  BF_CHECK((gemm2<TI, float, float, false, false>(grid, st, n, a.d_out, Np, d, d, (const TI*)a.h_src, a.ld_src,
                                                 a.layer1 ? blk->src_global : nullptr, n, a.agg, a.ld_agg, Wt,
                                                 a.d_out, Wt + (int64_t)d * a.d_out, a.d_out, a.b, !a.last, a.out,
                                                 a.ld_out)));
  return BUFFALO_OK;
}

buffalo_status lstm_fwd_ffma(const LstmArgs& a, cudaStream_t s) {
  return a.in_bf16 ? lstm_fwd_t<__nv_bfloat16>(a, s) : lstm_fwd_t<float>(a, s);
}

template <class TI>
static buffalo_status lstm_bwd_t(const LstmArgs& a, cudaStream_t st) {
  const buffalo_block* blk = a.blk;
  const int64_t n = blk->n_dst, e = blk->n_edges, ns = blk->n_src;
  const int d = a.d_in, d_out = a.d_out;
  const int64_t dp = pitch_of(d), ldg = pitch_of(4 * d);
  const int32_t* gidx = a.layer1 ? blk->src_global : nullptr;
  LstmSaved v = lstm_saved_view(a.saved, n, e, d);
  if (!a.last && n > 0) {
    k_dz_mask<float><<<grid_for(n * d_out, 256), 256, 0, st>>>(a.dh, a.ld_dh, a.h_dst, a.ld_hdst, n, d_out);
    BF_LAUNCHED("k_dz_mask");
  }
  const int S = dw_splits(n, d_out, d), S3 = lstm_dw_splits(e, d);
  char* q = (char*)a.scratch;
  float* dw_part = (float*)q; q += R((int64_t)S * d_out * 2 * d * 4);
  float* db_part = (float*)q; q += R((int64_t)S * pitch_of(d_out) * 4);
  float* dagg = (float*)q; q += R(n * dp * 4);
  float* Hprev = (float*)q; q += R(e * dp * 4);
  float* dX = nullptr;
  if (a.dh_src) { dX = (float*)q; q += R(e * dp * 4); }
  float* dwl_part = (float*)q; q += R((int64_t)S3 * 4 * d * d * 4);
  float* dbl_part = (float*)q;
  if (n > 0) {
    dim3 g((unsigned)ceil_div(2 * d, DW_T), (unsigned)ceil_div(d_out, DW_T), (unsigned)S);
    BF_CHECK((dw_partial<TI, float>(g, st, n, d_out, d, 2 * d, a.dh, a.ld_dh, (const TI*)a.h_src, a.ld_src, gidx,
                                               a.agg, a.ld_agg, ceil_div(n, S), dw_part, db_part)));
    k_reduce_partials<<<grid_for((int64_t)d_out * 2 * d, 256), 256, 0, st>>>(dw_part, S, (int64_t)d_out * 2 * d, a.dW);
    BF_LAUNCHED("k_reduce_partials");
    k_reduce_partials<<<1, 256, 0, st>>>(db_part, S, d_out, a.db);
    BF_LAUNCHED("k_reduce_partials");
    dim3 gg((unsigned)ceil_div(n, GB_M), (unsigned)ceil_div(dp, GB_N));
    BF_CHECK((gemm2<float, float, float, false, false>(gg, st, n, d, (int)dp, d_out, 0, a.dh, a.ld_dh, nullptr, n, nullptr, 0,
                                                    a.W + d, 2 * d, nullptr, 0, nullptr, 0, dagg, dp)));
    k_lstm_bwd_init<<<grid_for(n * dp, 256), 256, 0, st>>>(blk->cls_perm, dagg, n, dp, v.Hs, v.Cst);
    BF_LAUNCHED("k_lstm_bwd_init");
  }
  std::vector<int64_t> s, off;
  int T = 0;
  BF_CHECK(lstm_steps(blk, v.cnt, s, off, T, st));
  for (int t = T - 1; t >= 0; --t) {
    const int64_t c_t = n - s[t];
    k_lstm_cell_bwd<<<grid_for(c_t * d, 256), 256, 0, st>>>(v.G, ldg, v.Cs, dp, off[t], s[t], c_t, t ? off[t - 1] : 0,
                                                            t ? s[t - 1] : 0, t, d, v.Hs, v.Cst, Hprev);
    BF_LAUNCHED("k_lstm_cell_bwd");
    if (t > 0) {   // dh_{t-1} = dG_t W_hh into the running rows' state
      dim3 gg((unsigned)ceil_div(c_t, GB_M), (unsigned)ceil_div(dp, GB_N));
      BF_CHECK((gemm2<float, float, float, false, false>(gg, st, c_t, d, (int)dp, 4 * d, 0, v.G + off[t] * ldg, ldg, nullptr, c_t,
                                                      nullptr, 0, a.W_hh, d, nullptr, 0, nullptr, 0, v.Hs + s[t] * dp,
                                                      dp)));
    }
  }
  if (e > 0) {
    // dW_ih (+ db_lstm) = dG^T X over the packed rows, then dW_hh = dG^T H_prev
    dim3 g3((unsigned)ceil_div(d, DW_T), (unsigned)ceil_div(4 * d, DW_T), (unsigned)S3);
    BF_CHECK((dw_partial<TI, float>(g3, st, e, 4 * d, d, d, v.G, ldg, (const TI*)a.h_src, a.ld_src, v.gix, nullptr,
                                                0, ceil_div(e, S3), dwl_part, dbl_part)));
    k_reduce_partials<<<grid_for((int64_t)4 * d * d, 256), 256, 0, st>>>(dwl_part, S3, (int64_t)4 * d * d, a.dW_ih);
    BF_LAUNCHED("k_reduce_partials");
    k_reduce_partials<<<grid_for(4 * d, 256), 256, 0, st>>>(dbl_part, S3, 4 * d, a.db_lstm);
    BF_LAUNCHED("k_reduce_partials");
    BF_CHECK((dw_partial<float, float>(g3, st, e, 4 * d, d, d, v.G, ldg, Hprev, dp, nullptr, nullptr, 0,
                                                   ceil_div(e, S3), dwl_part, dbl_part)));
    k_reduce_partials<<<grid_for((int64_t)4 * d * d, 256), 256, 0, st>>>(dwl_part, S3, (int64_t)4 * d * d, a.dW_hh);
    BF_LAUNCHED("k_reduce_partials");
  }
  if (a.dh_src && ns > 0) {   // dH_{l-1} = pad(dZ W_self) + sum over edges of dG W_ih
    dim3 gg((unsigned)ceil_div(ns, GB_M), (unsigned)ceil_div(dp, GB_N));
    BF_CHECK((gemm2<float, float, float, false, false>(gg, st, ns, d, (int)dp, d_out, 0, a.dh, a.ld_dh, nullptr, n, nullptr, 0,
                                                    a.W, 2 * d, nullptr, 0, nullptr, 0, a.dh_src, a.ld_dh_src)));
    if (e > 0) {
      dim3 gx((unsigned)ceil_div(e, GB_M), (unsigned)ceil_div(dp, GB_N));
      BF_CHECK((gemm2<float, float, float, false, false>(gx, st, e, d, (int)dp, 4 * d, 0, v.G, ldg, nullptr, e, nullptr, 0,
                                                      a.W_ih, d, nullptr, 0, nullptr, 0, dX, dp)));
      k_lstm_scatterT<<<grid_for(ns * 32, 256, 16), 256, 0, st>>>(blk->t_row_ptr, blk->t_col, blk->row_ptr,
                                                                  blk->col_local, v.ppos, ns, dX, dp, d, a.dh_src,
                                                                  a.ld_dh_src);
      BF_LAUNCHED("k_lstm_scatterT");
    }
  }
  return BUFFALO_OK;
}

buffalo_status lstm_bwd_ffma(const LstmArgs& a, cudaStream_t s) {
  return a.in_bf16 ? lstm_bwd_t<__nv_bfloat16>(a, s) : lstm_bwd_t<float>(a, s);
}

// ================================================================== GAT (R30)
// One attention head per layer.  Z = H W^T over the block's src rows (SIMT GEMM), scores
// el[j] = a_l . Z[j], er[i] = a_r . Z[i]; per dst row (degree-class order) a warp takes the
// max and the sum of exp over its edges in a fixed lane/shuffle order, stores alpha per edge,
// then sums alpha Z[col] over the edges in CSR order (lanes over 4-column chunks).
__device__ __forceinline__ float leaky(float x) { return x > 0.f ? x : 0.2f * x; }

__device__ __forceinline__ float warp_dot(const float* __restrict__ a, const float* __restrict__ z, int d) {
  float s = 0.f;
  for (int k = threadIdx.x & 31; k < d; k += 32) s = fmaf(a[k], z[k], s);
#pragma unroll
  for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
  return s;
}

__global__ void __launch_bounds__(256) k_gat_scores(const float* __restrict__ Z, int64_t ldz, int64_t n_src,
                                                    int64_t n_dst, int d, const float* __restrict__ al,
                                                    const float* __restrict__ ar, float* __restrict__ el,
                                                    float* __restrict__ er) {
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_src; j += warps) {
    const float l = warp_dot(al, Z + j * ldz, d);
    const float r = j < n_dst ? warp_dot(ar, Z + j * ldz, d) : 0.f;
    if ((threadIdx.x & 31) == 0) {
      el[j] = l;
      if (j < n_dst) er[j] = r;
    }
  }
}

__global__ void __launch_bounds__(256) k_gat_attn(const int32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                  const int32_t* __restrict__ perm, int64_t n,
                                                  const float* __restrict__ Z, int64_t ldz, int d,
                                                  const float* __restrict__ el, const float* __restrict__ er,
                                                  const float* __restrict__ b, int elu, float* __restrict__ alpha,
                                                  float* __restrict__ out, int64_t ldo) {
  const int lane = threadIdx.x & 31;
  const int nch = (int)(pitch_of(d) / 4);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t w = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; w < n; w += warps) {
    const int64_t i = perm[w];
    const int32_t e0 = rp[i], e1 = rp[i + 1];
    const float eri = er[i];
    float m = -INFINITY;
    for (int32_t e = e0 + lane; e < e1; e += 32) m = fmaxf(m, leaky(el[col[e]] + eri));
#pragma unroll
    for (int o = 16; o; o >>= 1) m = fmaxf(m, __shfl_xor_sync(0xffffffffu, m, o));
    float sum = 0.f;
    for (int32_t e = e0 + lane; e < e1; e += 32) sum += expf(leaky(el[col[e]] + eri) - m);
#pragma unroll
    for (int o = 16; o; o >>= 1) sum += __shfl_xor_sync(0xffffffffu, sum, o);
    const float inv = 1.f / sum;
    for (int32_t e = e0 + lane; e < e1; e += 32) alpha[e] = expf(leaky(el[col[e]] + eri) - m) * inv;
    __syncwarp();
    for (int c = lane; c < nch; c += 32) {
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      for (int32_t e = e0; e < e1; ++e) {
        const float a = alpha[e];
        float v[4];
        VecIO<float, 4>::load(Z + (int64_t)col[e] * ldz + c * 4, v);
#pragma unroll
        for (int k = 0; k < 4; ++k) acc[k] = fmaf(a, v[k], acc[k]);
      }
#pragma unroll
      for (int k = 0; k < 4; ++k) {
        const int kk = c * 4 + k;
        float x = kk < d ? acc[k] + b[kk] : 0.f;
        if (elu && x <= 0.f) x = expm1f(x);
        acc[k] = x;
      }
      VecIO<float, 4>::store(out + i * ldo + c * 4, acc);
    }
  }
}

// dOut = dH * ELU'(out), ELU'(out) = 1 (H > 0) or H + 1 (H = expm1(out) <= 0)
__global__ void k_gat_elu_bwd(float* __restrict__ dh, int64_t ldd, const float* __restrict__ h, int64_t ldh,
                              int64_t n, int d) {
  const int64_t total = n * d;
  for (int64_t x = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; x < total; x += (int64_t)gridDim.x * blockDim.x) {
    const int64_t i = x / d;
    const int k = (int)(x - i * d);
    const float hv = h[i * ldh + k];
    if (!(hv > 0.f)) dh[i * ldd + k] *= hv + 1.f;
  }
}

// column sums of dOut, split-K: CTA (32 columns, row split z of rps rows), 8 warps over the
// rows, fixed-order combine into part[z][c]; k_reduce_partials then adds the splits in order

// per dst row: dalpha_e = dOut_i . Z[col_e] (kept in ds), then ds_e = alpha_e (dalpha_e - sum
// alpha dalpha) LeakyReLU'(s_e), d_er[i] = sum_e ds_e
__global__ void __launch_bounds__(256) k_gat_row_bwd(const int32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                     int64_t n, const float* __restrict__ Z, int64_t ldz, int d,
                                                     const float* __restrict__ dO, int64_t ldo,
                                                     const float* __restrict__ el, const float* __restrict__ er,
                                                     const float* __restrict__ alpha, float* __restrict__ ds,
                                                     float* __restrict__ d_er) {
  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n; i += warps) {
    const int32_t e0 = rp[i], e1 = rp[i + 1];
    float c = 0.f;
    for (int32_t e = e0; e < e1; ++e) {
      const float da = warp_dot(dO + i * ldo, Z + (int64_t)col[e] * ldz, d);
      if (lane == 0) ds[e] = da;
      c = fmaf(alpha[e], da, c);
    }
    __syncwarp();
    const float eri = er[i];
    float s = 0.f;
    for (int32_t e = e0 + lane; e < e1; e += 32) {
      const float x = el[col[e]] + eri;
      const float g = alpha[e] * (ds[e] - c) * (x > 0.f ? 1.f : 0.2f);
      ds[e] = g;
      s += g;
    }
#pragma unroll
    for (int o = 16; o; o >>= 1) s += __shfl_xor_sync(0xffffffffu, s, o);
    if (lane == 0) d_er[i] = s;
  }
}

// per src row j (transposed block, ascending dst i): dZ[j] = sum alpha_e dOut_i + d_el[j] a_l
// (+ d_er[j] a_r for j < n_dst), d_el[j] = sum ds_e; edge e = (i, j) found by a ballot.
__global__ void __launch_bounds__(256) k_gat_src_bwd(const int32_t* __restrict__ trp, const int32_t* __restrict__ tcol,
                                                     const int32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                     int64_t n_src, int64_t n_dst, const float* __restrict__ alpha,
                                                     const float* __restrict__ ds, const float* __restrict__ dO,
                                                     int64_t ldo, int d, const float* __restrict__ al,
                                                     const float* __restrict__ ar, const float* __restrict__ d_er,
                                                     float* __restrict__ d_el, float* __restrict__ dZ, int64_t ldz) {
  const int lane = threadIdx.x & 31;
  const int nch = (int)(pitch_of(d) / 4);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_src; j += warps) {
    const int32_t t0 = trp[j], t1 = trp[j + 1];
    float del = 0.f;
    for (int c0 = 0; c0 < nch; c0 += 32) {
      const int c = c0 + lane;
      float acc[4] = {0.f, 0.f, 0.f, 0.f};
      float dsum = 0.f;
      for (int32_t t = t0; t < t1; ++t) {
        const int32_t i = tcol[t];
        int32_t e = -1;
        for (int32_t e0 = rp[i]; e0 < rp[i + 1] && e < 0; e0 += 32) {
          const bool hit = e0 + lane < rp[i + 1] && col[e0 + lane] == (int32_t)j;
          const unsigned m = __ballot_sync(0xffffffffu, hit);
          if (m) e = e0 + __ffs(m) - 1;
        }
        const float a = alpha[e];
        dsum += ds[e];
        if (c < nch) {
          float v[4];
          VecIO<float, 4>::load(dO + (int64_t)i * ldo + c * 4, v);
#pragma unroll
          for (int k = 0; k < 4; ++k) acc[k] = fmaf(a, v[k], acc[k]);
        }
      }
      del = dsum;
      if (c < nch) {
        const float der = j < n_dst ? d_er[j] : 0.f;
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int kk = c * 4 + k;
          acc[k] = kk < d ? acc[k] + del * al[kk] + der * ar[kk] : 0.f;
        }
        VecIO<float, 4>::store(dZ + j * ldz + c * 4, acc);
      }
    }
    if (lane == 0) d_el[j] = del;
  }
}

// k_gat_src_bwd for pitch(d) <= 128 G floats: each lane holds G 4-float chunks of the row, so the
// edge search of an entry runs once (not once per 32-chunk pass) and the entry's dOut row loads
// are issued before it; the per-element sum order (t ascending, fmaf) is that of k_gat_src_bwd.
template <int G>
__global__ void __launch_bounds__(256) k_gat_src_bwd_g(const int32_t* __restrict__ trp, const int32_t* __restrict__ tcol,
                                                       const int32_t* __restrict__ rp, const int32_t* __restrict__ col,
                                                       int64_t n_src, int64_t n_dst, const float* __restrict__ alpha,
                                                       const float* __restrict__ ds, const float* __restrict__ dO,
                                                       int64_t ldo, int d, const float* __restrict__ al,
                                                       const float* __restrict__ ar, const float* __restrict__ d_er,
                                                       float* __restrict__ d_el, float* __restrict__ dZ, int64_t ldz) {
  const int lane = threadIdx.x & 31;
  const int nch = (int)(pitch_of(d) / 4);
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t j = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; j < n_src; j += warps) {
    const int32_t t0 = trp[j], t1 = trp[j + 1];
    float acc[G][4];
#pragma unroll
    for (int g = 0; g < G; ++g)
#pragma unroll
      for (int k = 0; k < 4; ++k) acc[g][k] = 0.f;
    float dsum = 0.f;
    for (int32_t t = t0; t < t1; ++t) {
      const int32_t i = tcol[t];
      float v[G][4];
#pragma unroll
      for (int g = 0; g < G; ++g) {
        const int c = g * 32 + lane;
        if (c < nch) VecIO<float, 4>::load(dO + (int64_t)i * ldo + c * 4, v[g]);
      }
      const int32_t eb = rp[i], ee = rp[i + 1];
      int32_t e = -1;
      for (int32_t e0 = eb; e0 < ee && e < 0; e0 += 32) {
        const bool hit = e0 + lane < ee && col[e0 + lane] == (int32_t)j;
        const unsigned m = __ballot_sync(0xffffffffu, hit);
        if (m) e = e0 + __ffs(m) - 1;
      }
      const float a = alpha[e];
      dsum += ds[e];
#pragma unroll
      for (int g = 0; g < G; ++g)
        if (g * 32 + lane < nch) {
#pragma unroll
          for (int k = 0; k < 4; ++k) acc[g][k] = fmaf(a, v[g][k], acc[g][k]);
        }
    }
    const float der = j < n_dst ? d_er[j] : 0.f;
#pragma unroll
    for (int g = 0; g < G; ++g) {
      const int c = g * 32 + lane;
      if (c < nch) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int kk = c * 4 + k;
          acc[g][k] = kk < d ? acc[g][k] + dsum * al[kk] + der * ar[kk] : 0.f;
        }
        VecIO<float, 4>::store(dZ + j * ldz + c * 4, acc[g]);
      }
    }
    if (lane == 0) d_el[j] = dsum;
  }
}

int gemm_splits(int64_t n_rows, int rows_out, int K) {
  const int64_t tiles = ceil_div(rows_out, 64) * ceil_div(K, 64);
  const int64_t a = ceil_div(592, tiles), b = ceil_div(n_rows > 0 ? n_rows : 1, 512);
  const int64_t sp = a < b ? a : b;
  return (int)(sp < 1 ? 1 : sp);
}

int64_t gat_saved_bytes(int64_t n_src, int64_t n_dst, int64_t e, int d_out) {
  return R(n_src * pitch_of(d_out) * 4) + R(4 * n_src) + R(4 * n_dst) + R(4 * e);
}

int64_t gat_bwd_scratch_bytes(int64_t n_src, int64_t n_dst, int64_t e, int d_in, int d_out) {
  const int S4 = gemm_splits(n_src, d_out, d_in), Sl = gemm_splits(n_src, 1, d_out), Sr = gemm_splits(n_dst, 1, d_out);
  return R(n_src * pitch_of(d_out) * 4) + R(4 * e) + R(4 * n_src) + R(4 * n_dst) +
         R((int64_t)S4 * d_out * d_in * 4) + R((int64_t)S4 * pitch_of(d_out) * 4) +
         R((int64_t)Sl * d_out * 4) + R((int64_t)Sl * 4) + R((int64_t)Sr * d_out * 4) + R((int64_t)Sr * 4);
}

struct GatSaved {
  float *Z, *el, *er, *alpha;
};
static GatSaved gat_saved_view(void* base, int64_t n_src, int64_t n_dst, int64_t e, int d_out) {
  char* q = (char*)base;
  GatSaved v;
  v.Z = (float*)q; q += R(n_src * pitch_of(d_out) * 4);
  v.el = (float*)q; q += R(4 * n_src);
  v.er = (float*)q; q += R(4 * n_dst);
  v.alpha = (float*)q;
  return v;
}

template <class TI>
static buffalo_status gat_fwd_t(const GatArgs& a, cudaStream_t st) {
  const buffalo_block* blk = a.blk;
  const int64_t ns = blk->n_src, nd = blk->n_dst, e = blk->n_edges;
  const int dl = a.d_out;
  const int64_t ldz = pitch_of(dl);
  GatSaved v = gat_saved_view(a.saved, ns, nd, e, dl);
  if (ns > 0) {
    dim3 grid((unsigned)ceil_div(ns, GB_M), (unsigned)ceil_div(ldz, GB_N));
    BF_CHECK((gemm2<TI, float, float, true, false>(grid, st, ns, dl, (int)ldz, a.d_in, 0, (const TI*)a.h_src, a.ld_src,
                                                         a.layer1 ? blk->src_global : nullptr, ns, nullptr, 0, a.W,
                                                         a.d_in, nullptr, 0, nullptr, 0, v.Z, ldz)));
    k_gat_scores<<<grid_for(ns * 32, 256, 16), 256, 0, st>>>(v.Z, ldz, ns, nd, dl, a.a_l, a.a_r, v.el, v.er);
    BF_LAUNCHED("k_gat_scores");
  }
  if (nd <= 0) return BUFFALO_OK;
  const ProfSlot ps = prof_begin_launch("gat_attn", st);
  k_gat_attn<<<grid_for(nd * 32, 256, 16), 256, 0, st>>>(blk->row_ptr, blk->col_local, blk->cls_perm, nd, v.Z, ldz, dl,
                                                         v.el, v.er, a.b, !a.last, v.alpha, a.out, a.ld_out);
  BF_LAUNCHED("k_gat_attn");
  // algorithmic bytes (each datum once; the three passes re-read indices and scores from L1/L2):
  // per row perm + row_ptr pair + er + the output row; per edge the index, el, the alpha
  // written and the Z row
  prof_end_launch(ps, st, (double)nd * (16.0 + 4.0 * ldz) + (double)e * (12.0 + 4.0 * ldz), 0.0);
  return BUFFALO_OK;
}

buffalo_status gat_fwd_ffma(const GatArgs& a, cudaStream_t s) {
  return a.in_bf16 ? gat_fwd_t<__nv_bfloat16>(a, s) : gat_fwd_t<float>(a, s);
}

template <class TI>
static buffalo_status gat_bwd_t(const GatArgs& a, cudaStream_t st) {
  const buffalo_block* blk = a.blk;
  const int64_t ns = blk->n_src, nd = blk->n_dst, e = blk->n_edges;
  const int dl = a.d_out, d_in = a.d_in;
  const int64_t ldz = pitch_of(dl);
  GatSaved v = gat_saved_view(a.saved, ns, nd, e, dl);
  const int S4 = gemm_splits(ns, dl, d_in), Sl = gemm_splits(ns, 1, dl), Sr = gemm_splits(nd, 1, dl);
  char* q = (char*)a.scratch;
  float* dZ = (float*)q; q += R(ns * ldz * 4);
  float* ds = (float*)q; q += R(4 * e);
  float* d_el = (float*)q; q += R(4 * ns);
  float* d_er = (float*)q; q += R(4 * nd);
  float* dw_part = (float*)q; q += R((int64_t)S4 * dl * d_in * 4);
  float* db_part = (float*)q; q += R((int64_t)S4 * pitch_of(dl) * 4);
  float* dal_part = (float*)q; q += R((int64_t)Sl * dl * 4);
  float* dal_b = (float*)q; q += R((int64_t)Sl * 4);
  float* dar_part = (float*)q; q += R((int64_t)Sr * dl * 4);
  float* dar_b = (float*)q;
  if (!a.last && nd > 0) {
    k_gat_elu_bwd<<<grid_for(nd * dl, 256), 256, 0, st>>>(a.dh, a.ld_dh, a.h_dst, a.ld_hdst, nd, dl);
    BF_LAUNCHED("k_gat_elu_bwd");
  }
  if (nd > 0) {
    // db: the da_r partial buffer (Sr x dl floats) holds the column-sum splits first
    k_colsum_partial<<<dim3((unsigned)ceil_div(dl, 32), (unsigned)Sr), 256, 0, st>>>(a.dh, a.ld_dh, nd, dl,
                                                                                     ceil_div(nd, Sr), dar_part);
    BF_LAUNCHED("k_colsum_partial");
    k_reduce_partials<<<1, 256, 0, st>>>(dar_part, Sr, dl, a.db);
    BF_LAUNCHED("k_reduce_partials");
    k_gat_row_bwd<<<grid_for(nd * 32, 256, 16), 256, 0, st>>>(blk->row_ptr, blk->col_local, nd, v.Z, ldz, dl, a.dh,
                                                              a.ld_dh, v.el, v.er, v.alpha, ds, d_er);
    BF_LAUNCHED("k_gat_row_bwd");
  }
  if (ns <= 0) return BUFFALO_OK;
  if (ldz <= 128) {
    k_gat_src_bwd_g<1><<<grid_for(ns * 32, 256, 16), 256, 0, st>>>(
        blk->t_row_ptr, blk->t_col, blk->row_ptr, blk->col_local, ns, nd, v.alpha, ds, a.dh, a.ld_dh, dl, a.a_l, a.a_r,
        d_er, d_el, dZ, ldz);
  } else if (ldz <= 256) {
    k_gat_src_bwd_g<2><<<grid_for(ns * 32, 256, 16), 256, 0, st>>>(
        blk->t_row_ptr, blk->t_col, blk->row_ptr, blk->col_local, ns, nd, v.alpha, ds, a.dh, a.ld_dh, dl, a.a_l, a.a_r,
        d_er, d_el, dZ, ldz);
  } else {
    k_gat_src_bwd<<<grid_for(ns * 32, 256, 16), 256, 0, st>>>(blk->t_row_ptr, blk->t_col, blk->row_ptr,
                                                              blk->col_local, ns, nd, v.alpha, ds, a.dh, a.ld_dh, dl,
                                                              a.a_l, a.a_r, d_er, d_el, dZ, ldz);
  }
  BF_LAUNCHED("k_gat_src_bwd");
  // da_l = d_el^T Z, da_r = d_er^T Z[:n_dst], dW = dZ^T H (deterministic split reductions)
  // (weighted column sums of Z over fixed row splits: one coalesced pass per vector; the dal_b /
  // dar_b slots of the scratch layout, R30, held the 1-row products' bias partials and stay
  // unused)
  (void)dal_b;
  (void)dar_b;
  k_colsum_partial<<<dim3((unsigned)ceil_div(dl, 32), (unsigned)Sl), 256, 0, st>>>(v.Z, ldz, ns, dl, ceil_div(ns, Sl),
                                                                                   dal_part, d_el);
  BF_LAUNCHED("k_colsum_partial");
  k_reduce_partials<<<1, 256, 0, st>>>(dal_part, Sl, dl, a.da_l);
  BF_LAUNCHED("k_reduce_partials");
  if (nd > 0) {
    k_colsum_partial<<<dim3((unsigned)ceil_div(dl, 32), (unsigned)Sr), 256, 0, st>>>(v.Z, ldz, nd, dl,
                                                                                     ceil_div(nd, Sr), dar_part, d_er);
    BF_LAUNCHED("k_colsum_partial");
    k_reduce_partials<<<1, 256, 0, st>>>(dar_part, Sr, dl, a.da_r);
    BF_LAUNCHED("k_reduce_partials");
  }
  dim3 gw((unsigned)ceil_div(d_in, DW_T), (unsigned)ceil_div(dl, DW_T), (unsigned)S4);
  BF_CHECK((dw_partial<TI, float>(gw, st, ns, dl, d_in, d_in, dZ, ldz, (const TI*)a.h_src, a.ld_src,
                                              a.layer1 ? blk->src_global : nullptr, nullptr, 0, ceil_div(ns, S4),
                                              dw_part, db_part)));
  k_reduce_partials<<<grid_for((int64_t)dl * d_in, 256), 256, 0, st>>>(dw_part, S4, (int64_t)dl * d_in, a.dW);
  BF_LAUNCHED("k_reduce_partials");
  if (a.dh_src) {   // dH_{l-1} = dZ W
    const int64_t dpi = pitch_of(d_in);
    dim3 gg((unsigned)ceil_div(ns, GB_M), (unsigned)ceil_div(dpi, GB_N));
    BF_CHECK((gemm2<float, float, float, false, false>(gg, st, ns, d_in, (int)dpi, dl, 0, dZ, ldz, nullptr, ns, nullptr, 0, a.W,
                                                    d_in, nullptr, 0, nullptr, 0, a.dh_src, a.ld_dh_src)));
  }
  return BUFFALO_OK;
}

buffalo_status gat_bwd_ffma(const GatArgs& a, cudaStream_t s) {
  return a.in_bf16 ? gat_bwd_t<__nv_bfloat16>(a, s) : gat_bwd_t<float>(a, s);
}

}  // namespace buffalo
