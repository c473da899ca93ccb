// tc_f32.cu — the fp32 dW reductions of the FFMA-mode paths on the 5th-gen tensor cores (sm_100a).
//
// dW partials part[s][m][col] = sum over a row split of Z[r][m] F(r, col) (the k_dw_partial
// contract, sage.cu) — the long reductions that dominate the pool / LSTM / GAT epochs on CUDA
// cores.  tcgen05.mma kind::tf32 multiplies 19-bit TF32 operands exactly and accumulates in
// fp32 (TMEM); every fp32 operand is split into NS = 3 TF32 terms x = x_0 + x_1 + x_2 (each the
// round-to-nearest TF32 value of the remainder: x is represented exactly) and the product is
// the sum of the 6 term products with i + j < 3 (only products below 2^-33 relative dropped).
// The tensor core's own accumulation is not IEEE-rounded, so each 32-row chunk goes into a
// fresh TMEM buffer (24 accumulation steps) which the staging warps add into fp32 registers
// (round-to-nearest, a fixed chunk order): fp32-level accuracy over millions of rows.
//
// One CTA computes one 128 (m) x 128 (col) tile over a row split: 16 staging warps (8 per
// operand) load each 32-row chunk (each thread a 4 x 4 block: four 16-B row-contiguous loads),
// transpose it in registers, split it and store the three terms as 16-B rows of K-major
// SWIZZLE_128B tiles (lane mapping chosen so a warp's stores cover all 32 banks); two stages,
// the next chunk's loads in flight while the tensor cores work; one elected lane issues the
// tcgen05.mma products of the chunk; two TMEM buffers alternate.
#include "tc_f32.cuh"

namespace buffalo {
namespace {

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c));
}
__device__ __forceinline__ void mb_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mb_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE_%=;\n\t"
      "bra WAIT_%=;\n\t"
      "DONE_%=:\n\t}" ::"r"(su32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// K-major SWIZZLE_128B descriptor: rows of 128 B, 8-row atoms of 1024 B (SBO), sm_100 version bit.
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void mma_tf32(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::tf32 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(bar))
               : "memory");
}
__device__ __forceinline__ void tmem_ld32(uint32_t taddr, float* v) {
  uint32_t r[32];
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 32; ++i) v[i] = __uint_as_float(r[i]);
}
__device__ __forceinline__ float tf32_rna(float x) {
  uint32_t r;
  asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(r) : "f"(x));
  return __uint_as_float(r);
}

constexpr int kTM = 128;                   // tile rows = TMEM lanes
constexpr int kKC = 32;                    // K per chunk: one 128-B swizzle row of fp32
constexpr int kTileA = kTM * 128;          // 16 KB per term

// Byte offset of (row, k) (k < 32) in a K-major SWIZZLE_128B tile.
__device__ __forceinline__ int swz(int row, int k) { return row * 128 + ((((k >> 2) ^ (row & 7))) << 4) + ((k & 3) << 2); }

template <int NS>
__device__ __forceinline__ void split_store4(uint8_t* tiles, int tile_bytes, int row, int k, float4 v) {
  float x[4] = {v.x, v.y, v.z, v.w};
  float t[NS][4];
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    float r = x[e];
#pragma unroll
    for (int s = 0; s < NS; ++s) {
      t[s][e] = tf32_rna(r);
      r -= t[s][e];
    }
  }
#pragma unroll
  for (int s = 0; s < NS; ++s)
    *reinterpret_cast<float4*>(tiles + s * tile_bytes + swz(row, k)) = make_float4(t[s][0], t[s][1], t[s][2], t[s][3]);
}

template <class T>
__device__ __forceinline__ float4 ld4(const T* p);
template <> __device__ __forceinline__ float4 ld4<float>(const float* p) { return __ldg(reinterpret_cast<const float4*>(p)); }
template <> __device__ __forceinline__ float4 ld4<__nv_bfloat16>(const __nv_bfloat16* p) {
  const uint2 u = __ldg(reinterpret_cast<const uint2*>(p));
  return make_float4(__uint_as_float(u.x << 16), __uint_as_float(u.x & 0xffff0000u), __uint_as_float(u.y << 16),
                     __uint_as_float(u.y & 0xffff0000u));
}
__device__ __forceinline__ float4 mask4(float4 v, int col, int lim) {
  if (col + 0 >= lim) v.x = 0.f;
  if (col + 1 >= lim) v.y = 0.f;
  if (col + 2 >= lim) v.z = 0.f;
  if (col + 3 >= lim) v.w = 0.f;
  return v;
}

// Shared-memory plan: two stages of NS A-term tiles (128 x 32 fp32) and NS B-term tiles
// (NT x 32 fp32), then the mbarriers and the TMEM address slot.
template <int NS, int NT>
struct Pipe {
  static constexpr int kTileB = NT * 128;
  static constexpr int kStage = NS * (kTileA + kTileB);
  static constexpr int kSmem = 2 * kStage + 128 + 1024;
};

}  // namespace

// ===================================================================== dW partials (split-K over rows)
// part[s][m][col] = sum_{r in split s} Z[r][m] * F(r, col), m < d_out, col < Kd where F(r, col) =
// col < d_in ? self[row(r)][col] : agg[r][col - d_in] (agg null: Kd = d_in).  F's columns are
// laid out in the tile as [self | pad | agg | pad] halves of Dp = round_up(d_in, 4), so no float4
// straddles the two sources; the epilogue maps them back to the dense [d_out][Kd] partial.
// Staging warps 0-7 stage Z (the A operand), warps 8-15 stage F (B).  Thread t of a group: row
// quad rq = t & 7 (rows 4 rq .. 4 rq + 3 of the chunk), column quad cq = t >> 3 (columns 4 cq ..
// 4 cq + 3 of the 128-wide tile); after the 4 x 4 transpose it stores, for each of its 4
// columns, the 16-B piece k = 4 rq .. 4 rq + 3 of that K-major row: a warp's eight lanes of one
// row cover all 32 banks.  All 16 warps drain the TMEM buffers (warp w: lane quadrant w & 3,
// columns 32 (w >> 2) ..) and keep 32 fp32 accumulators per thread.
constexpr int kStageWarps = 16;
constexpr int kDwThreads = (kStageWarps + 1) * 32;

template <class TS, class TG, int NS>
__global__ void __launch_bounds__(kDwThreads, 1) k_tcf_dw(const TcfDw p) {
  constexpr int NT = 128;
  using PP = Pipe<NS, NT>;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = (uint64_t*)(smem + 2 * PP::kStage);
  uint64_t* empty = full + 2;
  uint64_t* tfull = empty + 2;                         // chunk accumulator ready (per TMEM buffer)
  uint64_t* tempty = tfull + 2;                        // chunk accumulator drained
  uint32_t* tslot = (uint32_t*)(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  const int m0 = blockIdx.x * kTM;                     // output rows (d_out)
  const int j0 = blockIdx.y * NT;                      // padded F columns
  const int64_t r_beg = (int64_t)blockIdx.z * p.rows_per_split;
  const int64_t r_end = min(p.n, r_beg + p.rows_per_split);
  const int nch = r_end > r_beg ? (int)((r_end - r_beg + kKC - 1) / kKC) : 0;
  if (tid == 0) {
    for (int i = 0; i < 2; ++i) {
      mb_init(&full[i], kStageWarps * 32);
      mb_init(&empty[i], 1);
      mb_init(&tfull[i], 1);
      mb_init(&tempty[i], kStageWarps * 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kStageWarps) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(tslot)), "r"(2 * NT));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tslot;

  if (warp == kStageWarps) {
    if (lane == 0) {
      constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NT >> 3) << 17) |
                                 ((uint32_t)(kTM >> 4) << 24);
      for (int c = 0; c < nch; ++c) {
        const int st = c & 1;
        if (c >= 2) mb_wait(&tempty[st], (uint32_t)(((c >> 1) - 1) & 1));
        mb_wait(&full[st], (uint32_t)((c >> 1) & 1));
        fence_after();
        const uint32_t a0 = su32(smem + st * PP::kStage), b0 = a0 + NS * kTileA;
        const uint32_t d = tmem + st * NT;
#pragma unroll
        for (int kk = 0; kk < kKC / 8; ++kk)
#pragma unroll
          for (int i = 0; i < NS; ++i)
#pragma unroll
            for (int j = 0; j < NS - i; ++j)
              mma_tf32(d, desc_sw128(a0 + i * kTileA + kk * 32), desc_sw128(b0 + j * PP::kTileB + kk * 32), idesc,
                       (kk > 0 || i > 0 || j > 0) ? 1u : 0u);
        commit(&empty[st]);
        commit(&tfull[st]);
      }
    }
    __syncwarp();
  } else {
    const bool isA = warp < 8;
    const int t = tid & 255;
    const int rq = t & 7, cq = t >> 3;                 // 8 row quads x 32 column quads
    const int Dp = p.Dp;
    const int q = warp & 3, h = warp >> 2;             // drain: lane quadrant, 32-column quarter
    float acc[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) acc[k] = 0.f;
    float4 rv[4];                                      // [row of the quad], 4 columns each
    const int acol = m0 + 4 * cq;                      // A: output rows m (columns of Z)
    const int jc = j0 + 4 * cq;                        // B: padded F column
    const int bsrc = jc < Dp ? (jc < p.d_in ? 1 : 0) : ((p.agg && jc - Dp < p.d_in) ? 2 : 0);
    auto load = [&](int c) {
      const int64_t rb0 = r_beg + (int64_t)c * kKC + 4 * rq;
#pragma unroll
      for (int e = 0; e < 4; ++e) {
        const int64_t r = rb0 + e;
        float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
        if (r < r_end) {
          if (isA) {
            if (acol < p.d_out) v = mask4(ld4<float>(p.Z + r * p.ldz + acol), acol, p.d_out);
          } else if (bsrc == 1) {
            const int64_t sr = p.gidx ? (int64_t)__ldg(p.gidx + r) : r;
            v = mask4(ld4<TS>((const TS*)p.self + sr * p.lds + jc), jc, p.d_in);
          } else if (bsrc == 2) {
            v = mask4(ld4<TG>((const TG*)p.agg + r * p.lda + (jc - Dp)), jc - Dp, p.d_in);
          }
        }
        rv[e] = v;
      }
    };
    // the 4 x 4 block transposed: K-major row (4 cq + x) gets k = 4 rq .. 4 rq + 3
    auto store_t = [&](uint8_t* tiles, int tile_bytes) {
      const float col[4][4] = {{rv[0].x, rv[1].x, rv[2].x, rv[3].x}, {rv[0].y, rv[1].y, rv[2].y, rv[3].y},
                               {rv[0].z, rv[1].z, rv[2].z, rv[3].z}, {rv[0].w, rv[1].w, rv[2].w, rv[3].w}};
#pragma unroll
      for (int x = 0; x < 4; ++x)
        split_store4<NS>(tiles, tile_bytes, 4 * cq + x, 4 * rq, make_float4(col[x][0], col[x][1], col[x][2], col[x][3]));
    };
    auto drain = [&](int c) {                          // add chunk c's TMEM buffer into acc
      const int st = c & 1;
      mb_wait(&tfull[st], (uint32_t)((c >> 1) & 1));
      fence_after();
      float v[32];
      tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + st * NT + h * 32, v);
#pragma unroll
      for (int k = 0; k < 32; ++k) acc[k] += v[k];
      fence_before();
      mb_arrive(&tempty[st]);
    };
    if (nch > 0) load(0);
    for (int c = 0; c < nch; ++c) {
      const int st = c & 1;
      if (c >= 2) mb_wait(&empty[st], (uint32_t)(((c >> 1) - 1) & 1));
      uint8_t* sa = smem + st * PP::kStage;
      if (isA) store_t(sa, kTileA);
      else store_t(sa + NS * kTileA, PP::kTileB);
      fence_async_smem();
      mb_arrive(&full[st]);
      if (c + 1 < nch) load(c + 1);
      if (c >= 1) drain(c - 1);
    }
    if (nch > 0) drain(nch - 1);
    const int m = m0 + q * 32 + lane;
    const int Kd = p.agg ? 2 * p.d_in : p.d_in;
    float* P = p.part + (int64_t)blockIdx.z * p.d_out * Kd;
    if (m < p.d_out) {
#pragma unroll
      for (int k = 0; k < 32; ++k) {
        const int j = j0 + h * 32 + k;
        const int col = j < Dp ? (j < p.d_in ? j : -1) : (j - Dp < p.d_in ? p.d_in + (j - Dp) : -1);
        if (col >= 0 && col < Kd) P[(int64_t)m * Kd + col] = acc[k];
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == kStageWarps) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(2 * NT));
  }
}

// ===================================================================== host launcher
buffalo_status tcf_dw(TcfDw p, int S, bool self_bf16, cudaStream_t s) {
  if (p.n <= 0) return BUFFALO_OK;
  constexpr int NS = 3, NT = 128;
  p.Dp = (int)round_up(p.d_in, 4);
  p.rows_per_split = round_up(ceil_div(p.n, S), kKC);
  const int width = p.agg ? 2 * p.Dp : p.Dp;
  dim3 grid((unsigned)ceil_div(p.d_out, kTM), (unsigned)ceil_div(width, NT), (unsigned)S);
  if (self_bf16) {
    BF_CHECK((set_max_smem_once<k_tcf_dw<__nv_bfloat16, float, NS>>(Pipe<NS, NT>::kSmem)));
    k_tcf_dw<__nv_bfloat16, float, NS><<<grid, kDwThreads, Pipe<NS, NT>::kSmem, s>>>(p);
  } else {
    BF_CHECK((set_max_smem_once<k_tcf_dw<float, float, NS>>(Pipe<NS, NT>::kSmem)));
    k_tcf_dw<float, float, NS><<<grid, kDwThreads, Pipe<NS, NT>::kSmem, s>>>(p);
  }
  BF_LAUNCHED("k_tcf_dw");
  return BUFFALO_OK;
}

}  // namespace buffalo
