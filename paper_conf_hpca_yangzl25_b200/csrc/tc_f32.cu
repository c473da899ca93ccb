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
#include <cuda.h>

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

__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
}
__device__ __forceinline__ void tma_2d(void* dst, const CUtensorMap* map, int c0, int c1, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3}], [%4];" ::
          "r"(su32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(c1), "r"(su32(bar))
      : "memory");
}
__device__ __forceinline__ void tma_gather4(void* dst, const CUtensorMap* map, int c0, int r0, int r1, int r2, int r3,
                                            uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.tensor.2d.shared::cluster.global.tile::gather4.mbarrier::complete_tx::bytes [%0], [%1, {%2, %3, "
      "%4, %5, %6}], [%7];" ::"r"(su32(dst)),
      "l"(reinterpret_cast<uint64_t>(map)), "r"(c0), "r"(r0), "r"(r1), "r"(r2), "r"(r3), "r"(su32(bar))
      : "memory");
}
// MN-major descriptor for 32-bit operands: the only MN-major layout tcgen05 takes for tf32 is
// SWIZZLE_128B_BASE32B (layout type 1; TMA CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B): 128-B rows
// along M/N (32 fp32), 32-B granules swizzled over 4-row atoms along K (SBO 512 B), LBO = byte
// distance between consecutive 32-element M/N strips.
__device__ __forceinline__ uint64_t desc_mn(uint32_t saddr, uint32_t lbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)(512 >> 4) << 32) | ((uint64_t)1 << 46) | ((uint64_t)1 << 61);
}
// In-place split of 4 fp32 values at byte offset off of term tile 0 into NS TF32 terms (term s
// at tiles + s * tile_bytes + off): t_0 = rna(x), t_s = rna(x - t_0 - ... - t_{s-1}).
template <int NS>
__device__ __forceinline__ void split_inplace4(uint8_t* tiles, int tile_bytes, int off) {
  const float4 v = *reinterpret_cast<const float4*>(tiles + off);
  float x[4] = {v.x, v.y, v.z, v.w};
  float t[NS][4];
#pragma unroll
  for (int e = 0; e < 4; ++e) {
    float r = x[e];
#pragma unroll
    for (int k = 0; k < NS; ++k) {
      t[k][e] = k + 1 < NS ? tf32_rna(r) : r;    // the last term keeps the exact remainder
      r -= t[k][e];
    }
  }
#pragma unroll
  for (int k = 0; k < NS; ++k)
    *reinterpret_cast<float4*>(tiles + k * tile_bytes + off) = make_float4(t[k][0], t[k][1], t[k][2], t[k][3]);
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

// ===================================================================== dW partials, TMA-fed
// The same partials as k_tcf_dw for fp32 operands, loaded by TMA as they lie in memory: Z^T (A,
// M = d_out) and F (B, N = columns) are both MN-major over K = rows, so a 32-row chunk of a
// 128-wide tile is four {32 col, 32 row} SWIZZLE_128B_ATOM_32B boxes (gathered self rows: 32
// gather4).
// The raw fp32 chunk lands in term tile 0; the 16 worker warps split it in place into the NS = 3
// TF32 terms (linear 16-B accesses, conflict-free), then drain the previous chunk's TMEM buffer
// into their fp32 registers as in k_tcf_dw.  Warp 16 issues the TMA, warp 17 the MMAs.
constexpr int kDwWorkWarps = 16;
constexpr int kDwTmaWarp = kDwWorkWarps, kDwMmaWarp = kDwWorkWarps + 1;
constexpr int kDwTmaThreads = (kDwWorkWarps + 2) * 32;
constexpr int kDwStrip = kKC * 128;                   // one {32 col, 32 row} box: 4 KB
constexpr int kDwTile = 4 * kDwStrip;                 // 128 columns: 16 KB per term

struct TcfDwTmaP {
  int64_t n, rows_per_split;
  int d_out, d_in, tiles_self, Kd;
  const int32_t* gidx;
  float* part;
};

template <bool GATHER>
__global__ void __launch_bounds__(kDwTmaThreads, 1)
    k_tcf_dw_tma(const __grid_constant__ CUtensorMap z_map, const __grid_constant__ CUtensorMap self_map,
                 const __grid_constant__ CUtensorMap agg_map, const TcfDwTmaP p) {
  constexpr int NS = 3;
  constexpr int kOp = NS * kDwTile, kStage = 2 * kOp;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = (uint64_t*)(smem + 2 * kStage);
  uint64_t* split = full + 2;
  uint64_t* empty = split + 2;
  uint64_t* tfull = empty + 2;
  uint64_t* tempty = tfull + 2;
  uint32_t* tslot = (uint32_t*)(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  const int m0 = blockIdx.x * kTM;
  const int y = blockIdx.y;
  const bool self_tile = y < p.tiles_self;
  const int c0 = (self_tile ? y : y - p.tiles_self) * 128;   // first column of the tile in its source
  const int64_t r_beg = (int64_t)blockIdx.z * p.rows_per_split;
  const int64_t r_end = min(p.n, r_beg + p.rows_per_split);
  const int nch = r_end > r_beg ? (int)((r_end - r_beg + kKC - 1) / kKC) : 0;
  if (tid == 0) {
    for (int i = 0; i < 2; ++i) {
      mb_init(&full[i], 1);
      mb_init(&split[i], kDwWorkWarps * 32);
      mb_init(&empty[i], 1);
      mb_init(&tfull[i], 1);
      mb_init(&tempty[i], kDwWorkWarps * 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kDwMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(tslot)), "r"(256));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tslot;

  if (warp == kDwTmaWarp) {
    for (int c = 0; c < nch; ++c) {
      const int st = c & 1;
      const int r0 = (int)(r_beg + (int64_t)c * kKC);
      if (lane == 0) {
        if (c >= 2) mb_wait(&empty[st], (uint32_t)(((c >> 1) - 1) & 1));
        mb_expect(&full[st], 2 * kDwTile);
      }
      __syncwarp();
      uint8_t* sa = smem + st * kStage;
      uint8_t* sb = sa + kOp;
      if (lane == 0) {
#pragma unroll
        for (int j = 0; j < 4; ++j) tma_2d(sa + j * kDwStrip, &z_map, m0 + 32 * j, r0, &full[st]);
      }
      if (self_tile && GATHER) {
        // strip j = lane / 8, rows 4 (lane % 8) .. + 3 of the chunk
        int32_t rr[4];
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int64_t r = (int64_t)r0 + (lane & 7) * 4 + k;
          rr[k] = r < p.n ? __ldg(p.gidx + r) : 0;          // rows >= n: Z is zero there
        }
        tma_gather4(sb + (lane >> 3) * kDwStrip + (lane & 7) * 4 * 128, &self_map, c0 + 32 * (lane >> 3), rr[0], rr[1],
                    rr[2], rr[3], &full[st]);
      } else if (lane == 0) {
        const CUtensorMap* map = self_tile ? &self_map : &agg_map;
#pragma unroll
        for (int j = 0; j < 4; ++j) tma_2d(sb + j * kDwStrip, map, c0 + 32 * j, r0, &full[st]);
      }
      __syncwarp();
    }
  } else if (warp == kDwMmaWarp) {
    if (lane == 0) {
      constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (1u << 15) | (1u << 16) |
                                 ((uint32_t)(128 >> 3) << 17) | ((uint32_t)(kTM >> 4) << 24);
      for (int c = 0; c < nch; ++c) {
        const int st = c & 1;
        if (c >= 2) mb_wait(&tempty[st], (uint32_t)(((c >> 1) - 1) & 1));
        mb_wait(&split[st], (uint32_t)((c >> 1) & 1));
        fence_after();
        const uint32_t a0 = su32(smem + st * kStage), b0 = a0 + kOp;
        const uint32_t d = tmem + st * 128;
#pragma unroll
        for (int kk = 0; kk < kKC / 8; ++kk)
#pragma unroll
          for (int i = 0; i < NS; ++i)
#pragma unroll
            for (int j = 0; j < NS - i; ++j)
              mma_tf32(d, desc_mn(a0 + i * kDwTile + kk * 1024, kDwStrip), desc_mn(b0 + j * kDwTile + kk * 1024, kDwStrip),
                       idesc, (kk > 0 || i > 0 || j > 0) ? 1u : 0u);
        commit(&empty[st]);
        commit(&tfull[st]);
      }
    }
    __syncwarp();
  } else {
    const int q = warp & 3, h = warp >> 2;             // drain: lane quadrant, 32-column quarter
    float acc[32];
#pragma unroll
    for (int k = 0; k < 32; ++k) acc[k] = 0.f;
    auto drain = [&](int c) {
      const int st = c & 1;
      mb_wait(&tfull[st], (uint32_t)((c >> 1) & 1));
      fence_after();
      float v[32];
      tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + st * 128 + h * 32, v);
#pragma unroll
      for (int k = 0; k < 32; ++k) acc[k] += v[k];
      fence_before();
      mb_arrive(&tempty[st]);
    };
    for (int c = 0; c < nch; ++c) {
      const int st = c & 1;
      mb_wait(&full[st], (uint32_t)((c >> 1) & 1));
      uint8_t* sa = smem + st * kStage;
#pragma unroll
      for (int i = 0; i < 4; ++i) {
        const int idx = tid + kDwWorkWarps * 32 * i;   // 0 .. 2047: 16-B pieces of both raw tiles
        split_inplace4<NS>(sa + (idx >> 10) * kOp, kDwTile, (idx & 1023) * 16);
      }
      fence_async_smem();
      mb_arrive(&split[st]);
      if (c >= 1) drain(c - 1);
    }
    if (nch > 0) drain(nch - 1);
    const int m = m0 + q * 32 + lane;
    float* P = p.part + (int64_t)blockIdx.z * p.d_out * p.Kd;
    if (m < p.d_out) {
      const int cb = c0 + h * 32;
      const int col0 = self_tile ? cb : p.d_in + cb;
#pragma unroll
      for (int k = 0; k < 32; ++k)
        if (cb + k < p.d_in) P[(int64_t)m * p.Kd + col0 + k] = acc[k];
    }
  }
  fence_before();
  __syncthreads();
  if (warp == kDwMmaWarp) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(256));
  }
}

// ===================================================================== GEMM (the k_gemm2_tc contract)
// C[r][n] = act(sum_k A1[row1(r)][k] B1(k, n) + sum_k A2[r][k] B2(k, n) + bias[n]) for n < N, 0 for
// N <= n < Np; row1(r) = gidx ? gidx[r] : r for r < m1 (no A1 term beyond); B(k, n) = B[k][n], or
// Bt[n][k] when TB.  K = K1 + K2 <= 2 d is short, so the product accumulates in TMEM across all
// chunks (the error of the tensor pipe's accumulation is that of the mma.sync path it replaces),
// with NS = 2 terms (hi hi + hi lo + lo hi, the 3xTF32 scheme of the mma.sync kernel it replaces),
// or NS = 3 (six products, every fp32 operand represented exactly) when the caller asks for the
// FFMA path's fp32 accuracy.  Callers keep K <= kTcfMaxK (tc_f32.cuh).
// Persistent, warp-specialised: 16 staging warps (0-7: A rows, K-major as stored; 8-15: B, 4 x 4
// transposed when stored [k][n]) fill a 3-stage ring of 128 x 32 chunks; warp 16 (one lane)
// issues the MMAs into one of two 128-column TMEM accumulators; warps 17-20 drain the other
// (thread = output row) with bias / ReLU and write C while the next tile is computed.
constexpr int kGemmEpiWarps = 4;
constexpr int kGemmThreads = (kStageWarps + 1 + kGemmEpiWarps) * 32;

template <class TA1, bool TB, int NS>
__global__ void __launch_bounds__(kGemmThreads, 1) k_tcf_gemm(const TcfGemm p) {
  constexpr int NT = 128, NST = NS == 2 ? 3 : 2;
  constexpr int kTB = NT * 128, kStage = NS * (kTileA + kTB);
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = (uint64_t*)(smem + NST * kStage);
  uint64_t* empty = full + NST;
  uint64_t* tfull = empty + NST;
  uint64_t* tempty = tfull + 2;
  uint32_t* tslot = (uint32_t*)(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  const int tiles_n = (p.Np + NT - 1) / NT;
  const int64_t ntiles = (int64_t)((p.M + kTM - 1) / kTM) * tiles_n;
  const int nk1 = (p.K1 + kKC - 1) / kKC, nk2 = (p.K2 + kKC - 1) / kKC, nk = nk1 + nk2;
  if (tid == 0) {
    for (int i = 0; i < NST; ++i) {
      mb_init(&full[i], kStageWarps * 32);
      mb_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mb_init(&tfull[i], 1);
      mb_init(&tempty[i], kGemmEpiWarps * 32);
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
    if (lane == 0 && nk > 0) {
      constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | ((uint32_t)(NT >> 3) << 17) |
                                 ((uint32_t)(kTM >> 4) << 24);
      int64_t g = 0;
      int it = 0;
      for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++it) {
        const int ab = it & 1;
        if (it >= 2) mb_wait(&tempty[ab], (uint32_t)(((it >> 1) - 1) & 1));
        fence_after();
        const uint32_t d = tmem + ab * NT;
        for (int c = 0; c < nk; ++c, ++g) {
          const int st = (int)(g % NST);
          mb_wait(&full[st], (uint32_t)((g / NST) & 1));
          fence_after();
          const uint32_t a0 = su32(smem + st * kStage), b0 = a0 + NS * kTileA;
#pragma unroll
          for (int kk = 0; kk < kKC / 8; ++kk)
#pragma unroll
            for (int i = 0; i < NS; ++i)
#pragma unroll
              for (int j = 0; j < NS - i; ++j)
                mma_tf32(d, desc_sw128(a0 + i * kTileA + kk * 32), desc_sw128(b0 + j * kTB + kk * 32), idesc,
                         (c > 0 || kk > 0 || i > 0 || j > 0) ? 1u : 0u);
          commit(&empty[st]);
        }
        commit(&tfull[ab]);
      }
    }
    __syncwarp();
  } else if (warp < kStageWarps) {
    if (nk > 0) {
      const bool isA = warp < 8;
      const int t = tid & 255;
      const int kq = t & 7, sub = t >> 3;              // k quad; row (A, TB) or column quad (plain B)
      float4 rv[4];
      auto load = [&](int64_t tile, int c) {
        const int64_t m0 = (tile / tiles_n) * kTM;
        const int n0 = (int)(tile % tiles_n) * NT;
        const bool first = c < nk1;
        const int k = (first ? c : c - nk1) * kKC + 4 * kq;
        const int K = first ? p.K1 : p.K2;
        if (isA) {
#pragma unroll
          for (int e = 0; e < 4; ++e) {
            const int64_t r = m0 + sub + 32 * e;
            float4 v = make_float4(0.f, 0.f, 0.f, 0.f);
            if (k < K && r < p.M) {
              if (first) {
                if (r < p.m1) {
                  const int64_t sr = p.gidx ? (int64_t)__ldg(p.gidx + r) : r;
                  v = mask4(ld4<TA1>((const TA1*)p.A1 + sr * p.lda1 + k), k, K);
                }
              } else {
                v = mask4(ld4<float>(p.A2 + r * p.lda2 + k), k, K);
              }
            }
            rv[e] = v;
          }
        } else {
          const float* B = first ? p.B1 : p.B2;
          const int64_t ldb = first ? p.ldb1 : p.ldb2;
          if (TB) {
#pragma unroll
            for (int e = 0; e < 4; ++e) {
              const int n = n0 + sub + 32 * e;
              rv[e] = (k < K && n < p.N) ? mask4(ld4<float>(B + (int64_t)n * ldb + k), k, K)
                                         : make_float4(0.f, 0.f, 0.f, 0.f);
            }
          } else {
            const int n = n0 + 4 * sub;
#pragma unroll
            for (int e = 0; e < 4; ++e)
              rv[e] = (k + e < K && n < p.N) ? mask4(ld4<float>(B + (int64_t)(k + e) * ldb + n), n, p.N)
                                             : make_float4(0.f, 0.f, 0.f, 0.f);
          }
        }
      };
      auto store = [&](int st) {
        uint8_t* sa = smem + st * kStage;
        if (isA || TB) {
          uint8_t* base = isA ? sa : sa + NS * kTileA;
          const int tb = isA ? kTileA : kTB;
#pragma unroll
          for (int e = 0; e < 4; ++e) split_store4<NS>(base, tb, sub + 32 * e, 4 * kq, rv[e]);
        } else {
          const float col[4][4] = {{rv[0].x, rv[1].x, rv[2].x, rv[3].x}, {rv[0].y, rv[1].y, rv[2].y, rv[3].y},
                                   {rv[0].z, rv[1].z, rv[2].z, rv[3].z}, {rv[0].w, rv[1].w, rv[2].w, rv[3].w}};
#pragma unroll
          for (int x = 0; x < 4; ++x)
            split_store4<NS>(sa + NS * kTileA, kTB, 4 * sub + x, 4 * kq,
                             make_float4(col[x][0], col[x][1], col[x][2], col[x][3]));
        }
      };
      int64_t tile = blockIdx.x;
      int c = 0;
      if (tile < ntiles) load(tile, 0);
      for (int64_t g = 0; tile < ntiles; ++g) {
        const int st = (int)(g % NST);
        if (g >= NST) mb_wait(&empty[st], (uint32_t)(((g / NST) - 1) & 1));
        store(st);
        fence_async_smem();
        mb_arrive(&full[st]);
        if (++c == nk) {
          c = 0;
          tile += gridDim.x;
        }
        if (tile < ntiles) load(tile, c);
      }
    }
  } else {
    const int q = warp & 3;                            // TMEM lane quadrant of this warp
    const bool vec = (p.ldc & 3) == 0 && (((uintptr_t)p.C) & 15) == 0;
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++it) {
      const int ab = it & 1;
      const int64_t row = (tile / tiles_n) * kTM + q * 32 + lane;
      const int n0 = (int)(tile % tiles_n) * NT;
      if (nk > 0) {
        mb_wait(&tfull[ab], (uint32_t)((it >> 1) & 1));
        fence_after();
      }
#pragma unroll 1
      for (int h = 0; h < 4; ++h) {
        float v[32];
        if (nk > 0) {
          tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + ab * NT + h * 32, v);
        } else {
#pragma unroll
          for (int k = 0; k < 32; ++k) v[k] = 0.f;
        }
        const int nb = n0 + h * 32;
        if (row < p.M && nb < p.Np) {
          float* out = p.C + row * p.ldc + nb;
#pragma unroll
          for (int k = 0; k < 32; ++k) {
            const int nn = nb + k;
            float x = 0.f;
            if (nn < p.N) {
              x = v[k] + (p.bias ? __ldg(p.bias + nn) : 0.f);
              if (p.relu) x = fmaxf(x, 0.f);
            }
            v[k] = x;
          }
          if (vec && nb + 32 <= p.Np) {
#pragma unroll
            for (int k = 0; k < 32; k += 4) *reinterpret_cast<float4*>(out + k) = make_float4(v[k], v[k + 1], v[k + 2], v[k + 3]);
          } else {
#pragma unroll
            for (int k = 0; k < 32; ++k)
              if (nb + k < p.Np) out[k] = v[k];
          }
        }
      }
      if (nk > 0) {
        fence_before();
        mb_arrive(&tempty[ab]);
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

// ===================================================================== GEMM, TMA-fed (fp32 A)
// The k_tcf_gemm contract for fp32 A1, every operand loaded by TMA as it lies in memory: A rows
// K-major ({32 k, 128 row} SWIZZLE_128B box, or 32 gather4 of 4 rows for gathered A1 rows), B
// K-major when stored [n][k] (TB) or MN-major when stored [k][n] (four {32 n, 32 k}
// SWIZZLE_128B_ATOM_32B boxes).  The raw fp32 chunk lands in term tile 0; 8 worker warps split it
// in place into the NS TF32 terms (zeroing A1 rows >= m1 of a gathered A1), warp 8 issues the TMA,
// warp 9 the MMAs, warps 10-13 drain the two TMEM accumulators (bias / ReLU, C rows per thread).
constexpr int kGtWork = 8;
constexpr int kGtTma = kGtWork, kGtMma = kGtWork + 1, kGtEpi0 = kGtWork + 2;
constexpr int kGtThreads = (kGtWork + 2 + 4) * 32;

struct TcfGemmTmaP {
  int64_t M, m1;
  int N, Np, K1, K2;
  const int32_t* gidx;
  const float* bias;
  int relu;
  float* C;
  int64_t ldc;
};

template <bool TB, int NS, bool GATHER>
__global__ void __launch_bounds__(kGtThreads, 1)
    k_tcf_gemm_tma(const __grid_constant__ CUtensorMap a1_map, const __grid_constant__ CUtensorMap a2_map,
                   const __grid_constant__ CUtensorMap b1_map, const __grid_constant__ CUtensorMap b2_map,
                   const TcfGemmTmaP p) {
  constexpr int NT = 128, NST = NS == 2 ? 3 : 2;
  constexpr int kTile = kTM * 128;                      // 16 KB: 128 rows (or n) x 32 fp32
  constexpr int kOp = NS * kTile, kStage = 2 * kOp;
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  uint64_t* full = (uint64_t*)(smem + NST * kStage);
  uint64_t* split = full + NST;
  uint64_t* empty = split + NST;
  uint64_t* tfull = empty + NST;
  uint64_t* tempty = tfull + 2;
  uint32_t* tslot = (uint32_t*)(tempty + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, tid = threadIdx.x;
  const int tiles_n = (p.Np + NT - 1) / NT;
  const int64_t ntiles = (int64_t)((p.M + kTM - 1) / kTM) * tiles_n;
  const int nk1 = (p.K1 + kKC - 1) / kKC, nk2 = (p.K2 + kKC - 1) / kKC, nk = nk1 + nk2;
  if (tid == 0) {
    for (int i = 0; i < NST; ++i) {
      mb_init(&full[i], 1);
      mb_init(&split[i], kGtWork * 32);
      mb_init(&empty[i], 1);
    }
    for (int i = 0; i < 2; ++i) {
      mb_init(&tfull[i], 1);
      mb_init(&tempty[i], 4 * 32);
    }
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kGtMma) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(tslot)), "r"(2 * NT));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tslot;

  if (warp == kGtTma) {
    if (nk > 0) {
      int64_t g = 0;
      for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int64_t m0 = (tile / tiles_n) * kTM;
        const int n0 = (int)(tile % tiles_n) * NT;
        for (int c = 0; c < nk; ++c, ++g) {
          const int st = (int)(g % NST);
          const bool first = c < nk1;
          const int k0 = (first ? c : c - nk1) * kKC;
          if (lane == 0) {
            if (g >= NST) mb_wait(&empty[st], (uint32_t)(((g / NST) - 1) & 1));
            mb_expect(&full[st], 2 * kTile);
          }
          __syncwarp();
          uint8_t* sa = smem + st * kStage;
          uint8_t* sb = sa + kOp;
          if (first && GATHER) {
            int32_t rr[4];
#pragma unroll
            for (int k = 0; k < 4; ++k) {
              const int64_t r = m0 + lane * 4 + k;
              rr[k] = r < p.m1 ? __ldg(p.gidx + r) : 0;   // rows >= m1 are zeroed by the split
            }
            tma_gather4(sa + lane * 512, &a1_map, k0, rr[0], rr[1], rr[2], rr[3], &full[st]);
          } else if (lane == 0) {
            tma_2d(sa, first ? &a1_map : &a2_map, k0, (int)m0, &full[st]);
          }
          if (lane == 0) {
            const CUtensorMap* bm = first ? &b1_map : &b2_map;
            if (TB) {
              tma_2d(sb, bm, k0, n0, &full[st]);
            } else {
#pragma unroll
              for (int j = 0; j < 4; ++j) tma_2d(sb + j * kDwStrip, bm, n0 + 32 * j, k0, &full[st]);
            }
          }
          __syncwarp();
        }
      }
    }
  } else if (warp == kGtMma) {
    if (lane == 0 && nk > 0) {
      constexpr uint32_t idesc = (1u << 4) | (2u << 7) | (2u << 10) | (TB ? 0u : (1u << 16)) |
                                 ((uint32_t)(NT >> 3) << 17) | ((uint32_t)(kTM >> 4) << 24);
      int64_t g = 0;
      int it = 0;
      for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++it) {
        const int ab = it & 1;
        if (it >= 2) mb_wait(&tempty[ab], (uint32_t)(((it >> 1) - 1) & 1));
        fence_after();
        const uint32_t d = tmem + ab * NT;
        for (int c = 0; c < nk; ++c, ++g) {
          const int st = (int)(g % NST);
          mb_wait(&split[st], (uint32_t)((g / NST) & 1));
          fence_after();
          const uint32_t a0 = su32(smem + st * kStage), b0 = a0 + kOp;
#pragma unroll
          for (int kk = 0; kk < kKC / 8; ++kk)
#pragma unroll
            for (int i = 0; i < NS; ++i)
#pragma unroll
              for (int j = 0; j < NS - i; ++j) {
                const uint64_t bd = TB ? desc_sw128(b0 + j * kTile + kk * 32) : desc_mn(b0 + j * kTile + kk * 1024, kDwStrip);
                mma_tf32(d, desc_sw128(a0 + i * kTile + kk * 32), bd, idesc, (c > 0 || kk > 0 || i > 0 || j > 0) ? 1u : 0u);
              }
          commit(&empty[st]);
        }
        commit(&tfull[ab]);
      }
    }
    __syncwarp();
  } else if (warp < kGtWork) {
    if (nk > 0) {
      int64_t g = 0;
      for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x) {
        const int64_t m0 = (tile / tiles_n) * kTM;
        for (int c = 0; c < nk; ++c, ++g) {
          const int st = (int)(g % NST);
          mb_wait(&full[st], (uint32_t)((g / NST) & 1));
          uint8_t* sa = smem + st * kStage;
          const bool mask = GATHER && c < nk1 && m0 + kTM > p.m1;
#pragma unroll
          for (int i = 0; i < 8; ++i) {
            const int idx = tid + kGtWork * 32 * i;      // 0 .. 2047: 16-B pieces of both raw tiles
            const int op = idx >> 10, off = (idx & 1023) * 16;
            if (op == 0 && mask && m0 + (off >> 7) >= p.m1) {
#pragma unroll
              for (int k = 0; k < NS; ++k) *reinterpret_cast<float4*>(sa + k * kTile + off) = make_float4(0.f, 0.f, 0.f, 0.f);
            } else {
              split_inplace4<NS>(sa + op * kOp, kTile, off);
            }
          }
          fence_async_smem();
          mb_arrive(&split[st]);
        }
      }
    }
  } else {
    const int q = warp & 3;                            // TMEM lane quadrant of this warp
    const bool vec = (p.ldc & 3) == 0 && (((uintptr_t)p.C) & 15) == 0;
    int it = 0;
    for (int64_t tile = blockIdx.x; tile < ntiles; tile += gridDim.x, ++it) {
      const int ab = it & 1;
      const int64_t row = (tile / tiles_n) * kTM + q * 32 + lane;
      const int n0 = (int)(tile % tiles_n) * NT;
      if (nk > 0) {
        mb_wait(&tfull[ab], (uint32_t)((it >> 1) & 1));
        fence_after();
      }
#pragma unroll 1
      for (int h = 0; h < 4; ++h) {
        float v[32];
        if (nk > 0) {
          tmem_ld32(tmem + ((uint32_t)(q * 32) << 16) + ab * NT + h * 32, v);
        } else {
#pragma unroll
          for (int k = 0; k < 32; ++k) v[k] = 0.f;
        }
        const int nb = n0 + h * 32;
        if (row < p.M && nb < p.Np) {
          float* out = p.C + row * p.ldc + nb;
#pragma unroll
          for (int k = 0; k < 32; ++k) {
            const int nn = nb + k;
            float x = 0.f;
            if (nn < p.N) {
              x = v[k] + (p.bias ? __ldg(p.bias + nn) : 0.f);
              if (p.relu) x = fmaxf(x, 0.f);
            }
            v[k] = x;
          }
          if (vec && nb + 32 <= p.Np) {
#pragma unroll
            for (int k = 0; k < 32; k += 4) *reinterpret_cast<float4*>(out + k) = make_float4(v[k], v[k + 1], v[k + 2], v[k + 3]);
          } else {
#pragma unroll
            for (int k = 0; k < 32; ++k)
              if (nb + k < p.Np) out[k] = v[k];
          }
        }
      }
      if (nk > 0) {
        fence_before();
        mb_arrive(&tempty[ab]);
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == kGtMma) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(2 * NT));
  }
}

// ===================================================================== host launcher
typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

// fp32 2D tensor map over [rows][ld] (first cols columns), {32 col, box_rows} boxes, zero fill out
// of bounds; swz: SWIZZLE_128B (K-major operands) or SWIZZLE_128B_ATOM_32B (MN-major).
static buffalo_status encode_f32(CUtensorMap* map, const float* base, int64_t cols, int64_t rows, int64_t ld,
                                 int box_rows, CUtensorMapSwizzle swz) {
  static EncodeTiledFn fn = [] {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    if (cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q) != cudaSuccess ||
        q != cudaDriverEntryPointSuccess)
      f = nullptr;
    return (EncodeTiledFn)f;
  }();
  if (!fn) {
    set_error("cuTensorMapEncodeTiled unavailable");
    return BUFFALO_ERR_CUDA;
  }
  const cuuint64_t dims[2] = {(cuuint64_t)(cols > 0 ? cols : 1), (cuuint64_t)(rows > 0 ? rows : 1)};
  const cuuint64_t strides[1] = {(cuuint64_t)ld * 4};
  const cuuint32_t box[2] = {32, (cuuint32_t)box_rows};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_FLOAT32, 2, const_cast<float*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled (fp32) failed (%d)", (int)r);
    return BUFFALO_ERR_CUDA;
  }
  return BUFFALO_OK;
}

buffalo_status tcf_dw_tma(const TcfDw& q, int S, cudaStream_t s) {
  if (q.n <= 0) return BUFFALO_OK;
  constexpr int kSmem = 2 * 2 * 3 * kDwTile + 256 + 1024;
  CUtensorMap zm, sm, am;
  constexpr CUtensorMapSwizzle kMN = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
  BF_CHECK(encode_f32(&zm, q.Z, q.d_out, q.n, q.ldz, kKC, kMN));
  // gathered self rows: the table's height is not known here; the gather indices are the
  // block's validated node ids, so every requested row exists
  BF_CHECK(encode_f32(&sm, (const float*)q.self, q.d_in, q.gidx ? (int64_t)INT32_MAX : q.n, q.lds, q.gidx ? 1 : kKC,
                      kMN));
  BF_CHECK(encode_f32(&am, q.agg ? q.agg : (const float*)q.self, q.d_in, q.n, q.agg ? q.lda : q.lds, kKC, kMN));
  TcfDwTmaP p{};
  p.n = q.n;
  p.rows_per_split = round_up(ceil_div(q.n, S), kKC);
  p.d_out = q.d_out;
  p.d_in = q.d_in;
  p.tiles_self = (int)ceil_div(q.d_in, 128);
  p.Kd = q.agg ? 2 * q.d_in : q.d_in;
  p.gidx = q.gidx;
  p.part = q.part;
  dim3 grid((unsigned)ceil_div(q.d_out, kTM), (unsigned)(q.agg ? 2 * p.tiles_self : p.tiles_self), (unsigned)S);
  if (q.gidx) {
    BF_CHECK((set_max_smem_once<k_tcf_dw_tma<true>>(kSmem)));
    k_tcf_dw_tma<true><<<grid, kDwTmaThreads, kSmem, s>>>(zm, sm, am, p);
  } else {
    BF_CHECK((set_max_smem_once<k_tcf_dw_tma<false>>(kSmem)));
    k_tcf_dw_tma<false><<<grid, kDwTmaThreads, kSmem, s>>>(zm, sm, am, p);
  }
  BF_LAUNCHED("k_tcf_dw_tma");
  return BUFFALO_OK;
}

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

template <class TA1, bool TB, int NS>
static buffalo_status launch_tcf_gemm_ns(const TcfGemm& p, cudaStream_t s) {
  constexpr int kSmem = (NS == 2 ? 3 : 2) * NS * (kTileA + 128 * 128) + 256 + 1024;
  const int64_t tiles = ((p.M + kTM - 1) / kTM) * ((p.Np + 127) / 128);
  const int grid = (int)std::min<int64_t>(tiles, 148);
  BF_CHECK((set_max_smem_once<k_tcf_gemm<TA1, TB, NS>>(kSmem)));
  k_tcf_gemm<TA1, TB, NS><<<grid, kGemmThreads, kSmem, s>>>(p);
  BF_LAUNCHED("k_tcf_gemm");
  return BUFFALO_OK;
}
template <class TA1, bool TB>
static buffalo_status launch_tcf_gemm(const TcfGemm& p, bool exact, cudaStream_t s) {
  return exact ? launch_tcf_gemm_ns<TA1, TB, 3>(p, s) : launch_tcf_gemm_ns<TA1, TB, 2>(p, s);
}

template <bool TB, int NS, bool GATHER>
static buffalo_status launch_tcf_gemm_tma(const TcfGemm& q, cudaStream_t s) {
  constexpr int kSmem = (NS == 2 ? 3 : 2) * 2 * NS * kTM * 128 + 256 + 1024;
  constexpr CUtensorMapSwizzle kK = CU_TENSOR_MAP_SWIZZLE_128B, kMN = CU_TENSOR_MAP_SWIZZLE_128B_ATOM_32B;
  CUtensorMap a1, a2, b1, b2;
  const float* A1 = (const float*)q.A1;
  const float* A2 = q.A2 ? q.A2 : A1;
  const float* B2 = q.B2 ? q.B2 : q.B1;
  // A1 rows beyond m1 carry no A1 term: the map ends there (gathered: the split zeroes them)
  BF_CHECK(encode_f32(&a1, A1, q.K1, GATHER ? (int64_t)INT32_MAX : q.m1, q.lda1, GATHER ? 1 : kTM, kK));
  BF_CHECK(encode_f32(&a2, A2, q.K2 > 0 ? q.K2 : q.K1, q.M, q.A2 ? q.lda2 : q.lda1, kTM, kK));
  if (TB) {
    BF_CHECK(encode_f32(&b1, q.B1, q.K1, q.N, q.ldb1, 128, kK));
    BF_CHECK(encode_f32(&b2, B2, q.K2 > 0 ? q.K2 : q.K1, q.N, q.B2 ? q.ldb2 : q.ldb1, 128, kK));
  } else {
    BF_CHECK(encode_f32(&b1, q.B1, q.N, q.K1, q.ldb1, kKC, kMN));
    BF_CHECK(encode_f32(&b2, B2, q.N, q.K2 > 0 ? q.K2 : q.K1, q.B2 ? q.ldb2 : q.ldb1, kKC, kMN));
  }
  TcfGemmTmaP p{};
  p.M = q.M; p.m1 = q.m1; p.N = q.N; p.Np = q.Np; p.K1 = q.K1; p.K2 = q.K2;
  p.gidx = q.gidx; p.bias = q.bias; p.relu = q.relu; p.C = q.C; p.ldc = q.ldc;
  const int64_t tiles = ((q.M + kTM - 1) / kTM) * ((q.Np + 127) / 128);
  const int grid = (int)std::min<int64_t>(tiles, 148);
  BF_CHECK((set_max_smem_once<k_tcf_gemm_tma<TB, NS, GATHER>>(kSmem)));
  k_tcf_gemm_tma<TB, NS, GATHER><<<grid, kGtThreads, kSmem, s>>>(a1, a2, b1, b2, p);
  BF_LAUNCHED("k_tcf_gemm_tma");
  return BUFFALO_OK;
}
template <bool TB, int NS>
static buffalo_status launch_tcf_gemm_tma_g(const TcfGemm& q, cudaStream_t s) {
  return q.gidx && q.K1 > 0 ? launch_tcf_gemm_tma<TB, NS, true>(q, s) : launch_tcf_gemm_tma<TB, NS, false>(q, s);
}

buffalo_status tcf_gemm(const TcfGemm& p, bool a1_bf16, bool tb, bool exact, cudaStream_t s) {
  if (p.M <= 0 || p.Np <= 0) return BUFFALO_OK;
  if (!a1_bf16) {
    if (tb) return exact ? launch_tcf_gemm_tma_g<true, 3>(p, s) : launch_tcf_gemm_tma_g<true, 2>(p, s);
    return exact ? launch_tcf_gemm_tma_g<false, 3>(p, s) : launch_tcf_gemm_tma_g<false, 2>(p, s);
  }
  if (a1_bf16)
    return tb ? launch_tcf_gemm<__nv_bfloat16, true>(p, exact, s) : launch_tcf_gemm<__nv_bfloat16, false>(p, exact, s);
  return tb ? launch_tcf_gemm<float, true>(p, exact, s) : launch_tcf_gemm<float, false>(p, exact, s);
}

}  // namespace buffalo
