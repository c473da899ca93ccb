// tc_gemm.cu — the Update GEMM over contiguous operands, TMA-fed (sm_100a).
//
//   out[i] = act([self[i] || agg[i]] W^T + b) (* 1/D(i) optionally),   i < n_rows
//
// self and agg are row-major bf16 matrices whose rows are the tile rows (layers >= 2 of the
// forward: H_{l-1} and the saved h_agg; layer 1: feature rows gathered by tile::gather4), so
// both halves of the A operand are plain 2D tiles: one TMA load (box 64 x 128, SWIZZLE_128B)
// per K-chunk lands them in the UMMA K-major SW128 layout.  With agg = null the A operand is
// self alone (the backward's Ys = dZ W_self and Yn = dZ W_neigh / D products).  The
// pre-swizzled weight chunks stay resident in shared memory when they fit, else each comes
// with a 1D bulk copy into the A chunk's pipeline stage.  Roles: two producer warps issue the
// TMA loads, one elected lane issues tcgen05.mma into a double-buffered TMEM accumulator, and
// eight epilogue warps run tcgen05.ld -> +bias -> ReLU -> bf16 -> TMA store of the previous tile.
#include <cuda.h>

#include <algorithm>

#include "tc_sage.cuh"

namespace buffalo {

namespace {

__device__ __forceinline__ uint32_t su32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }
__device__ __forceinline__ void mb_init(uint64_t* b, uint32_t c) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(su32(b)), "r"(c));
}
__device__ __forceinline__ void mb_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(su32(b)) : "memory");
}
__device__ __forceinline__ void mb_expect(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(su32(b)), "r"(bytes) : "memory");
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
// TMA store of a {32 col, 32 row} bf16 box from SWIZZLE_64B-staged shared memory (bulk group).
__device__ __forceinline__ void tma_store_2d(const CUtensorMap* map, const void* src, int c0, int c1) {
  asm volatile("cp.async.bulk.tensor.2d.global.shared::cta.bulk_group [%0, {%2, %3}], [%1];" ::"l"(
                   reinterpret_cast<uint64_t>(map)),
               "r"(su32(src)), "r"(c0), "r"(c1)
               : "memory");
}
__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void bulk_wait_read() { asm volatile("cp.async.bulk.wait_group.read %0;" ::"n"(N) : "memory"); }
__device__ __forceinline__ void fence_async_smem() { asm volatile("fence.proxy.async.shared::cta;" ::: "memory"); }
// Row `lane` of a 32 x 64-B staging box, 16-B chunk k, in the SWIZZLE_64B layout (chunk ^= row>>1 & 3).
__device__ __forceinline__ void st_stage64(uint8_t* box, int lane, int k, uint4 v) {
  *reinterpret_cast<uint4*>(box + lane * 64 + ((k ^ ((lane >> 1) & 3)) << 4)) = v;
}

__device__ __forceinline__ void bulk_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile("cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                   su32(dst)),
               "l"(src), "r"(bytes), "r"(su32(bar))
               : "memory");
}
__device__ __forceinline__ void fence_after() { asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory"); }
__device__ __forceinline__ void fence_before() { asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory"); }
__device__ __forceinline__ uint64_t desc_sw128(uint32_t saddr) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)1 << 16) | ((uint64_t)(1024 >> 4) << 32) |
         ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}
__device__ __forceinline__ void mma_f16(uint32_t d, uint64_t a, uint64_t b, uint32_t idesc, uint32_t acc) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(d),
      "l"(a), "l"(b), "r"(idesc), "r"(acc));
}
__device__ __forceinline__ void commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(su32(bar))
               : "memory");
}
__device__ __forceinline__ void ld32(uint32_t taddr, float* v) {
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
// Split issue / wait so the next TMEM load overlaps the current group's epilogue math; the
// wait names the destination registers so no use of them can be scheduled above it.
__device__ __forceinline__ void ld32_issue(uint32_t taddr, uint32_t (&r)[32]) {
  asm volatile(
      "tcgen05.ld.sync.aligned.32x32b.x32.b32 {%0, %1, %2, %3, %4, %5, %6, %7, %8, %9, %10, %11, %12, %13, %14, "
      "%15, %16, %17, %18, %19, %20, %21, %22, %23, %24, %25, %26, %27, %28, %29, %30, %31}, [%32];"
      : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]), "=r"(r[7]),
        "=r"(r[8]), "=r"(r[9]), "=r"(r[10]), "=r"(r[11]), "=r"(r[12]), "=r"(r[13]), "=r"(r[14]), "=r"(r[15]),
        "=r"(r[16]), "=r"(r[17]), "=r"(r[18]), "=r"(r[19]), "=r"(r[20]), "=r"(r[21]), "=r"(r[22]), "=r"(r[23]),
        "=r"(r[24]), "=r"(r[25]), "=r"(r[26]), "=r"(r[27]), "=r"(r[28]), "=r"(r[29]), "=r"(r[30]), "=r"(r[31])
      : "r"(taddr));
}
__device__ __forceinline__ void ld32_wait(uint32_t (&r)[32]) {
  asm volatile("tcgen05.wait::ld.sync.aligned;"
               : "+r"(r[0]), "+r"(r[1]), "+r"(r[2]), "+r"(r[3]), "+r"(r[4]), "+r"(r[5]), "+r"(r[6]), "+r"(r[7]),
                 "+r"(r[8]), "+r"(r[9]), "+r"(r[10]), "+r"(r[11]), "+r"(r[12]), "+r"(r[13]), "+r"(r[14]),
                 "+r"(r[15]), "+r"(r[16]), "+r"(r[17]), "+r"(r[18]), "+r"(r[19]), "+r"(r[20]), "+r"(r[21]),
                 "+r"(r[22]), "+r"(r[23]), "+r"(r[24]), "+r"(r[25]), "+r"(r[26]), "+r"(r[27]), "+r"(r[28]),
                 "+r"(r[29]), "+r"(r[30]), "+r"(r[31])
               :
               : "memory");
}
__device__ __forceinline__ uint32_t pk(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}

constexpr int kTM = 128;
constexpr int kChunkA = kTM * 128;     // 16 KB: 128 rows x 64 bf16
constexpr int kEpiWarps = 8;       // two per TMEM lane quadrant (column groups interleaved)
// Producer warps: TMA issue is throughput-limited per issuing warp (tools/tma_bench.cu: one
// issuer reaches ~1.6 TB/s with gather4 and ~4.8 TB/s with 2D boxes, four reach 4.5 / 6.1 TB/s),
// so chunk g of the CTA's sequence is loaded by producer warp g % kProducers.
constexpr int kProducers = 2;
constexpr int kMmaWarp = kEpiWarps + kProducers;
constexpr int kGemmThreads = (kEpiWarps + kProducers + 1) * 32;

// 2-KB TMA-store staging boxes per epilogue warp: one (the warp waits for its previous store to
// have read the box) leaves 16 KB more for the A-operand pipeline — one more stage for the
// layer-1 Update with resident weights; measured 0.4 ms per products epoch faster than two
constexpr int kStageBufs = 1;

struct GemmParams {
  int64_t n_rows;
  int64_t self_tiles;         // tiles t >= self_tiles have no self rows: their self K-chunks are skipped
  const int32_t* self_idx;    // null: self rows are rows of the self map; else row i = self_idx[i] (gather4)
  int32_t self_oob;           // an out-of-bounds row index of the self map (zero rows)
  int nkc_self, nkc;          // K-chunks of the self half, total
  const uint8_t* wpk;         // pre-swizzled weight chunks (Np x 128 B each)
  int Np, d_out, pitch_out, ld_out, tmem_cols, nstages;
  // Resident weights (w_res): the CTA keeps the rows [half * Nsub, (half + 1) * Nsub) of every
  // weight chunk in shared memory for the whole launch (one 1D bulk copy per chunk at start), so
  // the pipeline stages carry A tiles only; with nsplit = 2 the two CTAs of a tile set compute
  // the two column halves of the same tiles (A is read twice, the second time from L2).
  int w_res, nsplit, Nsub;
  int stage_off, stage_bytes; // epilogue staging area (8 warps x kStageBufs x 2 KB)
  const float* bias;
  int relu, out_f32;
  const int32_t* scale_rp;    // non-null: output row i is scaled by 1 / D(i), D(i) = rp[i+1] - rp[i] (0 if D = 0)
  void* out;
};

__global__ void __launch_bounds__(kGemmThreads, 1)
    k_tc_gemm_tma(const __grid_constant__ CUtensorMap self_map, const __grid_constant__ CUtensorMap agg_map,
                  const __grid_constant__ CUtensorMap out_map, const GemmParams p) {
  pdl_wait();
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  // 1024-B alignment by offset (keeps the shared address space visible to the compiler)
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  const int NS = p.nstages;
  const int bbytes = p.Np * 128;                       // one packed weight chunk
  const int wsz = p.Nsub * 128;                        // this CTA's rows of a chunk
  const int half = (int)(blockIdx.x % p.nsplit);
  const int64_t set0 = blockIdx.x / p.nsplit, nsets = gridDim.x / p.nsplit;
  uint8_t* sA = smem;                                  // NS x 16 KB
  uint8_t* sB = smem + NS * kChunkA;                   // streamed: NS x Np x 128 B; resident: nkc x wsz
  uint64_t* full = (uint64_t*)(smem + p.stage_off + p.stage_bytes);   // after the store staging
  uint64_t* empty = full + NS;
  uint64_t* acc_full = empty + NS;
  uint64_t* acc_empty = acc_full + 2;
  uint64_t* wbar = acc_empty + 2;
  uint32_t* tmem_slot = (uint32_t*)(wbar + 2);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t ntiles = (p.n_rows + kTM - 1) / kTM;
  const int col_base = half * p.Nsub;                  // first output column of this CTA

  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) { mb_init(&full[i], 1); mb_init(&empty[i], 1); }
    for (int i = 0; i < 2; ++i) { mb_init(&acc_full[i], 1); mb_init(&acc_empty[i], kEpiWarps * 32); }
    mb_init(wbar, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(tmem_slot)),
                 "r"(p.tmem_cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;

  if (warp >= kEpiWarps && warp < kMmaWarp) {
    // ---------------- producer: A chunk (TMA 2D, or 32 x gather4 for gathered self rows) +
    // weight chunk (bulk) per stage
    const int pw = warp - kEpiWarps;                 // this producer's share: chunks g % kProducers == pw
    if (lane == 0) {
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&self_map)) : "memory");
      asm volatile("prefetch.tensormap [%0];" ::"l"(reinterpret_cast<uint64_t>(&agg_map)) : "memory");
      if (p.w_res && pw == 0) {                                   // the CTA's weight rows, once
        const int c_lo = p.self_tiles > 0 ? 0 : p.nkc_self;
        mb_expect(wbar, (uint32_t)((p.nkc - c_lo) * wsz));
        for (int c = c_lo; c < p.nkc; ++c)
          bulk_1d(sB + c * wsz, p.wpk + (int64_t)c * bbytes + (int64_t)col_base * 128, wsz, wbar);
      }
    }
    int64_t g = 0;
    for (int64_t t = set0; t < ntiles; t += nsets) {
      const int row0 = (int)(t * kTM);
      int32_t idx[4];
      if (p.self_idx) {
#pragma unroll
        for (int k = 0; k < 4; ++k) {
          const int64_t r = (int64_t)row0 + lane * 4 + k;
          idx[k] = r < p.n_rows ? __ldg(p.self_idx + r) : p.self_oob;
        }
      }
      const int cb = t >= p.self_tiles ? p.nkc_self : 0;
      for (int c = cb; c < p.nkc; ++c, ++g) {
        if ((int)(g % kProducers) != pw) continue;
        const int st = (int)(g % NS);
        if (lane == 0) {
          if (g >= NS) mb_wait(&empty[st], (uint32_t)(((g / NS) - 1) & 1));
          mb_expect(&full[st], kChunkA + (p.w_res ? 0 : bbytes));
        }
        __syncwarp();
        if (c < p.nkc_self && p.self_idx) {
          tma_gather4(sA + st * kChunkA + lane * 4 * 128, &self_map, c * 64, idx[0], idx[1], idx[2], idx[3], &full[st]);
        } else if (lane == 0) {
          if (c < p.nkc_self) tma_2d(sA + st * kChunkA, &self_map, c * 64, row0, &full[st]);
          else tma_2d(sA + st * kChunkA, &agg_map, (c - p.nkc_self) * 64, row0, &full[st]);
        }
        if (lane == 0 && !p.w_res) bulk_1d(sB + st * bbytes, p.wpk + (int64_t)c * bbytes, bbytes, &full[st]);
        __syncwarp();
      }
    }
  } else if (warp == kMmaWarp) {
    if (lane == 0) {
      // ---------------- MMA issuer
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(p.Nsub >> 3) << 17) |
                             ((uint32_t)(kTM >> 4) << 24);
      if (p.w_res) mb_wait(wbar, 0);
      int64_t g = 0, i = 0;
      for (int64_t t = set0; t < ntiles; t += nsets, ++i) {
        const int acc = (int)(i & 1);
        if (i >= 2) mb_wait(&acc_empty[acc], (uint32_t)(((i >> 1) - 1) & 1));
        fence_after();
        const uint32_t d = tmem + acc * p.Nsub;
        const int cb = t >= p.self_tiles ? p.nkc_self : 0;
        for (int c = cb; c < p.nkc; ++c, ++g) {
          const int st = (int)(g % NS);
          mb_wait(&full[st], (uint32_t)((g / NS) & 1));
          fence_after();
          const uint32_t a = su32(sA + st * kChunkA), b = su32(p.w_res ? sB + c * wsz : sB + st * bbytes);
#pragma unroll
          for (int k = 0; k < 4; ++k)
            mma_f16(d, desc_sw128(a + 32 * k), desc_sw128(b + 32 * k), idesc, (c > cb || k > 0) ? 1u : 0u);
          commit(&empty[st]);
        }
        commit(&acc_full[acc]);
      }
    }
    __syncwarp();
  } else {
    // ---------------- epilogue: warp e owns TMEM lane quadrant q = e & 3 (tile rows 32q..32q+31)
    // and the 32-column groups g = 2j + h (h = e >> 2): +bias, ReLU, optional 1/D row scale,
    // store.  The next TMEM load is issued before the current group's math.
    const int q = warp & 3, h = warp >> 2;
    float* sbias = reinterpret_cast<float*>(tmem_slot + 4);   // 16-B aligned
    uint8_t* stg = smem + p.stage_off + warp * (2048 * kStageBufs);   // this warp's 2-KB staging box(es)
    int sbuf = 0;
    for (int c = threadIdx.x; c < p.Nsub; c += kEpiWarps * 32)
      sbias[c] = (p.bias && col_base + c < p.d_out) ? __ldg(p.bias + col_base + c) : 0.f;
    asm volatile("bar.sync 1, %0;" ::"n"(kEpiWarps * 32) : "memory");
    const int ncol_cta = min(p.Nsub, p.pitch_out - col_base);   // output columns of this CTA
    const int ng = (ncol_cta + 31) / 32;
    const int nj = (ng - h + 1) / 2;              // groups of this warp (<= 4)
    int64_t i = 0;
    for (int64_t t = set0; t < ntiles; t += nsets, ++i) {
      const int acc = (int)(i & 1);
      mb_wait(&acc_full[acc], (uint32_t)((i >> 1) & 1));
      fence_after();
      const int64_t row = t * kTM + q * 32 + lane;
      const bool rok = row < p.n_rows;
      const uint32_t tbase = tmem + ((uint32_t)(q * 32) << 16) + acc * p.Nsub;
      float rscale = 1.f;
      if (rok && p.scale_rp) {
        const int32_t d = __ldg(p.scale_rp + row + 1) - __ldg(p.scale_rp + row);
        rscale = d > 0 ? 1.f / (float)d : 0.f;
      }
      uint32_t r[2][32];
      if (nj > 0) {
        ld32_issue(tbase + h * 32, r[0]);
        ld32_wait(r[0]);
      }
#pragma unroll
      for (int j = 0; j < 4; ++j) {
        if (j < nj) {
          const int c0 = (2 * j + h) * 32;
          if (j + 1 < nj) ld32_issue(tbase + c0 + 64, r[(j + 1) & 1]);
          const int ncols = min(32, ncol_cta - c0);      // multiple of 8
          const int gc0 = col_base + c0;                 // global output column
          float v[32];
#pragma unroll
          for (int k = 0; k < 32; ++k) v[k] = __uint_as_float(r[j & 1][k]);
#pragma unroll
          for (int k = 0; k < 32; k += 4) {
            const float4 bb = *reinterpret_cast<const float4*>(sbias + c0 + k);
            v[k] += bb.x; v[k + 1] += bb.y; v[k + 2] += bb.z; v[k + 3] += bb.w;
          }
          if (p.relu) {
#pragma unroll
            for (int k = 0; k < 32; ++k) v[k] = fmaxf(v[k], 0.f);
          }
          if (p.scale_rp) {
#pragma unroll
            for (int k = 0; k < 32; ++k) v[k] *= rscale;
          }
          if (p.out_f32) {
            if (rok) {
              float* o = (float*)p.out + row * p.ld_out + gc0;
#pragma unroll
              for (int k = 0; k < 32; k += 4)
                if (k < ncols) *reinterpret_cast<float4*>(o + k) = make_float4(v[k], v[k + 1], v[k + 2], v[k + 3]);
            }
          } else {
            // bf16 rows through a staging box and one TMA store per warp and column group
            // (coalesced, asynchronous; rows past n_rows are clipped by the map)
            uint8_t* box = stg + sbuf * 2048;
            sbuf = (sbuf + 1) % kStageBufs;
            if (lane == 0) bulk_wait_read<kStageBufs - 1>();   // the store that used this box has read it
            __syncwarp();
#pragma unroll
            for (int k = 0; k < 4; ++k)
              st_stage64(box, lane, k, make_uint4(pk(v[8 * k], v[8 * k + 1]), pk(v[8 * k + 2], v[8 * k + 3]),
                                                   pk(v[8 * k + 4], v[8 * k + 5]), pk(v[8 * k + 6], v[8 * k + 7])));
            fence_async_smem();
            __syncwarp();
            if (lane == 0) {
              tma_store_2d(&out_map, box, gc0, (int)(t * kTM + q * 32));
              bulk_commit();
            }
          }
          if (j + 1 < nj) ld32_wait(r[(j + 1) & 1]);
        }
      }
      fence_before();
      mb_arrive(&acc_empty[acc]);
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
    __syncwarp();
  }
  fence_before();
  __syncthreads();
  if (warp == kMmaWarp) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(p.tmem_cols));
  }
}


// ================================================================== dW on tensor cores, TMA-fed
// part[split][m][n'] = sum_{r in split} dZ[r][m] * Afwd[r][n'],  Afwd = [self || agg] with n'
// padded per half to Dp.  Both operands are MN-major in shared memory: a 64-column strip of 64
// rows is exactly one TMA box {64, 64} with SWIZZLE_128B (gathered self rows: 16 x gather4).
// One CTA owns all m-tiles (<= 2 x 128 TMEM lanes) of one 256-wide n'-tile and a row split.
constexpr int kDwR = 64;
constexpr int kDwStrip2 = kDwR * 128;      // 8 KB

struct DwParams {
  int64_t n, rows_per_split;
  int MT, NT, Dp, nself_strips, d_out, tmem_cols, nstages;
  const int32_t* gidx;                     // layer 1: self row r = gidx[r]
  float* part;
};

__device__ __forceinline__ uint64_t desc_mn(uint32_t saddr, uint32_t lbo) {
  return (uint64_t)((saddr >> 4) & 0x3FFF) | ((uint64_t)((lbo >> 4) & 0x3FFF) << 16) |
         ((uint64_t)(1024 >> 4) << 32) | ((uint64_t)1 << 46) | ((uint64_t)2 << 61);
}

constexpr int kDwProducers = 2;                 // chunk c is loaded by producer warp 4 + c % 2
constexpr int kDwMmaWarp = 4 + kDwProducers;
constexpr int kDwThreads2 = (kDwMmaWarp + 1) * 32;

__global__ void __launch_bounds__(kDwThreads2, 1)
    k_tc_dw_tma(const __grid_constant__ CUtensorMap z_map, const __grid_constant__ CUtensorMap self_map,
                const __grid_constant__ CUtensorMap agg_map, const DwParams p) {
  pdl_wait();
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = smem_raw + ((1024u - (su32(smem_raw) & 1023u)) & 1023u);
  const int NS = p.nstages;
  const int nA = 2 * p.MT, nB = p.NT / 64;
  const int stage = (nA + nB) * kDwStrip2;
  uint64_t* full = (uint64_t*)(smem + NS * stage);
  uint64_t* empty = full + NS;
  uint64_t* done = empty + NS;
  uint32_t* tmem_slot = (uint32_t*)(done + 1);
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int n0 = blockIdx.x * p.NT;
  const int64_t r_beg = (int64_t)blockIdx.y * p.rows_per_split;
  const int64_t r_end = min(p.n, r_beg + p.rows_per_split);
  const int nchunks = r_end > r_beg ? (int)((r_end - r_beg + kDwR - 1) / kDwR) : 0;
  if (threadIdx.x == 0) {
    for (int i = 0; i < NS; ++i) { mb_init(&full[i], 1); mb_init(&empty[i], 1); }
    mb_init(done, 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  if (warp == kDwMmaWarp) {
    asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(su32(tmem_slot)),
                 "r"(p.tmem_cols));
    asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
  }
  fence_before();
  __syncthreads();
  fence_after();
  const uint32_t tmem = *tmem_slot;
  if (warp >= 4 && warp < kDwMmaWarp) {
    // ---------------- producers
    for (int c = warp - 4; c < nchunks; c += kDwProducers) {
      const int st = c % NS;
      const int r0 = (int)(r_beg + (int64_t)c * kDwR);
      if (lane == 0) {
        if (c >= NS) mb_wait(&empty[st], (uint32_t)(((c / NS) - 1) & 1));
        mb_expect(&full[st], stage);
      }
      __syncwarp();
      uint8_t* sa = smem + st * stage;
      uint8_t* sb = sa + nA * kDwStrip2;
      if (lane == 0) {
        for (int j = 0; j < nA; ++j) tma_2d(sa + j * kDwStrip2, &z_map, j * 64, r0, &full[st]);
      }
      for (int j = 0; j < nB; ++j) {
        const int np = n0 + j * 64;               // first n' column of the strip
        if (np < p.Dp) {
          if (p.gidx) {
            // 64 gathered rows = 16 gather4; lanes 0..15 issue one each
            if (lane < 16) {
              int32_t rr[4];
#pragma unroll
              for (int k = 0; k < 4; ++k) {
                const int64_t r = (int64_t)r0 + lane * 4 + k;
                rr[k] = r < p.n ? __ldg(p.gidx + r) : 0;
              }
              tma_gather4(sb + j * kDwStrip2 + lane * 4 * 128, &self_map, np, rr[0], rr[1], rr[2], rr[3], &full[st]);
            }
          } else if (lane == 0) {
            tma_2d(sb + j * kDwStrip2, &self_map, np, r0, &full[st]);
          }
        } else if (lane == 0) {
          tma_2d(sb + j * kDwStrip2, &agg_map, np - p.Dp, r0, &full[st]);
        }
      }
      __syncwarp();
    }
  } else if (warp == kDwMmaWarp) {
    if (lane == 0) {
      const uint32_t idesc = (1u << 4) | (1u << 7) | (1u << 10) | (1u << 15) | (1u << 16) |
                             ((uint32_t)(p.NT >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
      for (int c = 0; c < nchunks; ++c) {
        const int st = c % NS;
        mb_wait(&full[st], (uint32_t)((c / NS) & 1));
        fence_after();
        const uint32_t a = su32(smem + st * stage), b = a + nA * kDwStrip2;
        for (int mt = 0; mt < p.MT; ++mt)
#pragma unroll
          for (int kk = 0; kk < kDwR / 16; ++kk)
            mma_f16(tmem + mt * p.NT, desc_mn(a + mt * 2 * kDwStrip2 + kk * 2048, kDwStrip2),
                    desc_mn(b + kk * 2048, kDwStrip2), idesc, (c > 0 || kk > 0) ? 1u : 0u);
        commit(&empty[st]);
      }
      if (nchunks > 0) commit(done);
    }
    __syncwarp();
  } else {
    // ---------------- epilogue: warp w -> TMEM lane quadrant w (m rows), all m-tiles
    if (nchunks > 0) {
      mb_wait(done, 0);
      fence_after();
    }
    const int64_t K2 = 2 * (int64_t)p.Dp;
    float* P = p.part + (int64_t)blockIdx.y * p.d_out * K2;
    for (int mt = 0; mt < p.MT; ++mt) {
      const int m = mt * 128 + warp * 32 + lane;
      for (int c0 = 0; c0 < p.NT; c0 += 32) {
        float v[32];
        if (nchunks > 0) {
          ld32(tmem + ((uint32_t)(warp * 32) << 16) + mt * p.NT + c0, v);
        } else {
#pragma unroll
          for (int k = 0; k < 32; ++k) v[k] = 0.f;
        }
        const int nn = n0 + c0;
        if (m < p.d_out && nn < K2) {
          float* o = P + (int64_t)m * K2 + nn;
#pragma unroll
          for (int k = 0; k < 32; k += 4) *reinterpret_cast<float4*>(o + k) = make_float4(v[k], v[k + 1], v[k + 2], v[k + 3]);
        }
      }
    }
  }
  fence_before();
  __syncthreads();
  if (warp == kDwMmaWarp) {
    fence_after();
    asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(tmem), "r"(p.tmem_cols));
  }
}

typedef CUresult (*EncodeTiledFn)(CUtensorMap*, CUtensorMapDataType, cuuint32_t, void*, const cuuint64_t*,
                                  const cuuint64_t*, const cuuint32_t*, const cuuint32_t*, CUtensorMapInterleave,
                                  CUtensorMapSwizzle, CUtensorMapL2promotion, CUtensorMapFloatOOBfill);

buffalo_status encode_map(CUtensorMap* map, const void* base, int64_t cols, int64_t rows, int64_t ld,
                          int box_rows = kTM, int box_cols = 64,
                          CUtensorMapSwizzle swz = CU_TENSOR_MAP_SWIZZLE_128B) {
  static EncodeTiledFn fn = nullptr;
  if (!fn) {
    void* f = nullptr;
    cudaDriverEntryPointQueryResult q;
    BF_CUDA(cudaGetDriverEntryPoint("cuTensorMapEncodeTiled", &f, cudaEnableDefault, &q));
    if (!f || q != cudaDriverEntryPointSuccess) {
      set_error("cuTensorMapEncodeTiled unavailable");
      return BUFFALO_ERR_CUDA;
    }
    fn = (EncodeTiledFn)f;
  }
  const cuuint64_t dims[2] = {(cuuint64_t)cols, (cuuint64_t)(rows > 0 ? rows : 1)};
  const cuuint64_t strides[1] = {(cuuint64_t)ld * 2};
  const cuuint32_t box[2] = {(cuuint32_t)box_cols, (cuuint32_t)box_rows};
  const cuuint32_t estr[2] = {1, 1};
  CUresult r = fn(map, CU_TENSOR_MAP_DATA_TYPE_BFLOAT16, 2, const_cast<void*>(base), dims, strides, box, estr,
                  CU_TENSOR_MAP_INTERLEAVE_NONE, swz, CU_TENSOR_MAP_L2_PROMOTION_L2_256B,
                  CU_TENSOR_MAP_FLOAT_OOB_FILL_NONE);
  if (r != CUDA_SUCCESS) {
    set_error("cuTensorMapEncodeTiled failed (%d)", (int)r);
    return BUFFALO_ERR_CUDA;
  }
  return BUFFALO_OK;
}

}  // namespace

// dW partials with TMA operands.  z: bf16 dZ [n][ldz] (first d_out columns); self: bf16 rows
// (gidx: gathered from a table), agg: bf16 saved h_agg [n][lda].  part: [S][d_out][2 Dp].
buffalo_status tc_dw_tma(int64_t n, int S, const __nv_bfloat16* z, int64_t ldz, int d_out,
                         const __nv_bfloat16* self, int64_t lds, const int32_t* gidx, int64_t self_table_rows,
                         const __nv_bfloat16* agg, int64_t lda, int d_in, float* part, cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  const int64_t Dp = round_up(d_in, 64);
  const int64_t pin = pitch_of(d_in), pz = pitch_of(d_out);
  CUtensorMap zm, sm, am;
  BF_CHECK(encode_map(&zm, z, pz, n, ldz, kDwR));
  BF_CHECK(encode_map(&sm, self, pin, gidx ? self_table_rows : n, lds, gidx ? 1 : kDwR));
  BF_CHECK(encode_map(&am, agg, pin, n, lda, kDwR));
  DwParams p{};
  p.n = n;
  p.MT = (int)ceil_div(d_out, 128);
  p.NT = (int)std::min<int64_t>(256, 2 * Dp);
  p.Dp = (int)Dp;
  p.d_out = d_out;
  p.gidx = gidx;
  p.part = part;
  p.rows_per_split = round_up(ceil_div(n, S), kDwR);
  int cols = 32;
  while (cols < p.MT * p.NT) cols *= 2;
  p.tmem_cols = cols;
  const int stage = (2 * p.MT + p.NT / 64) * kDwStrip2;
  p.nstages = std::max(2, std::min(6, (200 * 1024) / stage));
  const int smem = p.nstages * stage + 16 * p.nstages + 64 + 1024;
  BF_CHECK(set_max_smem_once<k_tc_dw_tma>(227 * 1024));
  dim3 grid((unsigned)ceil_div(2 * Dp, p.NT), (unsigned)S);
  launch_pdl(k_tc_dw_tma, grid, dim3(kDwThreads2), (size_t)smem, s, zm, sm, am, p);
  BF_LAUNCHED("k_tc_dw_tma");
  return BUFFALO_OK;
}

// out[n_rows][ld_out] = act([self || agg] W^T + b); self: bf16 [self_rows][ld_self] (first d_in
// columns used, columns up to round_up(d_in, 64) read as zero beyond the pitch), agg likewise.
buffalo_status tc_gemm_tma(int64_t n_rows, int64_t self_rows, const int32_t* self_idx, const __nv_bfloat16* self,
                           int64_t ld_self, const __nv_bfloat16* agg, int64_t ld_agg, int d_in, const uint8_t* wpk,
                           int d_out, const float* bias, int relu, int out_f32, void* out, int64_t ld_out,
                           cudaStream_t s, const int32_t* scale_rp) {
  if (n_rows <= 0) return BUFFALO_OK;
  CUtensorMap sm, am;
  const int64_t pin = pitch_of(d_in);
  // self_idx: self rows gathered (row i = self_idx[i] of a [self_rows] table, box 64 x 1);
  // else rows >= self_rows of the self half read as zero (TMA out-of-bounds fill).
  // agg = null: a single operand (K = d_in): out = self W^T over the first nkc_self weight chunks
  BF_CHECK(encode_map(&sm, self, pin, self_rows, ld_self, self_idx ? 1 : kTM));
  if (agg) BF_CHECK(encode_map(&am, agg, pin, n_rows, ld_agg));
  else am = sm;
  GemmParams p{};
  p.n_rows = n_rows;
  p.self_tiles = self_idx ? ceil_div(n_rows, kTM) : ceil_div(self_rows, kTM);
  p.self_idx = self_idx;
  p.self_oob = self_idx ? 0 : (int32_t)self_rows;
  p.nkc_self = (int)ceil_div(d_in, 64);
  p.nkc = agg ? 2 * p.nkc_self : p.nkc_self;
  p.scale_rp = scale_rp;
  p.wpk = wpk;
  p.Np = (int)round_up(d_out, 16);
  p.d_out = d_out;
  p.pitch_out = (int)pitch_of(d_out);
  p.ld_out = (int)ld_out;
  // resident weights when all weight chunks fit next to >= 4 A stages and the store staging
  // (a CTA-pair column split, nsplit = 2, is supported by the kernel but measured slower)
  const int64_t w_all = (int64_t)p.nkc * p.Np * 128;
  const int64_t kStaging = kEpiWarps * 2048 * kStageBufs;
  const int misc = 16 * 8 + 48 + 4 * p.Np + 1024;                    // barriers, slot, bias, alignment
  p.nsplit = 1;
  p.w_res = (227 * 1024 - w_all - kStaging - misc) / kChunkA >= 4 ? 1 : 0;
  p.Nsub = p.Np / p.nsplit;
  int cols = 32;
  while (cols < 2 * p.Nsub) cols *= 2;
  p.tmem_cols = cols;
  p.bias = bias;
  p.relu = relu;
  p.out_f32 = out_f32;
  p.out = out;
  int smem;
  if (p.w_res) {
    const int64_t wres = (int64_t)p.nkc * p.Nsub * 128;               // chunks < c_lo stay unused
    p.nstages = (int)std::min<int64_t>(8, (227 * 1024 - wres - kStaging - misc) / kChunkA);
    p.stage_off = (int)(p.nstages * kChunkA + wres);
  } else {
    const int stage = kChunkA + p.Np * 128;
    p.nstages = std::max(2, std::min<int>(8, (int)((227 * 1024 - kStaging - misc) / stage)));
    p.stage_off = p.nstages * stage;
  }
  p.stage_bytes = (int)kStaging;
  smem = (int)(p.stage_off + kStaging + misc);
  // output map for the TMA-store epilogue: {32 col, 32 row} boxes, SWIZZLE_64B staging
  CUtensorMap om;
  if (!out_f32) BF_CHECK(encode_map(&om, out, p.pitch_out, n_rows, ld_out, 32, 32, CU_TENSOR_MAP_SWIZZLE_64B));
  else om = am;                                                       // unused (fp32 rows stored directly)
  BF_CHECK(set_max_smem_once<k_tc_gemm_tma>(227 * 1024));
  const int64_t sets = std::min<int64_t>(ceil_div(n_rows, kTM), 148 / p.nsplit);
  const int grid = (int)(sets * p.nsplit);
  launch_pdl(k_tc_gemm_tma, dim3(grid), dim3(kGemmThreads), (size_t)smem, s, sm, am, om, p);
  BF_LAUNCHED("k_tc_gemm_tma");
  return BUFFALO_OK;
}

}  // namespace buffalo
