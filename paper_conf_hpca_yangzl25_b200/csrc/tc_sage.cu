// tc_sage.cu — fused GraphSAGE-mean forward on the 5th-gen tensor cores (sm_100a).
//
// One persistent CTA per SM walks tiles of 128 destination rows.  16 gather warps build the
// A operand [h_self || h_agg] (bf16) of the tile directly in shared memory, in the UMMA
// K-major SWIZZLE_128B layout, 64 columns (one 128-B swizzle atom) per K-chunk:
//   * self chunks: the dst rows' own features (row = gidx[i] for layer 1);
//   * agg chunks:  warp per dst row, 4 lane groups x 8 lanes x 16 B cover 4 neighbours x 64
//     columns per step; 32 column indices are fetched coalesced once and broadcast by
//     shuffles, so each lane keeps 8 independent 16-B loads in flight; fp32 accumulation,
//     one division by D (Alg. 2 l.8, R21); the mean is also written to the saved h_agg.
// One control warp streams pre-swizzled bf16 weight chunks with cp.async.bulk (mbarrier
// transaction counts) and one elected thread issues tcgen05.mma (M=128, N=Np, K=16) into a
// double-buffered TMEM accumulator; the gather warps run the epilogue of tile t-1
// (tcgen05.ld -> +bias -> ReLU -> store) after gathering tile t, so MMA latency hides under
// the next gather.  Rows with D > kHeavyT were pre-aggregated by k_agg_heavy (sage.cu).
#include <algorithm>
#include <cstdlib>

#include "tc_sage.cuh"

namespace buffalo {

// ------------------------------------------------------------------ PTX helpers
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* b, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(b)), "r"(count));
}
__device__ __forceinline__ void mbar_arrive(uint64_t* b) {
  asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(b)) : "memory");
}
__device__ __forceinline__ void mbar_arrive_expect_tx(uint64_t* b, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(b)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* b, uint32_t parity) {
  asm volatile(
      "{\n\t.reg .pred P1;\n\t"
      "WAIT_%=:\n\t"
      "mbarrier.try_wait.parity.shared::cta.b64 P1, [%0], %1;\n\t"
      "@P1 bra DONE_%=;\n\t"
      "bra WAIT_%=;\n\t"
      "DONE_%=:\n\t}" ::"r"(smem_u32(b)),
      "r"(parity)
      : "memory");
}
__device__ __forceinline__ void fence_barrier_init() {
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
}
__device__ __forceinline__ void fence_proxy_async_smem() {
  asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_before() {
  asm volatile("tcgen05.fence::before_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void tc_fence_after() {
  asm volatile("tcgen05.fence::after_thread_sync;" ::: "memory");
}
__device__ __forceinline__ void bulk_g2s(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}
__device__ __forceinline__ void tmem_alloc(uint32_t* dst_smem, uint32_t ncols) {
  asm volatile("tcgen05.alloc.cta_group::1.sync.aligned.shared::cta.b32 [%0], %1;" ::"r"(smem_u32(dst_smem)),
               "r"(ncols));
  asm volatile("tcgen05.relinquish_alloc_permit.cta_group::1.sync.aligned;");
}
__device__ __forceinline__ void tmem_dealloc(uint32_t taddr, uint32_t ncols) {
  asm volatile("tcgen05.dealloc.cta_group::1.sync.aligned.b32 %0, %1;" ::"r"(taddr), "r"(ncols));
}
// D[tmem] (+)= A[smem] * B[smem]^T, both K-major; kind::f16 (bf16 in, fp32 accumulate).
__device__ __forceinline__ void umma_bf16(uint32_t tmem_d, uint64_t adesc, uint64_t bdesc, uint32_t idesc,
                                          uint32_t accumulate) {
  asm volatile(
      "{\n\t.reg .pred p;\n\t"
      "setp.ne.b32 p, %4, 0;\n\t"
      "tcgen05.mma.cta_group::1.kind::f16 [%0], %1, %2, %3, p;\n\t}" ::"r"(tmem_d),
      "l"(adesc), "l"(bdesc), "r"(idesc), "r"(accumulate));
}
__device__ __forceinline__ void umma_commit(uint64_t* bar) {
  asm volatile("tcgen05.commit.cta_group::1.mbarrier::arrive::one.shared::cluster.b64 [%0];" ::"r"(
                   smem_u32(bar))
               : "memory");
}
__device__ __forceinline__ void tmem_ld8(uint32_t taddr, float* v) {
  uint32_t r[8];
  asm volatile("tcgen05.ld.sync.aligned.32x32b.x8.b32 {%0, %1, %2, %3, %4, %5, %6, %7}, [%8];"
               : "=r"(r[0]), "=r"(r[1]), "=r"(r[2]), "=r"(r[3]), "=r"(r[4]), "=r"(r[5]), "=r"(r[6]),
                 "=r"(r[7])
               : "r"(taddr));
  asm volatile("tcgen05.wait::ld.sync.aligned;" ::: "memory");
#pragma unroll
  for (int i = 0; i < 8; ++i) v[i] = __uint_as_float(r[i]);
}

// UMMA shared-memory descriptor: K-major, SWIZZLE_128B, SBO = 1024 B (8 rows x 128 B).
__device__ __forceinline__ uint64_t sw128_desc(uint32_t saddr) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)1 << 16;                 // LBO (unused for swizzled K-major)
  d |= (uint64_t)(1024 >> 4) << 32;       // SBO
  d |= (uint64_t)1 << 46;                 // descriptor version (sm100)
  d |= (uint64_t)2 << 61;                 // SWIZZLE_128B
  return d;
}
// Instruction descriptor, kind::f16: D fp32, A/B bf16, both K-major, M = 128, N = n.
__host__ __device__ constexpr uint32_t idesc_bf16(int n) {
  return (1u << 4) | (1u << 7) | (1u << 10) | ((uint32_t)(n >> 3) << 17) | ((uint32_t)(128 >> 4) << 24);
}

__device__ __forceinline__ uint32_t pack_bf16x2(float a, float b) {
  __nv_bfloat162 h = __floats2bfloat162_rn(a, b);
  return *reinterpret_cast<uint32_t*>(&h);
}
// L2 eviction-priority hints (createpolicy + .L2::cache_hint): the Aggregate's gathered rows are
// re-read across rows (hub rows, the dst-side Yn table of the backward), its output rows and
// per-row side inputs are touched once.
__device__ __forceinline__ uint64_t l2_policy_keep() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_policy_stream() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint4 ldg_pol(const void* ptr, uint64_t pol) {
  uint4 r;
  asm("ld.global.nc.L2::cache_hint.v4.u32 {%0, %1, %2, %3}, [%4], %5;"
      : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w)
      : "l"(ptr), "l"(pol));
  return r;
}
__device__ __forceinline__ void stg_pol(void* ptr, const uint4& v, uint64_t pol) {
  asm volatile("st.global.L2::cache_hint.v4.u32 [%0], {%1, %2, %3, %4}, %5;" ::"l"(ptr), "r"(v.x), "r"(v.y),
               "r"(v.z), "r"(v.w), "l"(pol)
               : "memory");
}
__device__ __forceinline__ void bf16x8_to_f32(const uint4& u, float* v) {
  const uint32_t w[4] = {u.x, u.y, u.z, u.w};
#pragma unroll
  for (int i = 0; i < 4; ++i) {
    v[2 * i] = __uint_as_float(w[i] << 16);
    v[2 * i + 1] = __uint_as_float(w[i] & 0xffff0000u);
  }
}

__device__ __forceinline__ void cp_async16(void* dst, const void* src, bool valid) {
  asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(smem_u32(dst)), "l"(src),
               "r"(valid ? 16 : 0)
               : "memory");
}
__device__ __forceinline__ void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ __forceinline__ void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }

// ------------------------------------------------------------------ kernel configuration
constexpr int kTileM = 128;
constexpr int kKC = 64;                    // bf16 columns per K-chunk (one 128-B swizzle row)
constexpr int kChunkBytesA = kTileM * 128; // 16 KB
constexpr int kSuper = 4;                  // K-chunks per A buffer
constexpr int kGatherWarps = 16;
constexpr int kGatherThreads = kGatherWarps * 32;
constexpr int kThreads = kGatherThreads + 32;

struct TcFwdParams {
  const int32_t* row_ptr;
  const int32_t* col;        // neighbour row ids into h (global for layer 1, local otherwise)
  const int32_t* gidx;       // self row ids (layer 1: src_global) or null (= i)
  int64_t n_dst;             // output rows (fwd: dst of the block; bwd: src of the block)
  int64_t self_rows;         // rows >= self_rows have a zero self half (bwd: n_dst of the block)
  const void* h;             // neighbour rows, bf16 or fp32
  int64_t ldh;               // elements
  const void* hs;            // self rows (fwd: = h)
  int64_t lds;
  const int32_t* perm;       // tile row order (degree-sorted dst) or null (natural order)
  const __nv_bfloat16* agg_src;  // MODE 2: the aggregate half, bf16 rows [n_dst][ld_agg_src]
  int64_t ld_agg_src;
  int a_chunks, nb;          // K-chunks per A buffer (2 buffers), weight stages
  int d_in, pitch_in;        // pitch_in: valid columns readable in a row (multiple of 8)
  int nkc_self, nkc;         // K-chunks for the self half, total (= 2 nkc_self)
  const uint8_t* wpk;        // pre-swizzled bf16 W chunks, each Np x 128 B
  int Np, d_out, ld_out, tmem_cols;
  const float* bias;
  int relu, out_f32;
  void* out;
  __nv_bfloat16* agg;        // saved h_agg, bf16 [n_dst][ld_agg]
  int64_t ld_agg;
};

template <class TI> struct InTraits;
template <> struct InTraits<__nv_bfloat16> {
  static constexpr int kElems = 8;     // per 16-B piece
};
template <> struct InTraits<float> {
  static constexpr int kElems = 4;
};

// Write v (kElems values, columns [piece*kElems, ...)) of row r into the swizzled A chunk.
template <int E>
__device__ __forceinline__ void st_swz(uint8_t* chunk, int r, int piece, const float* v) {
  if constexpr (E == 8) {
    const int off = r * 128 + (((piece) ^ (r & 7)) << 4);
    *reinterpret_cast<uint4*>(chunk + off) =
        make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                   pack_bf16x2(v[6], v[7]));
  } else {
    const int off = r * 128 + (((piece >> 1) ^ (r & 7)) << 4) + ((piece & 1) << 3);
    *reinterpret_cast<uint2*>(chunk + off) = make_uint2(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]));
  }
}
template <class TI>
__device__ __forceinline__ void ld_piece(const TI* p, float* v);
template <> __device__ __forceinline__ void ld_piece<__nv_bfloat16>(const __nv_bfloat16* p, float* v) {
  bf16x8_to_f32(__ldg(reinterpret_cast<const uint4*>(p)), v);
}
template <> __device__ __forceinline__ void ld_piece<float>(const float* p, float* v) {
  float4 a = __ldg(reinterpret_cast<const float4*>(p));
  v[0] = a.x; v[1] = a.y; v[2] = a.z; v[3] = a.w;
}

template <class TI>
__device__ __forceinline__ void raw_to_f32(const uint4& u, float* v);
template <> __device__ __forceinline__ void raw_to_f32<__nv_bfloat16>(const uint4& u, float* v) {
  bf16x8_to_f32(u, v);
}
template <> __device__ __forceinline__ void raw_to_f32<float>(const uint4& u, float* v) {
  v[0] = __uint_as_float(u.x); v[1] = __uint_as_float(u.y); v[2] = __uint_as_float(u.z); v[3] = __uint_as_float(u.w);
}

// acc[k] += element k of a 16-B piece (bf16: add_bf16x2, common.cuh).
template <class TI>
__device__ __forceinline__ void acc_piece(float* acc, const uint4& u);
template <> __device__ __forceinline__ void acc_piece<__nv_bfloat16>(float* acc, const uint4& u) {
  add_bf16x2(acc[0], acc[1], u.x);
  add_bf16x2(acc[2], acc[3], u.y);
  add_bf16x2(acc[4], acc[5], u.z);
  add_bf16x2(acc[6], acc[7], u.w);
}
template <> __device__ __forceinline__ void acc_piece<float>(float* acc, const uint4& u) {
  acc[0] += __uint_as_float(u.x); acc[1] += __uint_as_float(u.y);
  acc[2] += __uint_as_float(u.z); acc[3] += __uint_as_float(u.w);
}

// Super-chunk schedule of a tile (identical on the gather and the MMA side): the self half in
// groups of kSuper K-chunks, then the aggregate half in groups of kAggChunks(E) K-chunks
// (32 lanes x 16 B = one warp-wide row slice).
template <int E> struct Sched {
  static constexpr int kAggChunks = (32 * E) / kKC;          // 4 (bf16) or 2 (fp32)
  int nself_sc, nagg_sc, nkc_self, nkc, sup, agg;
  __device__ Sched(int nkc_self_, int nkc_, int a_chunks, bool copy_mode)
      : nkc_self(nkc_self_), nkc(nkc_), sup(a_chunks), agg(copy_mode ? a_chunks : kAggChunks) {
    nself_sc = (nkc_self + sup - 1) / sup;
    nagg_sc = (nkc - nkc_self + agg - 1) / agg;
  }
  __device__ int count() const { return nself_sc + nagg_sc; }
  __device__ int first(int sc) const {
    return sc < nself_sc ? sc * sup : nkc_self + (sc - nself_sc) * agg;
  }
  __device__ int size(int sc) const {
    const int f = first(sc);
    return sc < nself_sc ? min(sup, nkc_self - f) : min(agg, nkc - f);
  }
};

// Update GEMM for an fp32 feature table (layer 1, gemm_mode BF16): the self half is read from
// the fp32 rows and rounded to bf16 into the swizzled A tile, the aggregate half (the bf16
// h_agg written by the gather) is copied with cp.async; one elected lane issues tcgen05.mma
// into a double-buffered TMEM accumulator; the epilogue adds the bias, applies ReLU and stores.
// (bf16 tables take the TMA kernel of tc_gemm.cu.)
template <class TI>
__global__ void __launch_bounds__(kThreads, 1) k_tc_update_copy(const TcFwdParams p) {
  constexpr int E = InTraits<TI>::kElems;      // elements per 16-B piece
  constexpr int P = kKC / E;                   // pieces per 64-column chunk row (8 or 16)
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int AC = p.a_chunks, NB = p.nb;                        // chunks per A buffer, B stages
  uint8_t* sA = smem;                                          // 2 x AC x 16 KB
  uint8_t* sB = smem + 2 * AC * kChunkBytesA;                  // NB x Np x 128 B
  const int bbytes = p.Np * 128;
  uint64_t* bars = (uint64_t*)(sB + NB * bbytes);
  uint64_t* a_full = bars;        // [2]
  uint64_t* a_empty = bars + 2;   // [2]
  uint64_t* acc_full = bars + 4;  // [2]
  uint64_t* acc_empty = bars + 6; // [2]
  uint64_t* b_full = bars + 8;    // [NB]
  uint64_t* b_empty = bars + 8 + NB;  // [NB]
  uint32_t* tmem_slot = (uint32_t*)(bars + 8 + 2 * NB);

  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const int64_t ntiles = (p.n_dst + kTileM - 1) / kTileM;
  const Sched<E> sched(p.nkc_self, p.nkc, AC, true);
  const int nsc = sched.count();

  if (threadIdx.x == 0) {
    for (int i = 0; i < 2; ++i) {
      mbar_init(&a_full[i], kGatherThreads);
      mbar_init(&a_empty[i], 1);
      mbar_init(&acc_full[i], 1);
      mbar_init(&acc_empty[i], kGatherThreads);
    }
    for (int i = 0; i < NB; ++i) {
      mbar_init(&b_full[i], 1);
      mbar_init(&b_empty[i], 1);
    }
    fence_barrier_init();
  }
  if (warp == kGatherWarps) tmem_alloc(tmem_slot, p.tmem_cols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem_base = *tmem_slot;

  if (warp == kGatherWarps) {
    // ===================== control warp: weight chunks + MMA issue (one elected lane)
    if (lane == 0) {
      const uint32_t idesc = idesc_bf16(p.Np);
      int64_t g = 0;           // global chunk counter (B stage = g % NB)
      int64_t issued = 0;      // weight chunks loaded so far (chunk x goes to stage x % NB)
      int64_t q = 0;           // global super-chunk counter (A buffer = q & 1)
      int64_t i = 0;           // local tile counter
      const int64_t total_chunks = ((ntiles - blockIdx.x + gridDim.x - 1) / gridDim.x) * p.nkc;
      // keep up to NB - 1 weight chunks in flight ahead of the MMAs; a stage is refilled once
      // the MMAs of the chunk NB positions earlier have retired
      auto top_up = [&](int64_t upto) {
        while (issued < total_chunks && issued < upto) {
          const int st = (int)(issued % NB);
          if (issued >= NB) mbar_wait(&b_empty[st], (uint32_t)(((issued / NB) - 1) & 1));
          mbar_arrive_expect_tx(&b_full[st], bbytes);
          bulk_g2s(sB + st * bbytes, p.wpk + (int64_t)(issued % p.nkc) * bbytes, bbytes, &b_full[st]);
          ++issued;
        }
      };
      top_up(NB);
      for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
        const int acc = (int)(i & 1);
        if (i >= 2) mbar_wait(&acc_empty[acc], (uint32_t)(((i >> 1) - 1) & 1));
        tc_fence_after();
        const uint32_t tmem_d = tmem_base + acc * p.Np;
        for (int sc = 0; sc < nsc; ++sc, ++q) {
          const int buf = (int)(q & 1);
          mbar_wait(&a_full[buf], (uint32_t)((q >> 1) & 1));
          tc_fence_after();
          const int c0 = sched.first(sc), cn_ = sched.size(sc);
          for (int j = 0; j < cn_; ++j) {
            const int c = c0 + j;
            const int bs = (int)(g % NB);
            mbar_wait(&b_full[bs], (uint32_t)((g / NB) & 1));
            tc_fence_after();
            const uint32_t a_addr = smem_u32(sA + (buf * AC + j) * kChunkBytesA);
            const uint32_t b_addr = smem_u32(sB + bs * bbytes);
#pragma unroll
            for (int k = 0; k < kKC / 16; ++k)
              umma_bf16(tmem_d, sw128_desc(a_addr + 32 * k), sw128_desc(b_addr + 32 * k), idesc,
                        (c > 0 || k > 0) ? 1u : 0u);
            umma_commit(&b_empty[bs]);
            ++g;
            top_up(g + NB - 1);
          }
          umma_commit(&a_empty[buf]);
        }
        umma_commit(&acc_full[acc]);
      }
    }
    __syncwarp();
  } else {
    // ===================== gather + epilogue warps
    const TI* __restrict__ h = (const TI*)p.h;
    const TI* __restrict__ hs = (const TI*)p.hs;
    int64_t q = 0, i = 0;
    int64_t prev_tile = -1;
    auto row_of = [&](int64_t pos) -> int64_t { return p.perm ? (int64_t)__ldg(p.perm + pos) : pos; };
    auto epilogue = [&](int64_t tile, int64_t li) {
      const int acc = (int)(li & 1);
      mbar_wait(&acc_full[acc], (uint32_t)((li >> 1) & 1));
      tc_fence_after();
      const int quad = warp & 3, part = warp >> 2;
      const int r = quad * 32 + lane;
      const int64_t pos = tile * kTileM + r;
      const int64_t row = pos < p.n_dst ? row_of(pos) : -1;
      const int ngrp = (int)pitch_of(p.d_out) / 8;
      for (int grp = part; grp < ngrp; grp += 4) {
        float v[8];
        tmem_ld8(tmem_base + ((uint32_t)(quad * 32) << 16) + acc * p.Np + grp * 8, v);
        if (row >= 0) {
#pragma unroll
          for (int k = 0; k < 8; ++k) {
            const int cidx = grp * 8 + k;
            float x = v[k] + ((p.bias && cidx < p.d_out) ? __ldg(p.bias + cidx) : 0.f);
            v[k] = p.relu ? fmaxf(x, 0.f) : x;
          }
          if (p.out_f32) {
            float4* o = reinterpret_cast<float4*>((float*)p.out + row * p.ld_out + grp * 8);
            o[0] = make_float4(v[0], v[1], v[2], v[3]);
            o[1] = make_float4(v[4], v[5], v[6], v[7]);
          } else {
            *reinterpret_cast<uint4*>((__nv_bfloat16*)p.out + row * p.ld_out + grp * 8) =
                make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                           pack_bf16x2(v[6], v[7]));
          }
        }
      }
      tc_fence_before();
      mbar_arrive(&acc_empty[acc]);
    };

    for (int64_t t = blockIdx.x; t < ntiles; t += gridDim.x, ++i) {
      const int64_t pos0 = t * kTileM;
      for (int sc = 0; sc < nsc; ++sc, ++q) {
        const int buf = (int)(q & 1);
        if (q >= 2) mbar_wait(&a_empty[buf], (uint32_t)(((q >> 1) - 1) & 1));
        const int c0 = sched.first(sc), ncs = sched.size(sc);
        uint8_t* abuf = sA + buf * AC * kChunkBytesA;
        if (c0 < p.nkc_self) {
          // self rows: 128 rows x (ncs * P) pieces, strided over the gather threads
          const int pcs = ncs * P;
          for (int u = threadIdx.x; u < kTileM * pcs; u += kGatherThreads) {
            const int r = u / pcs, pc = u % pcs;
            const int64_t pos = pos0 + r;
            const int col0 = c0 * kKC + pc * E;
            int64_t hr = -1;
            if (pos < p.n_dst) {
              const int64_t row = row_of(pos);
              if (row < p.self_rows && col0 < p.pitch_in) hr = p.gidx ? (int64_t)p.gidx[row] : row;
            }
            if constexpr (E == 8) {
              const int off = r * 128 + (((pc % P) ^ (r & 7)) << 4);
              cp_async16(abuf + (pc / P) * kChunkBytesA + off, hr >= 0 ? (const void*)(hs + hr * p.lds + col0) : p.h,
                         hr >= 0);
            } else {
              float v[E];
#pragma unroll
              for (int k = 0; k < E; ++k) v[k] = 0.f;
              if (hr >= 0) ld_piece<TI>(hs + hr * p.lds + col0, v);
              st_swz<E>(abuf + (pc / P) * kChunkBytesA, r, pc % P, v);
            }
          }
        } else {
          // aggregate half precomputed (bf16 rows): plain copy
          const int cb = (c0 - p.nkc_self) * kKC;
          const int pcs = ncs * 8;
          for (int u = threadIdx.x; u < kTileM * pcs; u += kGatherThreads) {
            const int r = u / pcs, pc = u % pcs;
            const int64_t pos = pos0 + r;
            const int col0 = cb + pc * 8;
            const bool ok = pos < p.n_dst && col0 < p.pitch_in;
            const int off = r * 128 + (((pc & 7) ^ (r & 7)) << 4);
            cp_async16(abuf + (pc >> 3) * kChunkBytesA + off,
                       ok ? (const void*)(p.agg_src + row_of(pos) * p.ld_agg_src + col0) : (const void*)p.agg_src, ok);
          }
        }
        // keep two super-chunks of cp.async in flight; super-chunk q-1 is handed to the MMA
        // once its copies landed
        cp_async_commit();
        if (q > 0) {
          cp_async_wait<1>();
          fence_proxy_async_smem();
          mbar_arrive(&a_full[(q - 1) & 1]);
        }
      }
      if (prev_tile >= 0) epilogue(prev_tile, i - 1);
      prev_tile = t;
    }
    if (q > 0) {
      cp_async_wait<0>();
      fence_proxy_async_smem();
      mbar_arrive(&a_full[(q - 1) & 1]);
    }
    if (prev_tile >= 0) epilogue(prev_tile, i - 1);
  }
  tc_fence_before();
  __syncthreads();
  if (warp == kGatherWarps) {
    tc_fence_after();
    tmem_dealloc(tmem_base, p.tmem_cols);
  }
}

// ------------------------------------------------------------------ weight packing
// packed chunk c (c < nkc_self: W_self columns c*64.., else W_neigh) = Np rows x 128 B,
// row n, 16-B piece j stored at piece j ^ (n & 7) (the SWIZZLE_128B image).
__global__ void k_pack_w_tc(const float* __restrict__ W, int d_in, int d_out, int Np, int nkc_self,
                            __nv_bfloat16* __restrict__ out) {
  const int64_t total = (int64_t)2 * nkc_self * Np * kKC;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int kk = (int)(t % kKC);
    const int n = (int)((t / kKC) % Np);
    const int c = (int)(t / ((int64_t)kKC * Np));
    const bool self = c < nkc_self;
    const int col = (self ? c : c - nkc_self) * kKC + kk;
    float v = 0.f;
    if (n < d_out && col < d_in) v = W[(int64_t)n * 2 * d_in + (self ? 0 : d_in) + col];
    const int piece = kk >> 3, e = kk & 7;
    const int64_t off = (int64_t)c * Np * kKC + (int64_t)n * kKC + (((piece ^ (n & 7)) << 3) | e);
    out[off] = __float2bfloat16_rn(v);
  }
}

int64_t tc_fwd_packed_bytes(int64_t d_in, int64_t d_out) {
  return R(round_up(d_out, 16) * 2 * round_up(d_in, 64) * 2);
}
int64_t tc_packed_bytes(int64_t d_in, int64_t d_out) {
  return tc_fwd_packed_bytes(d_in, d_out) + tc_fwd_packed_bytes(d_out, d_in);
}

// Backward image: B[n][k] over n < d_in (output columns of dH), k in [0, 2 Kp):
// k < Kp -> W[k][n] (W_self^T), k >= Kp -> W[k - Kp][d_in + n] (W_neigh^T).
__global__ void k_pack_wt_tc(const float* __restrict__ W, int d_in, int d_out, int Np, int nkc_self,
                             __nv_bfloat16* __restrict__ out) {
  const int64_t total = (int64_t)2 * nkc_self * Np * kKC;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int kk = (int)(t % kKC);
    const int n = (int)((t / kKC) % Np);
    const int c = (int)(t / ((int64_t)kKC * Np));
    const bool self = c < nkc_self;
    const int k = (self ? c : c - nkc_self) * kKC + kk;
    float v = 0.f;
    if (n < d_in && k < d_out) v = W[(int64_t)k * 2 * d_in + (self ? 0 : d_in) + n];
    const int piece = kk >> 3, e = kk & 7;
    const int64_t off = (int64_t)c * Np * kKC + (int64_t)n * kKC + (((piece ^ (n & 7)) << 3) | e);
    out[off] = __float2bfloat16_rn(v);
  }
}

buffalo_status tc_pack_weights(const float* W, int d_in, int d_out, void* packed, cudaStream_t s) {
  const int Np = (int)round_up(d_out, 16), nkc_self = (int)ceil_div(d_in, kKC);
  k_pack_w_tc<<<grid_for((int64_t)2 * nkc_self * Np * kKC, 256), 256, 0, s>>>(W, d_in, d_out, Np, nkc_self,
                                                                            (__nv_bfloat16*)packed);
  BF_LAUNCHED("k_pack_w_tc");
  const int Npb = (int)round_up(d_in, 16), nkb = (int)ceil_div(d_out, kKC);
  __nv_bfloat16* pb = (__nv_bfloat16*)((char*)packed + tc_fwd_packed_bytes(d_in, d_out));
  k_pack_wt_tc<<<grid_for((int64_t)2 * nkb * Npb * kKC, 256), 256, 0, s>>>(W, d_in, d_out, Npb, nkb, pb);
  BF_LAUNCHED("k_pack_wt_tc");
  return BUFFALO_OK;
}

static int smem_bytes_for(int Np, int a_chunks, int nb) {
  return 2 * a_chunks * kChunkBytesA + nb * Np * 128 + 8 * (8 + 2 * nb) + 64 + 1024;
}
static int smem_bytes_for(int Np) { return smem_bytes_for(Np, kSuper, 2); }

bool tc_fwd_supported(const FwdArgs& a) {
  const int Np = (int)round_up(a.d_out, 16);
  return a.act_bf16 && Np <= 256 && smem_bytes_for(Np) <= 227 * 1024;
}

buffalo_status launch_agg_heavy_bf16(const FwdArgs& a, cudaStream_t s);


// ================================================================== high-occupancy gather
// Aggregate kernel used by launch_gather.  Lane groups of LPR lanes (one 16-B piece each,
// LPR a compile-time power of two covering the row) own one row each, rows taken in the
// degree-class order so the G = 32/LPR rows of a warp have (nearly) equal trip counts.  Per
// chunk of LPR edges every lane fetches one column index, then the group issues kU 16-B row
// loads per lane at once (indices broadcast by shuffles, -1 marks an absent edge).  Written for
// few instructions per loaded byte (the earlier row kernel ran ~75 instructions per 16-B load
// and was issue-bound): compile-time lane geometry, no spills (<= 40 registers, 48 warps per
// SM), and the next row's perm / row_ptr entries fetched one iteration ahead so short rows do
// not pay the whole perm -> row_ptr -> col -> row dependency chain each.  MODE 0 writes the
// mean as x * (1/D) corrected by one FMA residual step (Markstein), MODE 1 the plain sum; the
// per-row sum order is the CSR order (R21).  MODE 2 is the backward's transposed Aggregate with
// the layer-below epilogue fused (GatherEpi): for src row j the sum of the pre-scaled rows
// Yn[i] = (dZ_l W_neigh)[i] / D(i) over T(j), plus Ys[j] = (dZ_l W_self)[j] for j < n_dst, gives
// dH_{l-1}[j]; ReLU' with H_{l-1}[j] makes dZ_{l-1}[j], stored in bf16, and its columns are
// summed (db_{l-1}) per lane group in shared memory and per CTA in a fixed order (one partial
// row per CTA: deterministic).
// MODE 3 is MODE 0 over a node-range sharded feature table (buffalo_feature_shards): a
// neighbour's row address is shard[j / rps] + (j % rps) * row bytes, computed once per index by
// the lane that fetched it and broadcast as a 64-bit address; the dst row's own feature row
// (global id gidx[row]) is copied to self_out for the Update and dW GEMMs.
struct GatherEpi {
  const __nv_bfloat16* ys; int64_t ldy;   // Ys [n_self][ldy]
  int64_t n_self;
  const __nv_bfloat16* H; int64_t ldH;    // H_{l-1} (ReLU' mask source)
  int d;                                  // valid columns (d_{l-1}); pad columns are stored as 0
  float* db_part;                         // [gridDim.x][d]
  // MODE 3
  const char* shard[BUFFALO_MAX_SHARDS];
  uint32_t rps;                           // rows per shard
  const int32_t* gidx;                    // global id of each dst row (block 1's src_global)
  __nv_bfloat16* self_out; int64_t ld_self;
};

__device__ __forceinline__ long long shard_row(const GatherEpi& ep, int32_t j, int32_t ldb) {
  const uint32_t u = (uint32_t)j;
  return (long long)(ep.shard[u / ep.rps] + (int64_t)(u % ep.rps) * ldb);
}

template <class TI, int MODE, int LPR, int kU, int MINB, int HINT>
__global__ void __launch_bounds__(256, MINB) k_gather_v2(const int32_t* __restrict__ perm,
                                                         const int32_t* __restrict__ rp,
                                                         const int32_t* __restrict__ col, int32_t n,
                                                         const TI* __restrict__ h, int32_t ldb, int npieces,
                                                         __nv_bfloat16* __restrict__ out, int64_t ldo,
                                                         unsigned long long* __restrict__ edges_dev,
                                                         const GatherEpi ep) {
  pdl_wait();
  constexpr int E = InTraits<TI>::kElems;
  constexpr int G = 32 / LPR;
  constexpr unsigned kFull = 0xffffffffu;
  constexpr bool SH = MODE == 3;                      // sharded feature table
  // HINT bits: 1 = gathered rows evict_last, 2 = per-row side inputs (MODE 2: H, Ys) evict_first,
  // 4 = output rows evict_first
  uint64_t pol_keep = 0, pol_stream = 0;
  if constexpr (HINT & 1) pol_keep = l2_policy_keep();
  if constexpr (HINT & 6) pol_stream = l2_policy_stream();
  auto ld_row = [&](const void* ptr) -> uint4 {
    if constexpr (HINT & 1) return ldg_pol(ptr, pol_keep);
    else return __ldg(reinterpret_cast<const uint4*>(ptr));
  };
  const int lane = threadIdx.x & 31;
  const int g = lane / LPR, pc = lane & (LPR - 1);
  const int gbase = g * LPR;
  const int32_t warps = (int32_t)(gridDim.x * (blockDim.x >> 5));
  int32_t w = (int32_t)((blockIdx.x * blockDim.x + threadIdx.x) >> 5);
  unsigned my_edges = 0;
  // MODE 2: column sums of dZ_{l-1}, one slice per (warp, lane group) [8][G][ncols]
  extern __shared__ float sdb[];
  const int ncols = npieces * E;
  float* my_db = sdb + ((threadIdx.x >> 5) * G + g) * ncols;
  if constexpr (MODE == 2) {
    for (int c = threadIdx.x; c < 8 * G * ncols; c += blockDim.x) sdb[c] = 0.f;
    __syncthreads();
  }
  // row metadata of the first iteration
  int32_t row = -1, b = 0, e = 0;
  {
    const int32_t pos = w * G + g;
    if (pos < n) {
      row = perm ? __ldg(perm + pos) : pos;
      b = __ldg(rp + row);
      e = __ldg(rp + row + 1);
    }
  }
  for (; w * G < n; w += warps) {
    // next iteration's metadata, in flight while this row is gathered
    int32_t row_n = -1, b_n = 0, e_n = 0;
    {
      const int32_t pos = (w + warps) * G + g;
      if (pos < n) {
        row_n = perm ? __ldg(perm + pos) : pos;
        b_n = __ldg(rp + row_n);
        e_n = __ldg(rp + row_n + 1);
      }
    }
    const int32_t D = e - b;
    const int32_t Dl = (row < 0 || D > kHeavyT) ? 0 : D;
    const int32_t Dmax = __reduce_max_sync(kFull, Dl);
    if (edges_dev && pc == 0) my_edges += (unsigned)Dl;
    const bool uni = __reduce_min_sync(kFull, Dl) == Dmax;   // all rows of the warp equally long
    for (int p0 = 0; p0 < npieces; p0 += LPR) {
      const int piece = p0 + pc;
      const bool colok = piece < npieces;
      // lanes past the row read piece 0 again (same sectors, in bounds) and store nothing
      const char* hb = reinterpret_cast<const char*>(h) + (colok ? piece : 0) * 16;
      const int64_t poff = (colok ? piece : 0) * 16;
      // MODE 2: the row's H (ReLU' mask) and Ys pieces are independent of the neighbour sum:
      // issued before it, so their latency overlaps the Yn row loads
      uint4 h_pre = make_uint4(0u, 0u, 0u, 0u), y_pre = make_uint4(0u, 0u, 0u, 0u);
      if constexpr (MODE == 2) {
        if (row >= 0 && D <= kHeavyT && colok) {
          const __nv_bfloat16* hp = ep.H + (int64_t)row * ep.ldH + piece * 8;
          const __nv_bfloat16* yp = ep.ys + (int64_t)row * ep.ldy + piece * 8;
          if constexpr (HINT & 2) {
            h_pre = ldg_pol(hp, pol_stream);
            if (row < ep.n_self) y_pre = ldg_pol(yp, pol_stream);
          } else {
            h_pre = __ldg(reinterpret_cast<const uint4*>(hp));
            if (row < ep.n_self) y_pre = __ldg(reinterpret_cast<const uint4*>(yp));
          }
        }
      }
      float acc[E];
#pragma unroll
      for (int k = 0; k < E; ++k) acc[k] = 0.f;
      for (int32_t base = 0; base < Dmax; base += LPR) {
        const int32_t jj = (base + pc < Dl) ? __ldg(col + b + base + pc) : -1;
        long long ja = -1;                              // MODE 3: the row's address
        if constexpr (SH) {
          if (jj >= 0) ja = shard_row(ep, jj, ldb);
        }
        const int m = min(LPR, Dmax - base);
        int k = 0;
        // full groups of kU edges: no predicates.  Software-pipelined in the forward (the
        // backward's fused epilogue needs the registers): group g + 1's loads are issued before
        // group g is summed, so 2 kU row loads per lane stay in flight
        constexpr bool kPipe = MODE != 2;
        auto ld_group = [&](int k0, uint4 (&raw)[kU]) {
#pragma unroll
            for (int uu = 0; uu < kU; ++uu) {
              if constexpr (SH) {
                const long long an = __shfl_sync(kFull, ja, gbase + k0 + uu);
                raw[uu] = ld_row(reinterpret_cast<const void*>(an + poff));
              } else {
                const int32_t jn = __shfl_sync(kFull, jj, gbase + k0 + uu);
                raw[uu] = ld_row(hb + (int64_t)jn * ldb);
              }
            }
          };
        if (kPipe && uni && m >= kU) {
          uint4 cur[kU];
          ld_group(0, cur);
          for (; k + kU <= m; k += kU) {
            uint4 nxt[kU];
            const bool more = k + 2 * kU <= m;
            if (more) ld_group(k + kU, nxt);
#pragma unroll
            for (int uu = 0; uu < kU; ++uu) acc_piece<TI>(acc, cur[uu]);
            if (more) {
#pragma unroll
              for (int uu = 0; uu < kU; ++uu) cur[uu] = nxt[uu];
            }
          }
        } else if (uni) {
          for (; k + kU <= m; k += kU) {
            uint4 raw[kU];
            ld_group(k, raw);
#pragma unroll
            for (int uu = 0; uu < kU; ++uu) acc_piece<TI>(acc, raw[uu]);
          }
        }
        for (; k < m; k += kU) {                        // ragged rows / tail
          uint4 raw[kU];
          bool ok[kU];
#pragma unroll
          for (int uu = 0; uu < kU; ++uu) {
            if constexpr (SH) {
              const long long an = __shfl_sync(kFull, ja, gbase + ((k + uu) & (LPR - 1)));
              ok[uu] = k + uu < m && an != -1;
              if (ok[uu]) raw[uu] = ld_row(reinterpret_cast<const void*>(an + poff));
            } else {
              const int32_t jn = __shfl_sync(kFull, jj, gbase + ((k + uu) & (LPR - 1)));
              ok[uu] = k + uu < m && jn >= 0;
              if (ok[uu]) raw[uu] = ld_row(hb + (int64_t)jn * ldb);
            }
          }
#pragma unroll
          for (int uu = 0; uu < kU; ++uu)
            if (ok[uu]) acc_piece<TI>(acc, raw[uu]);
        }
      }
      if constexpr (SH) {                               // the dst row's own feature row
        if (row >= 0 && colok) {
          const long long sa = shard_row(ep, __ldg(ep.gidx + row), ldb);
          *reinterpret_cast<uint4*>(ep.self_out + (int64_t)row * ep.ld_self + piece * E) =
              __ldg(reinterpret_cast<const uint4*>(sa + poff));
        }
      }
      if (row >= 0 && D <= kHeavyT && colok) {
        float v[E];
        if ((MODE == 0 || MODE == 3) && D > 0) {
          const float fd = (float)D;
          const float y = 1.0f / fd;                    // once per row
#pragma unroll
          for (int k = 0; k < E; ++k) {
            const float q = acc[k] * y;
            v[k] = fmaf(fmaf(-q, fd, acc[k]), y, q);
          }
        } else {
#pragma unroll
          for (int k = 0; k < E; ++k) v[k] = acc[k];
        }
        if constexpr (MODE == 2) {
          static_assert(E == 8, "the backward epilogue reads bf16 rows");
          if (row < ep.n_self) {
            float y[8];
            bf16x8_to_f32(y_pre, y);
#pragma unroll
            for (int k = 0; k < 8; ++k) v[k] += y[k];
          }
          float hv[8];
          bf16x8_to_f32(h_pre, hv);
#pragma unroll
          for (int k = 0; k < 8; ++k)
            if (!(hv[k] > 0.f) || piece * 8 + k >= ep.d) v[k] = 0.f;
          float4* sd = reinterpret_cast<float4*>(my_db + piece * 8);
          float4 a0 = sd[0], a1 = sd[1];
          a0.x += v[0]; a0.y += v[1]; a0.z += v[2]; a0.w += v[3];
          a1.x += v[4]; a1.y += v[5]; a1.z += v[6]; a1.w += v[7];
          sd[0] = a0;
          sd[1] = a1;
        }
        __nv_bfloat16* dst = out + (int64_t)row * ldo + piece * E;
        if constexpr (E == 8) {
          const uint4 o = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]), pack_bf16x2(v[4], v[5]),
                                     pack_bf16x2(v[6], v[7]));
          if constexpr (HINT & 4) stg_pol(dst, o, pol_stream);
          else *reinterpret_cast<uint4*>(dst) = o;
        } else {
          *reinterpret_cast<uint2*>(dst) = make_uint2(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]));
        }
      }
    }
    row = row_n;
    b = b_n;
    e = e_n;
  }
  if (edges_dev) {                                      // one atomic per warp per launch
    my_edges = __reduce_add_sync(kFull, my_edges);
    if (lane == 0 && my_edges) atomicAdd(edges_dev, (unsigned long long)my_edges);
  }
  if constexpr (MODE == 2) {
    __syncthreads();
    for (int c = threadIdx.x; c < ep.d; c += blockDim.x) {
      float t = 0.f;
      for (int s2 = 0; s2 < 8 * G; ++s2) t += sdb[s2 * ncols + c];
      ep.db_part[(int64_t)blockIdx.x * ep.d + c] = t;
    }
  }
}

// The backward's long-tail kernel runs on a side stream next to the fused Aggregate
constexpr bool kHeavyOverlap = true;
// The layer's dW / db reductions run on a side stream next to its dH products and Aggregate
constexpr bool kDwOverlap = true;

// L2 eviction hints of the forward (MODE 0 / 3) and backward (MODE 2) Aggregate launches
constexpr int kHintFwd = 0, kHintBwd = 7;

template <class TI, int MODE>
static buffalo_status launch_gather(const int32_t* perm, const int32_t* rp, const int32_t* col, int64_t n,
                                    const TI* h, int64_t ldh, int pitch_in, __nv_bfloat16* out, int64_t ldo,
                                    cudaStream_t s) {
  if (n <= 0) return BUFFALO_OK;
  constexpr int E = InTraits<TI>::kElems;
  const int npieces = (pitch_in + E - 1) / E;
  int lpr_log = 0;
  while ((1 << lpr_log) < npieces && lpr_log < 5) ++lpr_log;
  if (n > INT32_MAX || ldh * (int64_t)sizeof(TI) > INT32_MAX) {
    set_error("gather: %lld rows of stride %lld elements exceed the 32-bit row / byte-stride range",
              (long long)n, (long long)ldh);
    return BUFFALO_ERR_INVALID_ARG;
  }
  const ProfSlot ps = prof_begin_launch("gather", s);
  // 2 row loads per lane per step, software-pipelined (4 in flight): 48 registers, 5 CTAs (40
  // warps) per SM — measured faster than 6 CTAs without the pipeline (layer 1: 48.2 -> 45.4 ms of
  // forward per products epoch; the 512-B rows of layers >= 2: a further 1.2 ms)
  constexpr int kU = 2;
  const int kMinB = 5;
  const int fgrid = (int)std::min<int64_t>(ceil_div(ceil_div(n, 32 >> std::max(lpr_log, 2)), 8), 148LL * kMinB * 4);
  const int32_t n32 = (int32_t)n;
  const int32_t ldb = (int32_t)(ldh * (int64_t)sizeof(TI));             // row stride in bytes
#define BF_V2(L) launch_pdl(k_gather_v2<TI, MODE, L, kU, 5, kHintFwd>, dim3(fgrid), dim3(256), 0, s, perm, rp, col, n32, h, ldb, \
                                                                                     npieces, out, ldo, ps.edges_dev, \
                                                                                     GatherEpi{})
  if (lpr_log <= 2) BF_V2(4);
  else if (lpr_log == 3) BF_V2(8);
  else if (lpr_log == 4) BF_V2(16);
  else BF_V2(32);
#undef BF_V2
  BF_LAUNCHED(MODE == 0 ? "k_gather_mean" : "k_gather_sum");
  // algorithmic bytes: per row perm + row_ptr pair + bf16 output row; per edge index + source row
  prof_end_launch(ps, s, (double)n * (12.0 + 2.0 * pitch_in), 4.0 + (double)pitch_in * sizeof(TI));
  return BUFFALO_OK;
}

// MODE 2 (backward, fused epilogue): a fixed grid of kGatherDbCtas CTAs (one db partial row
// each; the heavy-row kernel owns the kHeavyDbCtas rows after them).
constexpr int kGatherDbCtas = 148 * 5, kHeavyDbCtas = 148;
constexpr int kBwdDbParts = kGatherDbCtas + kHeavyDbCtas;

static buffalo_status launch_gather_epi(const int32_t* perm, const int32_t* rp, const int32_t* col, int64_t n,
                                        const __nv_bfloat16* yn, int64_t ldy, int pitch_in, __nv_bfloat16* out,
                                        int64_t ldo, const GatherEpi& ep, cudaStream_t s) {
  const int npieces = (pitch_in + 7) / 8;
  int lpr_log = 0;
  while ((1 << lpr_log) < npieces && lpr_log < 4) ++lpr_log;     // <= 16 lanes per row (short rows)
  lpr_log = std::max(lpr_log, 2);
  if (n > INT32_MAX || ldy * 2 > INT32_MAX) {
    set_error("gather: %lld rows of stride %lld elements exceed the 32-bit row / byte-stride range",
              (long long)n, (long long)ldy);
    return BUFFALO_ERR_INVALID_ARG;
  }
  const ProfSlot ps = prof_begin_launch("gather", s);
  constexpr int kU = 2, kMinB = 5;   // the H / Ys prefetch registers: 5 CTAs (40 warps) per SM
  const int G = 32 >> lpr_log;
  const int smem = 8 * G * npieces * 8 * 4;
  const int32_t n32 = (int32_t)(n > 0 ? n : 0);
  const int32_t ldb = (int32_t)(ldy * 2);
#define BF_V2E(L) launch_pdl(k_gather_v2<__nv_bfloat16, 2, L, kU, kMinB, kHintBwd>, dim3(kGatherDbCtas), dim3(256), \
      (size_t)smem, s, perm, rp, col, n32, yn, ldb, npieces, out, ldo, ps.edges_dev, ep)
  if (lpr_log <= 2) BF_V2E(4);
  else if (lpr_log == 3) BF_V2E(8);
  else BF_V2E(16);
#undef BF_V2E
  BF_LAUNCHED("k_gather_bwd_epi");
  // algorithmic bytes: per row perm + row_ptr pair + the H row + the bf16 dZ row (+ Ys for the
  // dst prefix rows, not counted); per edge index + the Yn row
  prof_end_launch(ps, s, (double)n * (12.0 + 4.0 * pitch_in), 4.0 + (double)pitch_in * 2);
  return BUFFALO_OK;
}

// MODE 3: the layer-1 Aggregate over a sharded feature table (bf16), plus the self-row copy.
static buffalo_status launch_gather_sharded(const buffalo_block* blk, const buffalo_feature_shards* sh, int64_t ld_src,
                                           int pitch_in, __nv_bfloat16* out, int64_t ldo, cudaStream_t s) {
  const int64_t n = blk->n_dst;
  if (n <= 0) return BUFFALO_OK;
  const int npieces = (pitch_in + 7) / 8;
  int lpr_log = 0;
  while ((1 << lpr_log) < npieces && lpr_log < 5) ++lpr_log;
  if (n > INT32_MAX || ld_src * 2 > INT32_MAX) {
    set_error("gather: %lld rows of stride %lld elements exceed the 32-bit row / byte-stride range",
              (long long)n, (long long)ld_src);
    return BUFFALO_ERR_INVALID_ARG;
  }
  GatherEpi ep{};
  for (int k = 0; k < sh->num_shards; ++k) ep.shard[k] = (const char*)sh->shard[k];
  ep.rps = (uint32_t)sh->rows_per_shard;
  ep.gidx = blk->src_global;
  ep.self_out = (__nv_bfloat16*)blk->self_rows;
  ep.ld_self = blk->ld_self;
  const ProfSlot ps = prof_begin_launch("gather", s);
  constexpr int kU = 2;
  const int kMinB = 5;
  const int fgrid = (int)std::min<int64_t>(ceil_div(ceil_div(n, 32 >> std::max(lpr_log, 2)), 8), 148LL * kMinB * 4);
  const int32_t n32 = (int32_t)n, ldb = (int32_t)(ld_src * 2);
  const __nv_bfloat16* h0 = (const __nv_bfloat16*)sh->shard[0];
#define BF_V2S(L) launch_pdl(k_gather_v2<__nv_bfloat16, 3, L, kU, 5, kHintFwd>, dim3(fgrid), dim3(256), 0, s, \
      (const int32_t*)nullptr, blk->row_ptr, blk->col_global, n32, h0, ldb, npieces, out, ldo, ps.edges_dev, ep)
  if (lpr_log <= 2) BF_V2S(4);
  else if (lpr_log == 3) BF_V2S(8);
  else if (lpr_log == 4) BF_V2S(16);
  else BF_V2S(32);
#undef BF_V2S
  BF_LAUNCHED("k_gather_sharded");
  // algorithmic bytes: per row row_ptr pair + id + the self row read and copied + bf16 output
  // row; per edge index + source row
  prof_end_launch(ps, s, (double)n * (12.0 + 6.0 * pitch_in), 4.0 + (double)pitch_in * 2);
  return BUFFALO_OK;
}

// Feature-table rows are addressed through src_global only; the gathered tensor map spans the
// largest row count TMA accepts and tile padding rows gather row 0 (their outputs are dropped).
constexpr int64_t kGatherTableRows = 0x7fffffff;

template <class TI>
static buffalo_status launch_tc_copy(TcFwdParams p, cudaStream_t s) {
  // small A buffers, deep weight prefetch (the weights stream once per tile)
  p.a_chunks = 2;
  const int budget = 220 * 1024 - smem_bytes_for(p.Np, 2, 0);
  p.nb = std::max(2, std::min(8, budget / (p.Np * 128)));
  const int smem = smem_bytes_for(p.Np, p.a_chunks, p.nb);
  BF_CHECK(set_max_smem_once<k_tc_update_copy<TI>>(227 * 1024));
  const int64_t ntiles = ceil_div(p.n_dst, kTileM);
  const int grid = (int)std::min<int64_t>(ntiles, 148);
  k_tc_update_copy<TI><<<grid, kThreads, smem, s>>>(p);
  BF_LAUNCHED("k_tc_update_copy");
  return BUFFALO_OK;
}

static int tmem_cols_for(int Np) {
  int cols = 32;
  while (cols < 2 * Np) cols *= 2;
  return cols;
}

template <class TI>
static buffalo_status tc_fwd_t(const FwdArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  if (blk->n_dst <= 0) return BUFFALO_OK;
  if (a.shards) {
    // sharded feature table (layer 1, sampled block): Aggregate + self-row copy, then the Update
    // over two contiguous bf16 operands
    BF_CHECK(launch_gather_sharded(blk, a.shards, a.ld_src, (int)pitch_of(a.d_in), (__nv_bfloat16*)a.agg, a.ld_agg,
                                   s));
    const uint8_t* wpk = (const uint8_t*)a.W_packed + R((int64_t)2 * a.d_in * a.d_out * 4);
    return tc_gemm_tma(blk->n_dst, blk->n_dst, nullptr, (const __nv_bfloat16*)blk->self_rows, blk->ld_self,
                       (const __nv_bfloat16*)a.agg, a.ld_agg, a.d_in, wpk, a.d_out, a.b, a.relu, a.out_f32, a.out,
                       a.ld_out, s);
  }
  BF_CHECK(launch_agg_heavy_bf16(a, s));
  TcFwdParams p{};
  p.row_ptr = blk->row_ptr;
  p.col = a.layer1 ? blk->col_global : blk->col_local;
  p.gidx = a.layer1 ? blk->src_global : nullptr;
  p.n_dst = blk->n_dst;
  p.self_rows = blk->n_dst;
  p.perm = blk->cls_perm;
  p.h = a.h_src;
  p.ldh = a.ld_src;
  p.hs = a.h_src;
  p.lds = a.ld_src;
  p.d_in = a.d_in;
  p.pitch_in = (int)pitch_of(a.d_in);
  p.nkc_self = (int)ceil_div(a.d_in, kKC);
  p.nkc = 2 * p.nkc_self;
  p.wpk = (const uint8_t*)a.W_packed + R((int64_t)2 * a.d_in * a.d_out * 4);
  p.Np = (int)round_up(a.d_out, 16);
  p.d_out = a.d_out;
  p.ld_out = (int)a.ld_out;
  p.tmem_cols = tmem_cols_for(p.Np);
  p.bias = a.b;
  p.relu = a.relu;
  p.out_f32 = a.out_f32;
  p.out = a.out;
  p.agg = (__nv_bfloat16*)a.agg;
  p.ld_agg = a.ld_agg;
  // high-occupancy gather of the non-heavy rows, then the Update GEMM over copies
  // sampled blocks (no row past the fanout): rows in natural order; else the degree-class order
  const int32_t* order = (blk->fanout > 0 && blk->fanout <= kHeavyT) ? nullptr : blk->cls_perm;
  BF_CHECK((launch_gather<TI, 0>(order, blk->row_ptr, p.col, blk->n_dst, (const TI*)a.h_src, a.ld_src,
                                 p.pitch_in, (__nv_bfloat16*)a.agg, a.ld_agg, s)));
  if (a.in_bf16)
    return tc_gemm_tma(blk->n_dst, a.layer1 ? kGatherTableRows : blk->n_dst, a.layer1 ? blk->src_global : nullptr,
                       (const __nv_bfloat16*)a.h_src, a.ld_src, (const __nv_bfloat16*)a.agg, a.ld_agg,
                       a.d_in, p.wpk, a.d_out, a.b, a.relu, a.out_f32, a.out, a.ld_out, s);
  p.perm = nullptr;
  p.agg_src = (const __nv_bfloat16*)a.agg;
  p.ld_agg_src = a.ld_agg;
  return launch_tc_copy<TI>(p, s);
}

buffalo_status tc_sage_fwd(const FwdArgs& a, cudaStream_t s) {
  if (a.in_bf16) return tc_fwd_t<__nv_bfloat16>(a, s);
  return tc_fwd_t<float>(a, s);
}

// ================================================================== backward
// dZ preparation: dZ = dH * 1[H > 0] in place (l < L); bf16 copies of dZ and dZ / D(i); and
// the column sums of dZ (db) as per-CTA partials over a fixed row split (deterministic).
constexpr int kDbSplits = 296;

template <class TH>
__global__ void __launch_bounds__(256) k_dz_prep(float* __restrict__ dz, int64_t ldz, const TH* __restrict__ h,
                                                 int64_t ldh, const int32_t* __restrict__ rp, int64_t n, int d,
                                                 int dp, __nv_bfloat16* __restrict__ zb,
                                                 __nv_bfloat16* __restrict__ zs, float* __restrict__ db_part) {
  __shared__ float red[256][9];
  const int per_row = dp / 8;                       // <= 32 column groups of 8
  const int rows_per_pass = 256 / per_row;
  const int cg = threadIdx.x % per_row, rsub = threadIdx.x / per_row;
  const int64_t rows_per_cta = (n + gridDim.x - 1) / gridDim.x;
  const int64_t r_beg = (int64_t)blockIdx.x * rows_per_cta, r_end = min(n, r_beg + rows_per_cta);
  float db[8] = {0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f, 0.f};
  const bool active = rsub < rows_per_pass;
  for (int64_t i = r_beg + rsub; active && i < r_end; i += rows_per_pass) {
    const int c0 = cg * 8;
    float v[8];
    const float4 a0 = *reinterpret_cast<const float4*>(dz + i * ldz + c0);
    const float4 a1 = *reinterpret_cast<const float4*>(dz + i * ldz + c0 + 4);
    v[0] = a0.x; v[1] = a0.y; v[2] = a0.z; v[3] = a0.w; v[4] = a1.x; v[5] = a1.y; v[6] = a1.z; v[7] = a1.w;
    if (h) {
      const uint4 hr = *reinterpret_cast<const uint4*>(reinterpret_cast<const __nv_bfloat16*>(h) + i * ldh + c0);
      float hv[8];
      bf16x8_to_f32(hr, hv);
      bool ch = false;
#pragma unroll
      for (int k = 0; k < 8; ++k)
        if (!(hv[k] > 0.f) && v[k] != 0.f) { v[k] = 0.f; ch = true; }
      if (ch) {
        *reinterpret_cast<float4*>(dz + i * ldz + c0) = make_float4(v[0], v[1], v[2], v[3]);
        *reinterpret_cast<float4*>(dz + i * ldz + c0 + 4) = make_float4(v[4], v[5], v[6], v[7]);
      }
    }
#pragma unroll
    for (int k = 0; k < 8; ++k) {
      if (c0 + k >= d) v[k] = 0.f;
      db[k] += v[k];
    }
    *reinterpret_cast<uint4*>(zb + i * dp + c0) = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]),
                                                              pack_bf16x2(v[4], v[5]), pack_bf16x2(v[6], v[7]));
    if (zs) {
      const float fd = (float)(rp[i + 1] - rp[i]);
#pragma unroll
      for (int k = 0; k < 8; ++k) v[k] = v[k] / fd;
      *reinterpret_cast<uint4*>(zs + i * dp + c0) = make_uint4(pack_bf16x2(v[0], v[1]), pack_bf16x2(v[2], v[3]),
                                                                pack_bf16x2(v[4], v[5]), pack_bf16x2(v[6], v[7]));
    }
  }
#pragma unroll
  for (int k = 0; k < 8; ++k) red[threadIdx.x][k] = db[k];
  __syncthreads();
  if (threadIdx.x < per_row) {
    for (int k = 0; k < 8; ++k) {
      float t = 0.f;
      for (int r = 0; r < rows_per_pass; ++r) t += red[r * per_row + threadIdx.x][k];
      const int c = threadIdx.x * 8 + k;
      if (c < d) db_part[(int64_t)blockIdx.x * d + c] = t;
    }
  }
}

// dW (tensor cores): D[m][n'] = sum_r dZ[r][m] * Afwd[r][n'] over a row range, both operands
// MN-major in shared memory (the reduction runs over rows, the slow dimension of both).
// Afwd columns are padded per half: n' < Dp -> self column n', n' >= Dp -> h_agg column n' - Dp.
constexpr int kDwThreads = 256;
constexpr int kDwRows = 64;                       // K per stage
constexpr int kDwStrip = kDwRows * 128;           // one 64-column MN strip of 64 rows (8 KB)
constexpr int kDwStages = 3;

struct TcDwParams {
  const __nv_bfloat16* zb;  int64_t ldz;          // dZ (bf16) [n][ldz]
  const void* self_; int64_t lds; const int32_t* gidx;  // self rows (feature table for layer 1)
  const __nv_bfloat16* agg; int64_t lda;          // saved h_agg
  int64_t n;
  int d_out, d_in, pitch_in, pz, Dp, NT, MT;      // NT: n' columns per CTA (<= 256); MT: m-tiles (<= 2)
  int64_t rows_per_split;
  float* part;                                    // [S][d_out][2 Dp]
};

// MN-major SWIZZLE_128B descriptor: LBO = stride between 64-element MN strips, SBO = 8 K-rows.
__device__ __forceinline__ uint64_t sw128_mn_desc(uint32_t saddr, uint32_t lbo) {
  uint64_t d = 0;
  d |= (uint64_t)((saddr >> 4) & 0x3FFF);
  d |= (uint64_t)((lbo >> 4) & 0x3FFF) << 16;
  d |= (uint64_t)(1024 >> 4) << 32;
  d |= (uint64_t)1 << 46;
  d |= (uint64_t)2 << 61;
  return d;
}
__host__ __device__ constexpr uint32_t idesc_bf16_mn(int n) {
  return (1u << 4) | (1u << 7) | (1u << 10) | (1u << 15) | (1u << 16) | ((uint32_t)(n >> 3) << 17) |
         ((uint32_t)(128 >> 4) << 24);
}

// One CTA: all m-tiles of d_out (each 128 TMEM lanes x NT columns) for one n'-tile, over a row
// split; both operands are read once.  3-stage cp.async pipeline, single-thread MMA issue.
template <class TS>
__global__ void __launch_bounds__(kDwThreads) k_tc_dw(const TcDwParams p) {
  extern __shared__ __align__(1024) uint8_t smem_raw[];
  uint8_t* smem = (uint8_t*)(((uintptr_t)smem_raw + 1023) & ~(uintptr_t)1023);
  const int nstripA = 2 * p.MT, nstripB = p.NT / 64;
  const int stage_bytes = (nstripA + nstripB) * kDwStrip;
  uint64_t* full = (uint64_t*)(smem + kDwStages * stage_bytes);
  uint64_t* empty = full + kDwStages;
  uint64_t* done = empty + kDwStages;
  uint32_t* tmem_slot = (uint32_t*)(done + 1);
  const int warp = threadIdx.x >> 5;
  const int n0 = blockIdx.x * p.NT;
  const int64_t r_beg = (int64_t)blockIdx.y * p.rows_per_split;
  const int64_t r_end = min(p.n, r_beg + p.rows_per_split);
  const int nchunks = r_end > r_beg ? (int)((r_end - r_beg + kDwRows - 1) / kDwRows) : 0;
  int tcols = 32;
  while (tcols < p.MT * p.NT) tcols <<= 1;
  if (threadIdx.x == 0) {
    for (int i = 0; i < kDwStages; ++i) { mbar_init(&full[i], kDwThreads); mbar_init(&empty[i], 1); }
    mbar_init(done, 1);
    fence_barrier_init();
  }
  if (warp == 0) tmem_alloc(tmem_slot, tcols);
  tc_fence_before();
  __syncthreads();
  tc_fence_after();
  const uint32_t tmem = *tmem_slot;
  const TS* __restrict__ selfp = (const TS*)p.self_;
  const uint32_t idesc = idesc_bf16_mn(p.NT);
  const void* dummy = p.zb;            // any global address: zero-fill copies read 0 bytes
  const int apcs = p.MT * 16;          // 16-B pieces of a dZ row slice (128 columns per m-tile)
  const int bpcs = p.NT / 8;

  auto load_chunk = [&](int c) {
    const int st = c % kDwStages;
    uint8_t* sa = smem + st * stage_bytes;
    uint8_t* sb = sa + nstripA * kDwStrip;
    const int64_t rbase = r_beg + (int64_t)c * kDwRows;
    for (int u = threadIdx.x; u < kDwRows * apcs; u += kDwThreads) {
      const int k = u / apcs, j = u % apcs;
      const int64_t r = rbase + k;
      const int m = j * 8;
      const bool ok = r < r_end && m < p.pz;
      cp_async16(sa + (j >> 3) * kDwStrip + k * 128 + (((j & 7) ^ (k & 7)) << 4),
                 ok ? (const void*)(p.zb + r * p.ldz + m) : dummy, ok);
    }
    for (int u = threadIdx.x; u < kDwRows * bpcs; u += kDwThreads) {
      const int k = u / bpcs, j = u % bpcs;
      const int64_t r = rbase + k;
      const int nn = n0 + j * 8;
      uint8_t* dst = sb + (j >> 3) * kDwStrip + k * 128 + (((j & 7) ^ (k & 7)) << 4);
      if constexpr (sizeof(TS) == 2) {
        const void* src = dummy;
        bool ok = false;
        if (r < r_end) {
          if (nn < p.Dp) {
            if (nn < p.pitch_in) {
              const int64_t rr = p.gidx ? (int64_t)p.gidx[r] : r;
              src = selfp + rr * p.lds + nn;
              ok = true;
            }
          } else if (nn - p.Dp < p.pitch_in) {
            src = p.agg + r * p.lda + (nn - p.Dp);
            ok = true;
          }
        }
        cp_async16(dst, src, ok);
      } else {
        uint4 v = make_uint4(0u, 0u, 0u, 0u);
        if (r < r_end) {
          if (nn < p.Dp) {
            if (nn < p.pitch_in) {
              const int64_t rr = p.gidx ? (int64_t)p.gidx[r] : r;
              const float4 a0 = *reinterpret_cast<const float4*>(selfp + rr * p.lds + nn);
              const float4 a1 = *reinterpret_cast<const float4*>(selfp + rr * p.lds + nn + 4);
              v = make_uint4(pack_bf16x2(a0.x, a0.y), pack_bf16x2(a0.z, a0.w), pack_bf16x2(a1.x, a1.y),
                             pack_bf16x2(a1.z, a1.w));
            }
          } else if (nn - p.Dp < p.pitch_in) {
            v = *reinterpret_cast<const uint4*>(p.agg + r * p.lda + (nn - p.Dp));
          }
        }
        *reinterpret_cast<uint4*>(dst) = v;
      }
    }
    cp_async_commit();
  };
  auto mma_chunk = [&](int c) {
    const int st = c % kDwStages;
    mbar_wait(&full[st], (uint32_t)((c / kDwStages) & 1));
    tc_fence_after();
    const uint32_t a_addr = smem_u32(smem + st * stage_bytes);
    const uint32_t b_addr = a_addr + nstripA * kDwStrip;
    for (int mt = 0; mt < p.MT; ++mt)
#pragma unroll
      for (int kk = 0; kk < kDwRows / 16; ++kk)
        umma_bf16(tmem + mt * p.NT, sw128_mn_desc(a_addr + mt * 2 * kDwStrip + kk * 2048, kDwStrip),
                  sw128_mn_desc(b_addr + kk * 2048, kDwStrip), idesc, (c > 0 || kk > 0) ? 1u : 0u);
    umma_commit(&empty[st]);
    if (c == nchunks - 1) umma_commit(done);
  };
  // pipeline: chunk c's copies are in flight while chunk c-1 is completed, fenced and issued
  for (int c = 0; c < nchunks; ++c) {
    if (c >= kDwStages) mbar_wait(&empty[c % kDwStages], (uint32_t)(((c / kDwStages) - 1) & 1));
    load_chunk(c);
    if (c >= 1) {
      cp_async_wait<1>();
      fence_proxy_async_smem();
      mbar_arrive(&full[(c - 1) % kDwStages]);
      if (threadIdx.x == 0) mma_chunk(c - 1);
      __syncwarp();
    }
  }
  if (nchunks > 0) {
    cp_async_wait<0>();
    fence_proxy_async_smem();
    mbar_arrive(&full[(nchunks - 1) % kDwStages]);
    if (threadIdx.x == 0) mma_chunk(nchunks - 1);
    __syncwarp();
  }
  // epilogue: warp w reads TMEM lane quadrant w % 4 of m-tile w / 4
  const int lane = threadIdx.x & 31;
  const int quad = warp & 3, mt = warp >> 2;
  const int64_t K2 = 2 * (int64_t)p.Dp;
  float* P = p.part + (int64_t)blockIdx.y * p.d_out * K2;
  const int m = mt * 128 + quad * 32 + lane;
  if (nchunks > 0) {
    mbar_wait(done, 0);
    tc_fence_after();
  }
  if (mt < p.MT) {
    for (int g = 0; g < p.NT / 8; ++g) {
      float v[8];
      if (nchunks > 0) {
        tmem_ld8(tmem + ((uint32_t)(quad * 32) << 16) + mt * p.NT + g * 8, v);
      } else {
#pragma unroll
        for (int k = 0; k < 8; ++k) v[k] = 0.f;
      }
      const int nn = n0 + g * 8;
      if (m < p.d_out && nn < K2) {
        float4* o = reinterpret_cast<float4*>(P + (int64_t)m * K2 + nn);
        o[0] = make_float4(v[0], v[1], v[2], v[3]);
        o[1] = make_float4(v[4], v[5], v[6], v[7]);
      }
    }
  }
  tc_fence_before();
  __syncthreads();
  if (warp == 0) {
    tc_fence_after();
    tmem_dealloc(tmem, tcols);
  }
}

// dW[m][n] += sum_s part[s][m][n'(n)] in split order (deterministic).
__global__ void k_reduce_dw(const float* __restrict__ part, int S, int d_out, int d_in, int Dp,
                            float* __restrict__ dW) {
  // thread per dW element, the S partials summed in split order (coalesced over the columns;
  // a float4-per-thread variant had 4x fewer loads in flight and measured slower)
  const int64_t total = (int64_t)d_out * 2 * d_in;
  const int64_t K2 = 2 * (int64_t)Dp;
  for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < total; t += (int64_t)gridDim.x * blockDim.x) {
    const int m = (int)(t / (2 * d_in)), n = (int)(t % (2 * d_in));
    const int np = n < d_in ? n : Dp + (n - d_in);
    float acc = 0.f;
    for (int q = 0; q < S; ++q) acc += part[(int64_t)q * d_out * K2 + (int64_t)m * K2 + np];
    dW[t] += acc;
  }
}

// db += sum of the S partial rows: CTA per 32 columns, warp w of 32 sums partials w, w + 32, ...
// and the 32 warp sums are combined in warp order (fixed order: deterministic).
__global__ void __launch_bounds__(1024) k_reduce_db(const float* __restrict__ part, int S, int d,
                                                    float* __restrict__ db) {
  __shared__ float sh[32][33];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int c = blockIdx.x * 32 + lane;
  float s = 0.f;
  if (c < d) {
#pragma unroll 4
    for (int q = w; q < S; q += 32) s += __ldg(part + (int64_t)q * d + c);
  }
  sh[w][lane] = s;
  __syncthreads();
  if (w == 0 && c < d) {
    float t = 0.f;
    for (int k = 0; k < 32; ++k) t += sh[k][lane];
    db[c] += t;
  }
}


// The backward's long-tail transposed rows (more than kHeavyT dst) with the fused epilogue of
// GatherEpi: 8 warps over the row's entries (warp w takes t = w, w+8, ...), combined in warp
// order (the split depends only on the row: deterministic), then + Ys[j] (j <
// n_self), ReLU' with H[j], bf16 dZ_{l-1}[j], and the column sums of this CTA's heavy rows (in
// row order) as db partial row kGatherDbCtas + blockIdx.x.  A fixed grid of kHeavyDbCtas CTAs:
// CTAs without heavy rows write zero partials.
__global__ void __launch_bounds__(256) k_heavy_bwd_epi(const int32_t* __restrict__ perm, int64_t n,
                                                       const int32_t* __restrict__ rp,
                                                       const int32_t* __restrict__ col,
                                                       const __nv_bfloat16* __restrict__ z, int64_t ldz, int dp,
                                                       __nv_bfloat16* __restrict__ out, int64_t ldo,
                                                       const GatherEpi ep, int part_row0) {
  __shared__ float part[8][32][8];
  __shared__ float sdb[256];
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  const int nch = dp / 8;                        // <= 32 pieces (d <= 256)
  for (int c = threadIdx.x; c < 256; c += blockDim.x) sdb[c] = 0.f;
  __syncthreads();
  for (int64_t hh = blockIdx.x; hh < n; hh += gridDim.x) {
    const int64_t j = perm[n - 1 - hh];          // heavy rows: the tail of the degree-class perm
    const int32_t b = rp[j], e_end = rp[j + 1];
    if (e_end - b <= kHeavyT) break;
    const int c = lane;
    float acc[8];
#pragma unroll
    for (int k = 0; k < 8; ++k) acc[k] = 0.f;
    if (c < nch) {
      int32_t t = b + w;
      for (; t + 24 < e_end; t += 32) {
        uint4 r[4];
#pragma unroll
        for (int u = 0; u < 4; ++u) r[u] = __ldg(reinterpret_cast<const uint4*>(z + (int64_t)col[t + 8 * u] * ldz + c * 8));
#pragma unroll
        for (int u = 0; u < 4; ++u) acc_piece<__nv_bfloat16>(acc, r[u]);
      }
      for (; t < e_end; t += 8)
        acc_piece<__nv_bfloat16>(acc, __ldg(reinterpret_cast<const uint4*>(z + (int64_t)col[t] * ldz + c * 8)));
    }
#pragma unroll
    for (int k = 0; k < 8; ++k) part[w][lane][k] = acc[k];
    __syncthreads();
    if (w == 0 && c < nch) {
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        float s2 = part[0][lane][k];
        for (int ww = 1; ww < 8; ++ww) s2 += part[ww][lane][k];
        acc[k] = s2;
      }
      if (j < ep.n_self) {
        float y[8];
        bf16x8_to_f32(__ldg(reinterpret_cast<const uint4*>(ep.ys + j * ep.ldy + c * 8)), y);
#pragma unroll
        for (int k = 0; k < 8; ++k) acc[k] += y[k];
      }
      float hv[8];
      bf16x8_to_f32(__ldg(reinterpret_cast<const uint4*>(ep.H + j * ep.ldH + c * 8)), hv);
#pragma unroll
      for (int k = 0; k < 8; ++k) {
        if (!(hv[k] > 0.f) || c * 8 + k >= ep.d) acc[k] = 0.f;
        sdb[c * 8 + k] += acc[k];
      }
      *reinterpret_cast<uint4*>(out + j * ldo + c * 8) =
          make_uint4(pack_bf16x2(acc[0], acc[1]), pack_bf16x2(acc[2], acc[3]), pack_bf16x2(acc[4], acc[5]),
                     pack_bf16x2(acc[6], acc[7]));
    }
    __syncthreads();
  }
  __syncthreads();
  for (int c = threadIdx.x; c < ep.d; c += blockDim.x)
    ep.db_part[(int64_t)(part_row0 + blockIdx.x) * ep.d + c] = sdb[c];
}

int tc_dw_splits(int64_t n, int d_out, int d_in) {
  (void)d_out;
  const int64_t Dp = round_up(d_in, 64);
  const int64_t tiles = ceil_div(2 * Dp, 256);
  int64_t sp = std::min<int64_t>(ceil_div(148, tiles), ceil_div(n > 0 ? n : 1, 512));
  return (int)std::max<int64_t>(1, sp);
}

int64_t tc_bwd_db_parts() { return kBwdDbParts; }

int64_t tc_bwd_scratch_bytes(int64_t n_dst, int64_t n_src, int64_t e, int layer, int d_in, int d_out, bool last) {
  (void)e;
  (void)n_src;
  const int S = tc_dw_splits(n_dst, d_out, d_in);
  const int64_t Dp = round_up(d_in, 64);
  int64_t b = 0;
  if (last) b += R(n_dst * pitch_of(d_out) * 2);                    // dZ bf16
  if (layer >= 2) b += 2 * R(n_dst * pitch_of(d_in) * 2);           // Ys = dZ W_self, Yn = dZ W_neigh / D (bf16)
  b += R((int64_t)S * d_out * 2 * Dp * 4);                          // dW partials
  if (last) b += R((int64_t)kDbSplits * d_out * 4);                 // db partials (dz_prep)
  return b;
}

bool tc_bwd_supported(const BwdArgs& a) {
  return a.act_bf16 && round_up(a.d_out, 16) <= 256 && (a.layer1 || round_up(a.d_in, 16) <= 256);
}

buffalo_status tc_sage_bwd(const BwdArgs& a, cudaStream_t s) {
  const buffalo_block* blk = a.blk;
  const int64_t n = blk->n_dst;
  const int d_in = a.d_in, d_out = a.d_out;
  const int dp = (int)pitch_of(d_out);
  const int dpp = (int)pitch_of(d_in);
  const int S = tc_dw_splits(n, d_out, d_in);
  const int64_t Dp = round_up(d_in, 64);
  // prepared input of this layer: bf16 dZ and db partials
  __nv_bfloat16* zb;
  float* db_part;
  int nparts;
  char* q = (char*)a.scratch;
  if (a.last) {
    zb = (__nv_bfloat16*)q; q += R(n * dp * 2);
  } else {
    zb = (__nv_bfloat16*)a.dh;
  }
  __nv_bfloat16 *ys = nullptr, *yn = nullptr;
  if (a.dh_src) {
    ys = (__nv_bfloat16*)q; q += R(n * dpp * 2);
    yn = (__nv_bfloat16*)q; q += R(n * dpp * 2);
  }
  float* dw_part = (float*)q; q += R((int64_t)S * d_out * 2 * Dp * 4);
  if (a.last) {
    db_part = (float*)q;
    nparts = kDbSplits;
  } else {
    db_part = (float*)((char*)a.dh + R(n * dp * 2));
    nparts = kBwdDbParts;
  }
  if (n <= 0) return BUFFALO_OK;
  if (a.last) {
    k_dz_prep<__nv_bfloat16><<<kDbSplits, 256, 0, s>>>(a.dh, a.ld_dh, nullptr, 0, blk->row_ptr, n, d_out, dp, zb,
                                                       nullptr, db_part);
    BF_LAUNCHED("k_dz_prep");
  }
  // dW (TMA-fed tensor cores, deterministic split reduction) and db: on side stream 1 when the
  // layer also has the dH products and the transposed Aggregate to run (independent work: both
  // only read dZ), joined before returning
  SideFork dwf(s, 1, kDwOverlap && a.dh_src != nullptr);
  {
  cudaStream_t s = dwf.stream();
  if (a.shards) {            // layer 1 of a sharded table: the self rows were copied by the forward
    BF_CHECK(tc_dw_tma(n, S, zb, dp, d_out, (const __nv_bfloat16*)blk->self_rows, blk->ld_self, nullptr, n,
                       (const __nv_bfloat16*)a.agg, a.ld_agg, d_in, dw_part, s));
  } else if (a.in_bf16) {
    BF_CHECK(tc_dw_tma(n, S, zb, dp, d_out, (const __nv_bfloat16*)a.h_src, a.ld_src,
                       a.layer1 ? blk->src_global : nullptr, kGatherTableRows, (const __nv_bfloat16*)a.agg,
                       a.ld_agg, d_in, dw_part, s));
  } else {
    TcDwParams w{};
    w.zb = zb; w.ldz = dp;
    w.self_ = a.h_src; w.lds = a.ld_src; w.gidx = a.layer1 ? blk->src_global : nullptr;
    w.agg = (const __nv_bfloat16*)a.agg; w.lda = a.ld_agg;
    w.n = n; w.d_out = d_out; w.d_in = d_in; w.pitch_in = (int)pitch_of(d_in); w.pz = dp; w.Dp = (int)Dp;
    w.NT = (int)std::min<int64_t>(256, 2 * Dp);
    w.MT = (int)ceil_div(d_out, 128);
    w.rows_per_split = ceil_div(n, S);
    w.part = dw_part;
    const int smem = kDwStages * (2 * w.MT + w.NT / 64) * kDwStrip + 128 + 1024;
    dim3 grid((unsigned)ceil_div(2 * Dp, w.NT), (unsigned)S);
    constexpr int kMaxDwSmem = kDwStages * (4 + 4) * kDwStrip + 128 + 1024;
    BF_CHECK(set_max_smem_once<k_tc_dw<float>>(kMaxDwSmem));
    k_tc_dw<float><<<grid, kDwThreads, smem, s>>>(w);
    BF_LAUNCHED("k_tc_dw");
  }
  k_reduce_dw<<<grid_for((int64_t)d_out * 2 * d_in, 256), 256, 0, s>>>(dw_part, S, d_out, d_in, (int)Dp, a.dW);
  BF_LAUNCHED("k_reduce_dw");
  k_reduce_db<<<(unsigned)ceil_div(d_out, 32), 1024, 0, s>>>(db_part, nparts, d_out, a.db);
  BF_LAUNCHED("k_reduce_db");
  }
  // dH_{l-1}[j] = [j < n_dst] (dZ W_self)[j] + sum_{i in T(j)} (dZ W_neigh)[i] / D(i): the two
  // products over the n_dst rows first (tcgen05, the 1/D row scale in the epilogue), then the
  // transposed Aggregate over the n_src rows with the layer-below epilogue fused (+ Ys, ReLU'
  // with H_{l-1}, bf16 dZ_{l-1}, db_{l-1} partials) — no n_src x d intermediate.
  if (a.dh_src) {
    const uint8_t* wpk = (const uint8_t*)a.W_packed + R((int64_t)2 * d_in * d_out * 4) + tc_fwd_packed_bytes(d_in, d_out);
    const int64_t wchunk = round_up(d_in, 16) * 128;              // one packed K-chunk (Np rows x 128 B)
    const int nkc = (int)ceil_div(d_out, kKC);
    BF_CHECK(tc_gemm_tma(n, n, nullptr, zb, dp, nullptr, 0, d_out, wpk, d_in, nullptr, 0, 0, ys, dpp, s));
    BF_CHECK(tc_gemm_tma(n, n, nullptr, zb, dp, nullptr, 0, d_out, wpk + nkc * wchunk, d_in, nullptr, 0, 0, yn, dpp,
                         s, blk->row_ptr));
    const int64_t ns = blk->n_src;
    GatherEpi ep{};
    ep.ys = ys;
    ep.ldy = dpp;
    ep.n_self = n;
    ep.H = (const __nv_bfloat16*)a.h_src;
    ep.ldH = a.ld_src;
    ep.d = d_in;
    ep.db_part = (float*)((char*)a.dh_src + R(ns * dpp * 2));
    __nv_bfloat16* zprev = (__nv_bfloat16*)a.dh_src;
    // the long-tail rows (a CTA each: hub src rows with thousands of entries) on side stream 0, so
    // their tail overlaps the regular rows' gather (disjoint dZ rows and db partial rows)
    SideFork hv(s, 0, kHeavyOverlap);
    k_heavy_bwd_epi<<<kHeavyDbCtas, 256, 0, hv.stream()>>>(blk->t_perm, ns, blk->t_row_ptr, blk->t_col, yn, dpp, dpp,
                                                            zprev, dpp, ep, kGatherDbCtas);
    BF_LAUNCHED("k_heavy_bwd_epi");
    BF_CHECK(launch_gather_epi(blk->t_perm, blk->t_row_ptr, blk->t_col, ns, yn, dpp, dpp, zprev, dpp, ep, s));
    if (!hv.join() || !dwf.join()) {
      set_error("sage_bwd: side-stream join failed");
      return BUFFALO_ERR_CUDA;
    }
  }
  return BUFFALO_OK;
}

}  // namespace buffalo
