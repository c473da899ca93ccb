// philox.cuh — Philox4x32-10 (Salmon, Moraes, Dror, Shaw, SC'11) for the CUDA path.
// Independent of oracle/buffalo_oracle.c and synth/philox.py; all three are pinned to the
// Random123 known-answer vectors (tests/golden/philox_kat.txt).
#pragma once
#include <stdint.h>

namespace buffalo {

struct u32x4 { uint32_t x, y, z, w; };

__host__ __device__ __forceinline__ u32x4 philox4x32_10(u32x4 c, uint32_t k0, uint32_t k1) {
#pragma unroll
  for (int r = 0; r < 10; ++r) {
    if (r) { k0 += 0x9E3779B9u; k1 += 0xBB67AE85u; }
#ifdef __CUDA_ARCH__
    const uint32_t lo0 = 0xD2511F53u * c.x, hi0 = __umulhi(0xD2511F53u, c.x);
    const uint32_t lo1 = 0xCD9E8D57u * c.z, hi1 = __umulhi(0xCD9E8D57u, c.z);
#else
    const uint64_t p0 = (uint64_t)0xD2511F53u * c.x, p1 = (uint64_t)0xCD9E8D57u * c.z;
    const uint32_t lo0 = (uint32_t)p0, hi0 = (uint32_t)(p0 >> 32);
    const uint32_t lo1 = (uint32_t)p1, hi1 = (uint32_t)(p1 >> 32);
#endif
    c = u32x4{hi1 ^ c.y ^ k0, lo1, hi0 ^ c.w ^ k1, lo0};
  }
  return c;
}

// Stream tags.
constexpr uint32_t kTagSample = 0;

// Draw t of node v's sampling stream at hop h: word (t & 3) of
// Philox(key = seed; ctr = (v, h, t >> 2, tag 0)).
__device__ __forceinline__ uint32_t sample_draw(uint64_t seed, uint32_t v, uint32_t hop, uint32_t t) {
  u32x4 o = philox4x32_10(u32x4{v, hop, t >> 2, kTagSample}, (uint32_t)seed, (uint32_t)(seed >> 32));
  const uint32_t w[4] = {o.x, o.y, o.z, o.w};
  return w[t & 3];
}

}  // namespace buffalo
