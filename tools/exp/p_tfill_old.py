# A/B: k_tfill one row per warp iteration (before the kR unroll)
import sys
p = sys.argv[1] + "/build.cu"
s = open(p).read()
a = s[s.index("  // kR rows per warp and iteration: their first 32 entries' cursor atomics"):s.index("// Ascending sort of the transposed rows")]
s = s.replace(a, """  const int lane = threadIdx.x & 31;
  const int64_t warps = (int64_t)gridDim.x * (blockDim.x >> 5);
  for (int64_t i = (blockIdx.x * (int64_t)blockDim.x + threadIdx.x) >> 5; i < n; i += warps)
    for (int32_t k = rp[i] + lane; k < rp[i + 1]; k += 32) tcol[atomicAdd(&cursor[col_local[k]], 1)] = (int32_t)i;
}
""")
open(p, "w").write(s)
