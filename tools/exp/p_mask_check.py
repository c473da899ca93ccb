# A/B: scheduler mask propagation skips the atomicOr when the target word already holds the bits
import sys
p = sys.argv[1] + "/build.cu"
s = open(p).read()
a = "    if (mask[w]) atomicOr(&m_out[(int64_t)u * W + w], mask[w]);"
assert a in s
s = s.replace(a, """    if (mask[w]) {
      unsigned long long* t = &m_out[(int64_t)u * W + w];
      if ((__ldcg(t) & mask[w]) != mask[w]) atomicOr(t, mask[w]);
    }""")
open(p, "w").write(s)
