# A/B: the layer's dW / db reductions back on the caller's stream
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
a = "constexpr bool kDwOverlap = true;"
assert a in s
s = s.replace(a, "constexpr bool kDwOverlap = false;")
open(p, "w").write(s)
