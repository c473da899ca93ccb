# A/B: the forward Aggregate's pipeline for equal-length warps only (unpredicated)
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
a = "constexpr bool kPipeRagged = true;"
assert a in s
s = s.replace(a, "constexpr bool kPipeRagged = false;")
open(p, "w").write(s)
