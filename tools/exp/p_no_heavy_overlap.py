# A/B: the backward's long-tail kernel back on the caller's stream
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
a = "constexpr bool kHeavyOverlap = true;"
assert a in s
s = s.replace(a, "constexpr bool kHeavyOverlap = false;")
open(p, "w").write(s)
