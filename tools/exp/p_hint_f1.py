# A/B: L2 eviction hint bits of the Aggregate (forward 1, backward 7)
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
a = "constexpr int kHintFwd = 0, kHintBwd = 7;"
assert a in s
s = s.replace(a, "constexpr int kHintFwd = 1, kHintBwd = 7;")
open(p, "w").write(s)
