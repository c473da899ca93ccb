# A/B: L2 eviction hint bits of the Aggregate (forward 0, backward 1)
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
a = "constexpr int kHintFwd = 0, kHintBwd = 7;"
assert a in s
s = s.replace(a, "constexpr int kHintFwd = 0, kHintBwd = 1;")
open(p, "w").write(s)
