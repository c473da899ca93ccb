# A/B: forward Aggregate with 3 row loads per lane per group (6 in flight) at 4 CTAs per SM
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
i = s.index("static buffalo_status launch_gather(")
j = s.index("BF_LAUNCHED(MODE == 0 ? \"k_gather_mean\" : \"k_gather_sum\");")
seg = s[i:j]
seg2 = seg.replace("constexpr int kU = 2;", "constexpr int kU = 3;").replace("const int kMinB = 5;", "const int kMinB = 4;")
seg2 = seg2.replace("k_gather_v2<TI, MODE, L, kU, 5, kHintFwd>", "k_gather_v2<TI, MODE, L, kU, 4, kHintFwd>")
assert seg2 != seg
s = s[:i] + seg2 + s[j:]
open(p, "w").write(s)
