# A/B: forward Aggregate at 4 CTAs per SM (64 registers)
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
s = s.replace("k_gather_v2<TI, MODE, L, kU, 5>", "k_gather_v2<TI, MODE, L, kU, 4>")
s = s.replace("  const int kMinB = 5;\n  const int fgrid", "  const int kMinB = 4;\n  const int fgrid", 1)
open(p, "w").write(s)
