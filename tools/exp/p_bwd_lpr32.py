# A/B: the backward fused Aggregate with 32 lanes per 512-B row (one pass over the pieces)
import sys
p = sys.argv[1] + "/tc_sage.cu"
s = open(p).read()
a = "while ((1 << lpr_log) < npieces && lpr_log < 4) ++lpr_log;     // <= 16 lanes per row (short rows)"
assert a in s
s = s.replace(a, "while ((1 << lpr_log) < npieces && lpr_log < 5) ++lpr_log;")
a = "  else BF_V2E(16);"
assert a in s
s = s.replace(a, "  else if (lpr_log == 4) BF_V2E(16);\n  else BF_V2E(32);")
open(p, "w").write(s)
