import sys
p = sys.argv[1] + "/tc_gemm.cu"; s = open(p).read()
s = s.replace("constexpr int kProducers = 2;", "constexpr int kProducers = 1;")
open(p, "w").write(s)
