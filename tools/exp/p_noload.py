import sys
p = sys.argv[1] + "/tc_gemm.cu"; s = open(p).read()
old = "mb_expect(&full[st], kChunkA + (p.w_res ? 0 : bbytes));"
assert old in s
s = s.replace(old, "mb_expect(&full[st], 0);")
old = "        if (c < p.nkc_self && p.self_idx) {"
assert old in s
s = s.replace(old, "        if (p.n_rows < 0) {")
old = "        } else if (lane == 0) {\n          if (c < p.nkc_self) tma_2d"
assert old in s
s = s.replace(old, "        } else if (lane == 0 && p.n_rows < 0) {\n          if (c < p.nkc_self) tma_2d")
old = "if (lane == 0 && !p.w_res) bulk_1d("
assert old in s
s = s.replace(old, "if (lane == 0 && !p.w_res && p.n_rows < 0) bulk_1d(")
open(p, "w").write(s)
