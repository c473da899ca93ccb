# A/B baseline: tc_sage.cu and tc_gemm.cu as committed at HEAD
import subprocess, sys
for f in ("tc_sage.cu", "tc_gemm.cu"):
    src = subprocess.check_output(["git", "show", "HEAD:paper_conf_hpca_yangzl25_b200/csrc/" + f]).decode()
    open(sys.argv[1] + "/" + f, "w").write(src)
