# A/B baseline: tc_sage.cu as committed at HEAD
import subprocess, sys
src = subprocess.check_output(["git", "show", "HEAD:paper_conf_hpca_yangzl25_b200/csrc/tc_sage.cu"]).decode()
open(sys.argv[1] + "/tc_sage.cu", "w").write(src)
