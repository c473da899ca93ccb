# A/B baseline: build.cu as committed at HEAD
import subprocess, sys
src = subprocess.check_output(["git", "show", "HEAD:paper_conf_hpca_yangzl25_b200/csrc/build.cu"]).decode()
open(sys.argv[1] + "/build.cu", "w").write(src)
