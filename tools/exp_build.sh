# Build an experimental libbuffalo variant from a patched copy of csrc (diagnostics only).
# usage: bash tools/exp_build.sh <name> <python-patch-script>   -> tools/exp/libbuffalo_<name>.so
set -e
NAME=$1; PATCH=$2
D=/tmp/exp_$NAME/a/b; rm -rf /tmp/exp_$NAME; mkdir -p $D; cp -r paper_conf_hpca_yangzl25_b200/csrc $D/; cp -r include /tmp/exp_$NAME/a/
python $PATCH $D/csrc
mkdir -p tools/exp
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -Xcompiler -fvisibility=hidden --expt-relaxed-constexpr"
for s in api build sage tc_sage tc_gemm tc_f32 cluster; do /usr/local/cuda/bin/nvcc $F -c $D/csrc/$s.cu -o $D/$s.o & done; wait
/usr/local/cuda/bin/nvcc -gencode arch=compute_100a,code=sm_100a -shared -o tools/exp/libbuffalo_$NAME.so $D/*.o
echo built tools/exp/libbuffalo_$NAME.so
