# Launch-list timing of selected kernels under experimental builds (diagnostic).
# usage: EXPS="base nogather" bash tools/gpu_ncu_exp.sh <regex> <count>
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null
for e in ${EXPS:-base}; do
  if [ "$e" = base ]; then unset BUFFALO_LIB; else export BUFFALO_LIB=$PWD/tools/exp/libbuffalo_$e.so; fi
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
    -k regex:"$1" -c ${2:-10} --log-file gpurun_out/exp_$e.csv python tools/prof_step.py products 1 auto > gpurun_out/exp_$e.log 2>&1
  echo "== $e"; python tools/launch_table.py gpurun_out/exp_$e.csv
done
