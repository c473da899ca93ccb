# ncu --set full of selected launches (diagnostic).  usage: bash tools/gpu_ncu_k.sh <regex> <skip> <count> <tag> [config]
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
CFG=${5:-products}; AUTO=""; [ "$CFG" = products ] && AUTO=auto
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"$1" --launch-skip $2 -c $3 \
  -o gpurun_out/k_$4 -f python tools/prof_step.py $CFG 1 $AUTO > gpurun_out/ncu_k_$4.log 2>&1
tail -n 4 gpurun_out/ncu_k_$4.log
