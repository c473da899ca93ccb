# Profiling pass (diagnostic): launch list with DRAM bytes over one products epoch, ncu --set full
# of the first gathers (fwd + fused bwd) and of the build's relabel kernels.
# usage: bash tools/gpu_prof2.sh <tag>
set -x
TAG=${1:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_products_${TAG}.csv python tools/prof_step.py products 1 auto > gpurun_out/prof_${TAG}.log 2>&1
python tools/launches.py gpurun_out/launches_products_${TAG}.csv > gpurun_out/launches_products_${TAG}_summary.txt
cat gpurun_out/launches_products_${TAG}_summary.txt
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gather -c 5 \
  -o gpurun_out/gather_${TAG} -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_gather_${TAG}.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_mark_bits|k_col_local|k_emit_bits|k_cache_fill|k_tfill" -c 10 \
  -o gpurun_out/build_${TAG} -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_build_${TAG}.log 2>&1
tail -n 3 gpurun_out/ncu_gather_${TAG}.log gpurun_out/ncu_build_${TAG}.log
