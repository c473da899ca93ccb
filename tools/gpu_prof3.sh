# launch list of one products epoch (library kernels only) + ncu --set full of the first gathers
set -x
TAG=${1:-r02}
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu -k regex:"k_" --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_products_${TAG}.csv python tools/prof_step.py products 1 auto > gpurun_out/prof_${TAG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather -c 6 \
  -o gpurun_out/gather_${TAG} -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_gather_${TAG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tc_gemm_tma|k_tc_dw_tma" -c 4 \
  -o gpurun_out/gemm_${TAG} -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_gemm_${TAG}.log 2>&1
tail -2 gpurun_out/prof_${TAG}.log gpurun_out/ncu_gather_${TAG}.log
