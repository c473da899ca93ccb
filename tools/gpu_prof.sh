# Profiling pass on one B200 (diagnostic): bench line, launch list with DRAM bytes, ncu --set full
# of the Aggregate (gather) launches of the first groups and of one GEMM / dW launch.
# usage: bash tools/gpu_prof.sh <config> <tag>
set -x
CFG=${1:-products}; TAG=${2:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 900 python bench.py --config $CFG > gpurun_out/bench_${CFG}_${TAG}.json 2> gpurun_out/bench_${CFG}_${TAG}.err
timeout 300 python tools/phase_times.py $CFG > gpurun_out/phase_${CFG}_${TAG}.txt 2>&1
AUTO=""; [ "$CFG" = products ] && AUTO=auto
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${CFG}_${TAG}.csv python tools/prof_step.py $CFG 1 $AUTO > gpurun_out/prof_${CFG}_${TAG}.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gather -c ${NG:-15} \
  -o gpurun_out/gather_${CFG}_${TAG} -f python tools/prof_step.py $CFG 1 $AUTO > gpurun_out/ncu_${CFG}_${TAG}.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tc_gemm_tma|k_tc_dw_tma" -c 6 \
  -o gpurun_out/gemm_${CFG}_${TAG} -f python tools/prof_step.py $CFG 1 $AUTO > gpurun_out/ncu_gemm_${CFG}_${TAG}.log 2>&1
cat gpurun_out/bench_${CFG}_${TAG}.json gpurun_out/phase_${CFG}_${TAG}.txt; tail -n 3 gpurun_out/bench_${CFG}_${TAG}.err; tail -n 3 gpurun_out/ncu_${CFG}_${TAG}.log
