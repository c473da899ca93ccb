# Profiling pass on one B200 (diagnostic): bench line, launch list with DRAM bytes, ncu --set full of gathers.
# usage: bash tools/gpu_prof.sh <config> <tag>
set -x
CFG=${1:-products}; TAG=${2:-x}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python bench.py --config $CFG --steps 10 --warmup 3 > gpurun_out/bench_${CFG}_${TAG}.json 2> gpurun_out/bench_${CFG}_${TAG}.err
AUTO=""; [ "$CFG" = products ] && AUTO=auto
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_${CFG}_${TAG}.csv python tools/prof_step.py $CFG 1 $AUTO > gpurun_out/prof_${CFG}_${TAG}.log 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_gather_rows -c ${NG:-12} \
  -o gpurun_out/gather_${CFG}_${TAG} -f python tools/prof_step.py $CFG 1 $AUTO > gpurun_out/ncu_${CFG}_${TAG}.log 2>&1
cat gpurun_out/bench_${CFG}_${TAG}.json; tail -n 3 gpurun_out/bench_${CFG}_${TAG}.err; tail -n 5 gpurun_out/ncu_${CFG}_${TAG}.log
