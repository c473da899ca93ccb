# Round-end GPU pass: full GPU suite, smoke, the default bench line, products phase times and the
# ncu launch list of one products epoch (bench-equivalent, tools/prof_step.py).
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -6 > gpurun_out/pytest_gpu_final.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
timeout 600 python tools/phase_times.py products > gpurun_out/phase_final.txt 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_final.csv python tools/prof_step.py products 1 auto > gpurun_out/prof_final.log 2>&1
cat gpurun_out/pytest_gpu_final.txt gpurun_out/smoke_final.txt gpurun_out/bench_final.json gpurun_out/phase_final.txt
tail -n 3 gpurun_out/bench_final.err
