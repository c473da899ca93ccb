# GPU pass: full GPU suite, smoke, the default bench line, and one bench line per widened model
# (SAGE-pool / GAT on products, SAGE-LSTM on the paper's arxiv LSTM workload) + GAT launch list.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -8 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 900 python bench.py --aggregator gat --steps 5 --warmup 3 > gpurun_out/bench_gat.json 2> gpurun_out/bench_gat.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_gat.csv python bench.py --aggregator gat --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_table.py gpurun_out/launches_gat.csv > gpurun_out/launches_gat.txt 2>&1
cat gpurun_out/pytest_gpu.txt gpurun_out/smoke.txt gpurun_out/bench.json gpurun_out/bench_gat.json
tail -3 gpurun_out/bench.err gpurun_out/bench_gat.err
