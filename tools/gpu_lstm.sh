# GPU pass for the GraphSAGE-LSTM aggregator (NEXT 1): parity tests, the paper's LSTM workload
# (arxiv-shaped, 2-layer, fanout (10,25)) bench line and its launch list.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_lstm.py tests/test_gpu_pool.py -x -q 2>&1 | tail -5 > gpurun_out/pytest_lstm.txt
cat gpurun_out/pytest_lstm.txt
timeout 900 python bench.py --config arxiv_lstm --aggregator lstm --steps 5 --warmup 3 > gpurun_out/bench_lstm.json 2> gpurun_out/bench_lstm.err
cat gpurun_out/bench_lstm.json; tail -5 gpurun_out/bench_lstm.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_lstm.csv python bench.py --config arxiv_lstm --aggregator lstm --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_table.py gpurun_out/launches_lstm.csv > gpurun_out/launches_lstm.txt 2>&1
tail -3 gpurun_out/launches_lstm.txt
