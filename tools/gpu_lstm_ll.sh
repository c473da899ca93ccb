set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed --clock-control none --csv \
  --log-file gpurun_out/launches_lstm2.csv python bench.py --config arxiv_lstm --aggregator lstm --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
python tools/launches.py gpurun_out/launches_lstm2.csv | head -12
