# Full-size IGB-shaped sharded parity; papers100M-shaped scheduler timing and its launch list
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests/test_gpu_fullsize_igb.py -x -q -p no:cacheprovider 2>&1 | tail -4
timeout 900 python tools/sched_time.py papers 2>&1 | tail -3
timeout 1500 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  -k regex:"k_mask|k_seed|k_part|k_scan|k_scatter|k_sample|k_cache|k_check" \
  --log-file gpurun_out/launches_papers_sched.csv python tools/sched_time.py papers > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_papers_sched.csv > gpurun_out/launches_papers_sched_summary.txt 2>&1; head -20 gpurun_out/launches_papers_sched_summary.txt
