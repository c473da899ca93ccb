# GPU pass for the GraphSAGE-pool aggregator (NEXT 2): parity tests, then the products-shaped
# pool bench line (FFMA) and its launch list.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_pool.py tests/test_gpu_parity.py -x -q 2>&1 | tail -15 > gpurun_out/pytest_pool.txt
cat gpurun_out/pytest_pool.txt
timeout 900 python bench.py --aggregator pool --steps 5 --warmup 3 > gpurun_out/bench_pool.json 2> gpurun_out/bench_pool.err
cat gpurun_out/bench_pool.json; tail -5 gpurun_out/bench_pool.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_pool_products.csv python bench.py --aggregator pool --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_table.py gpurun_out/launches_pool_products.csv > gpurun_out/launches_pool_products.txt 2>&1
tail -5 gpurun_out/launches_pool_products.txt
