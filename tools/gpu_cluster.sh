# GPU pass for the clustering coefficient (NEXT row 4): parity tests, timing, ncu of k_tri.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_clustering.py -x -q 2>&1 | tail -15 > gpurun_out/pytest_cluster.txt
timeout 300 python tools/bench_clustering.py products 5 > gpurun_out/cluster_products.json 2>&1
timeout 300 python tools/bench_clustering.py arxiv 5 > gpurun_out/cluster_arxiv.json 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_cluster_products.csv python tools/bench_clustering.py products 1 > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tri -c 1 \
  -o gpurun_out/ncu_tri_products -f python tools/bench_clustering.py products 1 > gpurun_out/ncu_tri.log 2>&1
cat gpurun_out/pytest_cluster.txt gpurun_out/cluster_products.json gpurun_out/cluster_arxiv.json
tail -3 gpurun_out/ncu_tri.log
