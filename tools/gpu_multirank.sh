set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_multirank.py -x -q 2>&1 | tail -15
BUFFALO_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
  --master-port 29533 bench.py --gpus 2 --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_2ranks_gloo.json 2> gpurun_out/bench_2ranks.err
cat gpurun_out/bench_2ranks_gloo.json; tail -n 5 gpurun_out/bench_2ranks.err
