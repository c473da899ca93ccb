set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_parity.py tests/test_gpu_pipeline.py -x -q -p no:cacheprovider 2>&1 | tail -5
BUFFALO_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 4 --warmup 3 --no-cpu-baseline > gpurun_out/bench_2r.json 2> gpurun_out/bench_2r.err; echo rc=$?
head -c 600 gpurun_out/bench_2r.json; tail -3 gpurun_out/bench_2r.err
