set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_pipeline.py tests/test_gpu_parity.py -x -q 2>&1 | tail -4
timeout 900 python bench.py --steps 20 --no-cpu-baseline > gpurun_out/bench_pipe.json 2> gpurun_out/bench_pipe.err
timeout 900 python bench.py --steps 20 --no-cpu-baseline --no-pipeline > gpurun_out/bench_nopipe.json 2> gpurun_out/bench_nopipe.err
cat gpurun_out/bench_pipe.json gpurun_out/bench_nopipe.json; tail -n 3 gpurun_out/bench_pipe.err
