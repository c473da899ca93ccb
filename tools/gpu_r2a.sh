# Round-2 check: build, GPU tests (sanitizers separately), smoke, bench line.
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()"
timeout 1800 python -m pytest tests -m gpu -x -q --deselect tests/test_gpu_sanitizer.py -p no:cacheprovider --durations=25 > gpurun_out/pytest_gpu.txt 2>&1; echo "pytest rc=$?"
tail -45 gpurun_out/pytest_gpu.txt
timeout 1500 python -m pytest tests/test_gpu_sanitizer.py -q -p no:cacheprovider > gpurun_out/pytest_san.txt 2>&1; echo "san rc=$?"
tail -30 gpurun_out/pytest_san.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1; tail -2 gpurun_out/smoke.txt
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
cat gpurun_out/bench.json; tail -5 gpurun_out/bench.err
