# One GPU pass: build, GPU parity tests, smoke, default bench line, products phase times.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.txt 2>&1
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 600 python tools/phase_times.py products > gpurun_out/phase_products.txt 2>&1
cat gpurun_out/pytest_gpu.txt gpurun_out/smoke.txt gpurun_out/bench.json gpurun_out/phase_products.txt
tail -3 gpurun_out/bench.err
