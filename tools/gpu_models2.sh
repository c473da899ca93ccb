# GPU pass: widened-model parity tests + one bench line per widened model.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_gat.py tests/test_gpu_pool.py tests/test_gpu_lstm.py tests/test_gpu_parity.py -x -q 2>&1 | tail -4
timeout 900 python bench.py --aggregator gat --steps 5 --warmup 3 > gpurun_out/bench_gat.json 2> gpurun_out/bench_gat.err
timeout 900 python bench.py --aggregator pool --steps 5 --warmup 3 > gpurun_out/bench_pool.json 2> gpurun_out/bench_pool.err
timeout 900 python bench.py --config arxiv_lstm --aggregator lstm --steps 5 --warmup 3 > gpurun_out/bench_lstm.json 2> gpurun_out/bench_lstm.err
cat gpurun_out/bench_gat.json gpurun_out/bench_pool.json gpurun_out/bench_lstm.json
tail -n 3 gpurun_out/bench_gat.err gpurun_out/bench_pool.err gpurun_out/bench_lstm.err
