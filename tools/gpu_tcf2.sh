set -x
python -c "import __graft_entry__ as g; g.build()"
for t in test_gpu_pool test_gpu_lstm test_gpu_gat test_gpu_parity test_gpu_memory; do
  timeout 300 python -m pytest tests/$t.py -x -q -p no:cacheprovider 2>&1 | tail -3
done
for a in pool gat; do
  timeout 900 python bench.py --aggregator $a --steps 3 --warmup 2 > gpurun_out/bench_products_$a.json 2> gpurun_out/bench_$a.err; echo "$a rc=$?"
done
timeout 600 python bench.py --config arxiv_lstm --aggregator lstm --steps 10 --warmup 3 > gpurun_out/bench_arxiv_lstm.json 2> gpurun_out/bench_lstm.err; echo "lstm rc=$?"
for f in gpurun_out/bench_products_pool.json gpurun_out/bench_products_gat.json gpurun_out/bench_arxiv_lstm.json; do python -c "
import json; d=json.load(open('$f')); print('$f', round(d['ms_per_step'],1), 'K', d['config']['K'])"; done
for f in gpurun_out/bench_products_pool.json gpurun_out/bench_products_gat.json gpurun_out/bench_arxiv_lstm.json; do python -c "
import json; d=json.load(open('$f')); print('$f', d['config'].get('phases_ms_sequential'))"; done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_lstm_tcf.csv python bench.py --config arxiv_lstm --aggregator lstm --steps 1 --warmup 1 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_lstm_tcf.csv 2>&1 | head -20
