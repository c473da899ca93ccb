# TMA-fed tcgen05 fp32 GEMM + dW: parity of every fp32 path, bench lines, fp32-kernel launch lists.
set -x
python -c "import __graft_entry__ as g; g.build()"
for t in test_gpu_pool test_gpu_lstm test_gpu_gat test_gpu_parity test_gpu_memory test_gpu_edges; do
  timeout 300 python -m pytest tests/$t.py -x -q -p no:cacheprovider 2>&1 | grep -E "passed|failed|Error|out of tol|Mismatch|Max" | head -8
done
for a in pool gat; do
  timeout 900 python bench.py --aggregator $a --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_$a.json 2> gpurun_out/bench_$a.err; echo "$a rc=$?"
done
timeout 600 python bench.py --gemm ffma --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_ffma.json 2> gpurun_out/bench_ffma.err; echo "ffma rc=$?"
timeout 600 python bench.py --config arxiv_lstm --aggregator lstm --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_arxiv_lstm.json 2> gpurun_out/bench_lstm.err; echo "lstm rc=$?"
for f in products_pool products_gat products_ffma arxiv_lstm; do python -c "
import json; d=json.load(open('gpurun_out/bench_$f.json')); print('$f', round(d['ms_per_step'],1), 'K', d['config']['K'], d['config'].get('phases_ms_sequential'))" || tail -3 gpurun_out/bench_*.err; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_pool_tcf.csv python bench.py --aggregator pool --steps 1 --warmup 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_pool_tcf.csv 2>&1 | head -14
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_lstm_tcf.csv python bench.py --config arxiv_lstm --aggregator lstm --steps 1 --warmup 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_lstm_tcf.csv 2>&1 | head -10
