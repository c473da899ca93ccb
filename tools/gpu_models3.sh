# Widened models (fp32 tcgen05 path) and the mean FFMA parity path: bench lines + launch lists
python -c "import __graft_entry__ as g; g.build()"
for a in pool gat; do
  timeout 900 python bench.py --aggregator $a --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_$a.json 2> gpurun_out/bench_$a.err; echo "$a rc=$?"
done
timeout 600 python bench.py --gemm ffma --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_ffma.json 2> gpurun_out/bench_ffma.err; echo "ffma rc=$?"
timeout 600 python bench.py --config arxiv_lstm --aggregator lstm --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_arxiv_lstm.json 2> gpurun_out/bench_lstm.err; echo "lstm rc=$?"
for f in products_pool products_gat products_ffma arxiv_lstm; do python -c "
import json; d=json.load(open('gpurun_out/bench_$f.json')); print('$f', round(d['ms_per_step'],1), 'K', d['config']['K'], d['roofline']['kernel'][:30], round(d['roofline']['frac'],3), d['config'].get('phases_ms_sequential'))" || tail -3 gpurun_out/bench_*.err; done
for a in pool gat lstm mean_ffma; do
  timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
    --log-file gpurun_out/launches_model_$a.csv python tools/prof_model.py $a > /dev/null 2>&1
  python tools/launch_summary.py gpurun_out/launches_model_$a.csv > gpurun_out/launches_model_${a}_summary.txt 2>&1; head -10 gpurun_out/launches_model_${a}_summary.txt
done
