# Full GPU suite, the fp32-path bench lines, and one ncu --set full capture of each tcgen05 fp32 kernel (pool, products).
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests -m gpu -q -p no:cacheprovider 2>&1 | tail -4
for a in pool gat; do
  timeout 900 python bench.py --aggregator $a --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_$a.json 2> gpurun_out/bench_$a.err; echo "$a rc=$?"
done
timeout 600 python bench.py --gemm ffma --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_ffma.json 2> gpurun_out/bench_ffma.err; echo "ffma rc=$?"
timeout 600 python bench.py --config arxiv_lstm --aggregator lstm --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bench_arxiv_lstm.json 2> gpurun_out/bench_lstm.err; echo "lstm rc=$?"
for f in products_pool products_gat products_ffma arxiv_lstm; do python -c "
import json; d=json.load(open('gpurun_out/bench_$f.json')); print('$f', round(d['ms_per_step'],1), 'K', d['config']['K'], d['config'].get('phases_ms_sequential'))" || tail -3 gpurun_out/bench_*.err; done
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tcf_gemm" -s 40 -c 1 -o gpurun_out/ncu_tcf_gemm_pool -f \
  python bench.py --aggregator pool --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_gemm.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tcf_dw" -s 40 -c 1 -o gpurun_out/ncu_tcf_dw_pool -f \
  python bench.py --aggregator pool --steps 1 --warmup 0 --no-cpu-baseline > gpurun_out/ncu_dw.log 2>&1
tail -2 gpurun_out/ncu_gemm.log gpurun_out/ncu_dw.log
