# GAT backward: weighted column sums for da_l / da_r, single-pass src kernel; FFMA Aggregate roofline
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_gat.py tests/test_gpu_fullsize_models.py tests/test_gpu_determinism.py -x -q -p no:cacheprovider 2>&1 | tail -3
timeout 900 python bench.py --aggregator gat --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_gat2.json 2> gpurun_out/bench_gat2.err; echo "gat rc=$?"
timeout 600 python bench.py --gemm ffma --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_products_ffma2.json 2> gpurun_out/bench_ffma2.err; echo "ffma rc=$?"
for f in products_gat2 products_ffma2; do python -c "
import json; d=json.load(open('gpurun_out/bench_$f.json')); print('$f', round(d['ms_per_step'],1), 'K', d['config']['K'], d['roofline']['kernel'][:30], round(d['roofline']['frac'],3), d['config'].get('phases_ms_sequential'))"; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_model_gat2.csv python tools/prof_model.py gat > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_model_gat2.csv > gpurun_out/launches_model_gat2_summary.txt 2>&1; head -12 gpurun_out/launches_model_gat2_summary.txt
