# Round-2 final evidence: full GPU suite, smoke, default bench line (with cpu_baseline), the other
# configs' bench lines, the products launch list, and ncu --set full captures of the top kernels.
set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_r02.txt 2>&1; tail -1 gpurun_out/smoke_r02.txt
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_r02.txt 2>&1; tail -4 gpurun_out/pytest_gpu_r02.txt
timeout 900 python bench.py > gpurun_out/bench_products_r02_final.json 2> gpurun_out/bench_final.err; echo "bench rc=$?"
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_reference_r02.json 2> gpurun_out/bench_ref.err; echo "ref rc=$?"
timeout 1500 python bench.py --config papers --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_papers_r02.json 2> gpurun_out/bench_papers.err; echo "papers rc=$?"
timeout 1500 python bench.py --config igb_small --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_igb_small_r02.json 2> gpurun_out/bench_igb.err; echo "igb rc=$?"
timeout 900 python bench.py --config arxiv --steps 20 --warmup 5 > gpurun_out/bench_arxiv_r02.json 2> gpurun_out/bench_arxiv.err; echo "arxiv rc=$?"
for f in products_r02_final papers_r02 igb_small_r02 arxiv_r02; do python -c "
import json; d=json.load(open('gpurun_out/bench_$f.json')); c=d['config']
print('$f', round(d['ms_per_step'],2), '%.3g'%d['value'], 'frac', round(d['roofline']['frac'],3), 'e2e %.3g'%d['e2e']['value'], 'K', c.get('K'), d['clocks'], c.get('phases_ms_sequential'), (d.get('cpu_baseline') or {}).get('value'))" || tail -3 gpurun_out/bench_*.err; done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_products_r02_final.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_products_r02_final.csv > gpurun_out/launches_products_r02_final_summary.txt 2>&1; head -24 gpurun_out/launches_products_r02_final_summary.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gather_v2 --launch-skip 60 -c 6 \
  -o gpurun_out/ncu_gather_r02_final -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_gather.log 2>&1; echo "ncu gather rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tc_gemm_tma|k_tc_dw_tma" --launch-skip 40 -c 10 \
  -o gpurun_out/ncu_tc_r02_final -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_tc.log 2>&1; echo "ncu tc rc=$?"
python tools/ncu_summary.py gpurun_out/ncu_gather_r02_final.ncu-rep > gpurun_out/ncu_gather_r02_final.txt 2>&1; head -30 gpurun_out/ncu_gather_r02_final.txt
python tools/ncu_summary.py gpurun_out/ncu_tc_r02_final.ncu-rep > gpurun_out/ncu_tc_r02_final.txt 2>&1; head -5 gpurun_out/ncu_tc_r02_final.txt
