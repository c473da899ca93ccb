# After the scheduler count change: products default line, papers line and papers 8-rank shared-stats world-sim
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_products_r02_final2.json 2> gpurun_out/bench_final2.err; echo "bench rc=$?"
timeout 1500 python bench.py --config papers --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/bench_papers_r02b.json 2> gpurun_out/bench_papers2.err; echo "papers rc=$?"
for f in products_r02_final2 papers_r02b; do python -c "
import json; d=json.load(open('gpurun_out/bench_$f.json')); c=d['config']
print('$f', round(d['ms_per_step'],2), '%.3g'%d['value'], 'frac', round(d['roofline']['frac'],3), 'e2e %.3g'%d['e2e']['value'], 'K', c.get('K'), d['clocks'], c.get('phases_ms_sequential'), (d.get('cpu_baseline') or {}).get('value'))" || tail -3 gpurun_out/bench_*2.err; done
timeout 1500 python bench.py --config papers --world-sim 8 --sim-shared --steps 4 --warmup 2 > gpurun_out/wsims_papers_8.json 2> gpurun_out/wsims_papers_8.err
timeout 1500 python bench.py --config papers --world-sim 8 --sim-shared --rank-balanced-k --steps 4 --warmup 2 > gpurun_out/wsims_papers_8_rb.json 2>> gpurun_out/wsims_papers_8.err
timeout 900 python bench.py --world-sim 8 --sim-shared --rank-balanced-k --steps 5 --warmup 2 > gpurun_out/wsims_products_8_rb.json 2> gpurun_out/wsims_products_8.err
for f in gpurun_out/wsims_papers_8.json gpurun_out/wsims_papers_8_rb.json gpurun_out/wsims_products_8_rb.json; do python -c "
import json
d=json.load(open('$f')); print('$f', d['K'], round(d['projected_epoch_ms'],2), round(d['rank_spread_max_over_min'],3), [round(p['ms_per_step'],1) for p in d['per_rank']], [p['groups'] for p in d['per_rank']])"; done
