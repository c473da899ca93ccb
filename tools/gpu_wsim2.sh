# World-sim with shared scheduler statistics (--sim-shared): products 2/4/8, papers 8 (R31 and plain)
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_determinism.py tests/test_gpu_edges.py -x -q -p no:cacheprovider 2>&1 | tail -2
for v in a b; do
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/red_$v.json 2> gpurun_out/red_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/red_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -3 gpurun_out/red_$v.err
done
for N in 8 4 2; do
  timeout 900 python bench.py --world-sim $N --sim-shared --rank-balanced-k --steps 5 --warmup 2 > gpurun_out/wsims_products_${N}_rb.json 2> gpurun_out/wsims_products_$N.err
  timeout 900 python bench.py --world-sim $N --sim-shared --steps 5 --warmup 2 > gpurun_out/wsims_products_$N.json 2>> gpurun_out/wsims_products_$N.err
done
timeout 1500 python bench.py --config papers --world-sim 8 --sim-shared --rank-balanced-k --steps 4 --warmup 2 > gpurun_out/wsims_papers_8_rb.json 2> gpurun_out/wsims_papers_8.err
timeout 1500 python bench.py --config papers --world-sim 8 --sim-shared --steps 4 --warmup 2 > gpurun_out/wsims_papers_8.json 2>> gpurun_out/wsims_papers_8.err
for f in gpurun_out/wsims_*.json; do python -c "
import json,sys
d=json.load(open('$f')); print('$f', d['K'], round(d['projected_epoch_ms'],2), round(d['rank_spread_max_over_min'],3), [round(p['ms_per_step'],1) for p in d['per_rank']], [p['groups'] for p in d['per_rank']], d.get('allgathers_per_epoch'), round(d.get('record_s',0),1))" || tail -4 ${f%.json}.err; done
tail -3 gpurun_out/wsims_papers_8.err gpurun_out/wsims_products_8.err
