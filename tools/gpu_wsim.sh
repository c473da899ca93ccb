set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -p no:cacheprovider -k "plan" 2>&1 | tail -3
for N in 2 4 8; do
  timeout 900 python bench.py --world-sim $N --steps 5 --warmup 3 > gpurun_out/wsim_products_$N.json 2> gpurun_out/wsim_products_$N.err
  timeout 900 python bench.py --world-sim $N --rank-balanced-k --steps 5 --warmup 3 > gpurun_out/wsim_products_${N}_rb.json 2>> gpurun_out/wsim_products_$N.err
done
timeout 1200 python bench.py --config papers --world-sim 8 --steps 4 --warmup 2 > gpurun_out/wsim_papers_8.json 2> gpurun_out/wsim_papers_8.err
timeout 1200 python bench.py --config papers --world-sim 8 --rank-balanced-k --steps 4 --warmup 2 > gpurun_out/wsim_papers_8_rb.json 2>> gpurun_out/wsim_papers_8.err
for f in gpurun_out/wsim_*.json; do python -c "
import json,sys
d=json.load(open('$f')); print('$f', d['K'], round(d['projected_epoch_ms'],2), round(d['rank_spread_max_over_min'],3), [round(p['ms_per_step'],1) for p in d['per_rank']], [p['groups'] for p in d['per_rank']])"; done
tail -3 gpurun_out/wsim_papers_8.err
