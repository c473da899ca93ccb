set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_multirank.py tests/test_gpu_parity.py tests/test_gpu_pipeline.py tests/test_gpu_sharded.py -x -q -p no:cacheprovider 2>&1 | tail -5
for N in 8; do
  timeout 900 python bench.py --world-sim $N --rank-balanced-k --steps 5 --warmup 3 > gpurun_out/wsim_products_${N}_rb.json 2> gpurun_out/wsim.err
done
timeout 1200 python bench.py --config papers --world-sim 8 --rank-balanced-k --steps 4 --warmup 2 > gpurun_out/wsim_papers_8_rb.json 2>> gpurun_out/wsim.err
for f in gpurun_out/wsim_products_8_rb.json gpurun_out/wsim_papers_8_rb.json; do python -c "
import json
d=json.load(open('$f')); print('$f'.split('/')[-1], 'K',d['K'], 'proj', round(d['projected_epoch_ms'],2), 'spread', round(d['rank_spread_max_over_min'],3), [round(p['ms_per_step'],1) for p in d['per_rank']], [p['groups'] for p in d['per_rank']])"; done
tail -2 gpurun_out/wsim.err
