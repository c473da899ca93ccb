# A/B of the gather column-index prefetch: HEAD (base), prefetch at 5 CTAs/SM (main lib), at 4 (m4)
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_sharded.py tests/test_gpu_fullsize.py -x -q -p no:cacheprovider 2>&1 | tail -3
for v in base main m4 base main m4; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/ab_$v.json 2> gpurun_out/ab_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/ab_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])"
done
