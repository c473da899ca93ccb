# A/B: forward Aggregate kU = 3 at 4 CTAs/SM (ku3) vs kU = 2 at 5 (main)
python -c "import __graft_entry__ as g; g.build()"
BUFFALO_LIB=tools/exp/libbuffalo_ku3.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py -x -q -p no:cacheprovider 2>&1 | tail -1
for v in main ku3 main ku3; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/k3_$v.json 2> gpurun_out/k3_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/k3_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -3 gpurun_out/k3_$v.err
done
