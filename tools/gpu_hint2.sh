# A/B: hint bits (main = fwd 0 / bwd 7), forward rows-only, backward subsets; scheduler atomic filter
python -c "import __graft_entry__ as g; g.build()"
for v in main f1 b1 b3 b5 mchk main f1 b1 b3 b5 mchk; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/hint2_$v.json 2> gpurun_out/hint2_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/hint2_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -3 gpurun_out/hint2_$v.err
done
