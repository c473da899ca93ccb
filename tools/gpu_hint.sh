# A/B: L2 eviction hints in the Aggregate (none / backward / forward / both)
python -c "import __graft_entry__ as g; g.build()"
for v in main hbwd hfwd hboth main hbwd hfwd hboth; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/hint_$v.json 2> gpurun_out/hint_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/hint_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -3 gpurun_out/hint_$v.err
done
