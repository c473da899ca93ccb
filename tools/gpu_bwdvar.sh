# A/B: backward fused Aggregate variants — 32 lanes per 512-B row (lpr32), software-pipelined (bpipe) vs main
python -c "import __graft_entry__ as g; g.build()"
for v in lpr32 bpipe; do
  BUFFALO_LIB=tools/exp/libbuffalo_$v.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py -x -q -p no:cacheprovider 2>&1 | tail -1 | sed "s/^/$v /"
done
for v in main lpr32 bpipe main lpr32 bpipe; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/bv_$v.json 2> gpurun_out/bv_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/bv_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -3 gpurun_out/bv_$v.err
done
