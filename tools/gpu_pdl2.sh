# A/B: PDL also for the forward / backward gathers and tcgen05 GEMMs (main) vs build only (hd)
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_sharded.py tests/test_gpu_determinism.py tests/test_gpu_pipeline.py tests/test_gpu_memory.py tests/test_gpu_abi_errors.py -x -q -p no:cacheprovider 2>&1 | tail -2
for v in main hd main hd; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/pdl2_$v.json 2> gpurun_out/pdl2_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/pdl2_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -3 gpurun_out/pdl2_$v.err
done
