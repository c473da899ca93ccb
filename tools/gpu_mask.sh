# ReLU' bit mask for the backward's fused transposed Aggregate: parity suites + bench
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_memory.py tests/test_gpu_edges.py tests/test_gpu_abi_errors.py tests/test_gpu_determinism.py tests/test_gpu_sharded.py tests/test_gpu_pipeline.py tests/test_gpu_fullsize.py tests/test_gpu_multirank.py -x -q -p no:cacheprovider 2>&1 | tail -5
for v in a b; do
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/mask_$v.json 2> gpurun_out/mask_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/mask_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'], d['memory']['measured_within_exact_model'])" || tail -5 gpurun_out/mask_$v.err
done
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_mask.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_mask.csv > gpurun_out/launches_mask_summary.txt 2>&1; head -12 gpurun_out/launches_mask_summary.txt
