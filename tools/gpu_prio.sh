# A/B: training stream at high priority (default) vs the same priority as the scheduler's side stream
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -m pytest tests/test_gpu_nccl.py tests/test_gpu_pipeline.py -x -q -p no:cacheprovider 2>&1 | tail -3
for v in hi same hi same; do
  if [ $v = hi ]; then P=""; else P="--main-priority 0"; fi
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $P > gpurun_out/prio_$v.json 2> gpurun_out/prio_$v.err
  python -c "
import json; d=json.load(open('gpurun_out/prio_$v.json')); c=d['config']
print('$v', round(d['ms_per_step'],2), 'frac', round(d['roofline']['frac'],3), c['phases_ms_sequential'])" || tail -5 gpurun_out/prio_$v.err
done
