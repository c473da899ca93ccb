# A/B of gather variants on one B200 (diagnostic): parity tests, then bench lines per variant.
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
cat gpurun_out/pytest_gpu.txt
for v in ${VARIANTS:-row 0 1 2}; do
  if [ "$v" = row ]; then export BUFFALO_ROW_GATHER=1; else export BUFFALO_ROW_GATHER=0 BUFFALO_GATHER_VARIANT=$v; fi
  timeout 600 python bench.py --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ab_$v.json 2> gpurun_out/ab_$v.err
  python -c "import json,sys; d=json.load(open('gpurun_out/ab_$v.json')); print('$v', d['config']['config'], round(d['ms_per_step'],2), 'ms', round(d['roofline']['achieved']), 'GB/s', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3))" || tail -n 5 gpurun_out/ab_$v.err
done
