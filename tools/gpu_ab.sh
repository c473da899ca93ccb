# A/B of environment switches on one B200 (diagnostic): parity tests, then one bench line per case.
# usage: CASES="base: stream:BUFFALO_GEMM_STREAM_W=1" bash tools/gpu_ab.sh
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/pytest_gpu.txt
cat gpurun_out/pytest_gpu.txt
for c in ${CASES:-base:}; do
  name=${c%%:*}; envs=${c#*:}
  env $(echo $envs | tr ',' ' ') timeout 600 python bench.py --steps ${STEPS:-10} --warmup 3 --no-cpu-baseline ${BENCH_ARGS} > gpurun_out/ab_$name.json 2> gpurun_out/ab_$name.err
  python -c "import json,sys; d=json.load(open('gpurun_out/ab_$name.json')); print('$name', d['config']['config'], round(d['ms_per_step'],2), 'ms', round(d['roofline']['achieved']), 'GB/s', round(d['roofline']['frac'],3), 'share', round(d['roofline']['share_of_step'],3))" || tail -n 5 gpurun_out/ab_$name.err
done
