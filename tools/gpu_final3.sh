set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_final3.json 2> gpurun_out/bench_final3.err
timeout 600 python tools/phase_times.py products > gpurun_out/phase_final3.txt 2>&1
timeout 900 python bench.py --config papers --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_papers3.json 2> gpurun_out/bench_papers3.err
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv \
  --log-file gpurun_out/launches_final3.csv python tools/prof_step.py products 1 auto > gpurun_out/prof_final3.log 2>&1
python -c "
import json
for f in ['bench_final3', 'bench_papers3']:
    d=json.load(open('gpurun_out/%s.json' % f)); print(f, d['ms_per_step'], d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks']['sm_mhz'], d['memory'])"
cat gpurun_out/phase_final3.txt
