set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/bench_final4.json 2> gpurun_out/bench_final4.err
timeout 600 python tools/phase_times.py products > gpurun_out/phase_final4.txt 2>&1
python -c "
import json
d=json.load(open('gpurun_out/bench_final4.json')); print(d['ms_per_step'], d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'])"
