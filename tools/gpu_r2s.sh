# Round-2 session check: build, smoke, the whole GPU suite, the default bench line, launch list.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > gpurun_out/gputests.log 2>&1; echo "tests rc=$?"; tail -5 gpurun_out/gputests.log
timeout 900 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
python -c "
import json
d=json.load(open('gpurun_out/bench.json')); print(d['ms_per_step'], d['value'], d['roofline']['frac'], d['e2e']['value'], d['clocks'], d['config']['phases_ms_sequential'])"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_products.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_products.csv > gpurun_out/launches_products_summary.txt 2>&1; head -24 gpurun_out/launches_products_summary.txt
