# Last validation: build, smoke, the whole GPU suite, the default bench line, launch list
python -c "import __graft_entry__ as g; g.build()"
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider > gpurun_out/pytest_gpu_r02.txt 2>&1; tail -3 gpurun_out/pytest_gpu_r02.txt
timeout 900 python bench.py > gpurun_out/bench_products_r02_final.json 2> gpurun_out/bench_final.err; echo "bench rc=$?"
python -c "
import json; d=json.load(open('gpurun_out/bench_products_r02_final.json')); c=d['config']
print(round(d['ms_per_step'],2), '%.3g'%d['value'], 'frac', round(d['roofline']['frac'],3), 'e2e %.3g'%d['e2e']['value'], d['clocks'], c.get('phases_ms_sequential'), d['cpu_baseline']['value'], d['gpu_launches'])"
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv -k regex:"k_" \
  --log-file gpurun_out/launches_products_r02_final.csv python bench.py --steps 1 --warmup 0 --no-cpu-baseline > /dev/null 2>&1
python tools/launch_summary.py gpurun_out/launches_products_r02_final.csv > gpurun_out/launches_products_r02_final_summary.txt 2>&1; head -16 gpurun_out/launches_products_r02_final_summary.txt
