set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python -m pytest tests -m gpu -x -q -p no:cacheprovider --deselect tests/test_gpu_sanitizer.py --deselect tests/test_gpu_fullsize.py::test_products_plan_equals_oracle_schedule > gpurun_out/pytest_q2.txt 2>&1; echo "pytest rc=$?"
tail -15 gpurun_out/pytest_q2.txt
timeout 900 python bench.py --steps 20 --warmup 4 --no-cpu-baseline > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; echo "bench rc=$?"
python - <<'PY'
import json
d = json.load(open("gpurun_out/bench_q.json"))
c = d["config"]
print("ms", d["ms_per_step"], "val", d["value"], "frac", d["roofline"]["frac"], "share", d["roofline"]["share_of_step"], "e2e", d["e2e"]["value"])
print("phases", c["phases_ms_sequential"], "K", c["K"], c["block_build"])
PY
tail -3 gpurun_out/bench_q.err
