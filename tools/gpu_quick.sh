# quick GPU pass: build, main parity tests, bench line
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_memory.py tests/test_gpu_pipeline.py tests/test_gpu_determinism.py tests/test_gpu_edges.py -x -q -p no:cacheprovider > gpurun_out/pytest_quick.txt 2>&1; echo "pytest rc=$?"
tail -30 gpurun_out/pytest_quick.txt
timeout 900 python bench.py --steps 20 --warmup 4 --no-cpu-baseline > gpurun_out/bench_q.json 2> gpurun_out/bench_q.err; echo "bench rc=$?"
python - <<'PY'
import json
d = json.load(open("gpurun_out/bench_q.json"))
c = d["config"]
print("ms", d["ms_per_step"], "val", d["value"], "frac", d["roofline"]["frac"], "share", d["roofline"]["share_of_step"], "e2e", d["e2e"]["value"])
print("phases", c["phases_ms_sequential"], "K", c["K"])
print("mem", {k: d["memory"][k] for k in ("measured_high_water_max_bytes", "measured_within_exact_model", "exact_lo_minus_measured_max_bytes")})
PY
tail -3 gpurun_out/bench_q.err
