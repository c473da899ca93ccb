set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python bench.py --config igb_small --steps 6 --warmup 3 > gpurun_out/bench_igb_small.json 2> gpurun_out/bench_igb_small.err; echo "rc=$?"
tail -5 gpurun_out/bench_igb_small.err
python - <<'PY'
import json
d = json.load(open("gpurun_out/bench_igb_small.json"))
c = d["config"]
print("ms", d["ms_per_step"], "val", d["value"], "frac", d["roofline"]["frac"], "share", d["roofline"]["share_of_step"], "e2e", d["e2e"]["value"])
print("phases", c["phases_ms_sequential"], "K", c["K"], "red", c["redundancy"])
print("mem", d["memory"])
PY
