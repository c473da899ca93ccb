# papers100M-shaped run on one B200 (BASELINE.json configs[3] at N=1): bench line + memory peak.
set -x
python -c "import __graft_entry__ as g; g.build()"
nvidia-smi --query-gpu=memory.used,memory.total --format=csv -lms 2000 > gpurun_out/papers_mem.csv &
SMI=$!
timeout 1700 python bench.py --config papers --steps 3 --warmup 3 --no-cpu-baseline > gpurun_out/bench_papers.json 2> gpurun_out/bench_papers.err
kill $SMI
cat gpurun_out/bench_papers.json; tail -n 25 gpurun_out/bench_papers.err
sort -t, -k1 -n gpurun_out/papers_mem.csv | tail -2
