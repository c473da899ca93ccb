set -x
python -c "import __graft_entry__ as g; g.build()"
for t in test_gpu_pool test_gpu_lstm test_gpu_gat test_gpu_parity; do
  timeout 300 python -m pytest tests/$t.py -x -q -p no:cacheprovider 2>&1 | grep -E "passed|failed|Error|out of tol|Mismatch|Max" | head -8
done
