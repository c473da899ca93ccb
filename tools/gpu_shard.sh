set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_sharded.py tests/test_gpu_parity.py -x -q -p no:cacheprovider 2>&1 | tail -30
