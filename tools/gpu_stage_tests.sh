# Parity of the single-staging-box GEMM epilogue: the tensor-core suites
python -c "import __graft_entry__ as g; g.build()"
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_sharded.py tests/test_gpu_determinism.py tests/test_gpu_pipeline.py tests/test_gpu_memory.py tests/test_gpu_abi_errors.py tests/test_gpu_multirank.py tests/test_gpu_fullsize_igb.py -x -q -p no:cacheprovider 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
