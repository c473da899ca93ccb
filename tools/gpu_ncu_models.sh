# ncu --set full captures: the widened models' HBM kernels (traffic for the bench roofline) and
# the tensor-core GEMMs of the products epoch.
set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_gat_attn --launch-skip 20 -c 3 \
  -o gpurun_out/ncu_gat_attn -f python bench.py --aggregator gat --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_gat.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_pool_max --launch-skip 20 -c 3 \
  -o gpurun_out/ncu_pool_max -f python bench.py --aggregator pool --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_pool.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_tc_gemm_tma --launch-skip 30 -c 9 \
  -o gpurun_out/ncu_tcgemm -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_tcgemm.log 2>&1
tail -n 2 gpurun_out/ncu_gat.log gpurun_out/ncu_pool.log gpurun_out/ncu_tcgemm.log
