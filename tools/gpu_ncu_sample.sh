set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_sample_fill|k_mask_layer" --launch-skip 10 -c 6 \
  -o gpurun_out/ncu_sample -f python tools/prof_step.py products 1 auto > gpurun_out/ncu_sample.log 2>&1
tail -n 2 gpurun_out/ncu_sample.log
