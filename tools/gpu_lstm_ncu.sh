set -x
python -c "import __graft_entry__ as g; g.build()"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:"k_gemm2|k_dw_partial" --launch-skip 400 -c 4 \
  -o gpurun_out/ncu_lstm_simt -f python bench.py --config arxiv_lstm --aggregator lstm --steps 1 --warmup 1 --no-cpu-baseline > gpurun_out/ncu_lstm_simt.log 2>&1
tail -n 3 gpurun_out/ncu_lstm_simt.log
