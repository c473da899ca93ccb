# Bit-sliced item counters in k_mask_count: plan parity + scheduler timing (papers, products) vs HEAD (hb)
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py tests/test_gpu_multirank.py -x -q -p no:cacheprovider 2>&1 | tail -2
for v in main hb; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 900 python tools/sched_time.py papers 2>&1 | tail -2 | sed "s/^/$v /"
  BUFFALO_LIB=$L timeout 900 python tools/sched_time.py products 2>&1 | tail -2 | sed "s/^/$v /"
done
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -x -q -p no:cacheprovider 2>&1 | tail -2
