# A/B: k_mask_count nodes per thread by layer size (main) vs fixed (hb = HEAD): scheduler timing + plan parity
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_edges.py -x -q -p no:cacheprovider 2>&1 | tail -2
for v in main hb main hb; do
  if [ $v = main ]; then L=""; else L="tools/exp/libbuffalo_$v.so"; fi
  BUFFALO_LIB=$L timeout 900 python tools/sched_time.py papers 2>&1 | tail -2 | sed "s/^/$v /"
  BUFFALO_LIB=$L timeout 900 python tools/sched_time.py products 2>&1 | tail -2 | sed "s/^/$v /"
done
python tools/sched_prof.py papers 2>&1 | tail -8
