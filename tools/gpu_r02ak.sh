# round-2 call ak: idle-warp back-off cap of the tiny queue with the faster tiny nodes
D=gpurun_out/r02ak; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for v in 64 256 2048 512 64; do
  BF_TQ_SLEEP_MAX=$v timeout 600 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1
  echo "sleep_max=$v"; grep "subtree\]" $D/stats_$v.txt | head -1
done
