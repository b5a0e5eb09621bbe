# round-2 call al: ballot-built member masks (BF_TINY_V=2) vs the position table (1); back-off 512 default
D=gpurun_out/r02al; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or tiny or config" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
BF_TINY_V=2 timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config" > $D/pytest2.log 2>&1; echo "pytest tv2 rc=$?" >> $D/pytest2.log
tail -n 2 $D/pytest.log $D/pytest2.log
for v in 1 2; do
  BF_TINY_V=$v timeout 600 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1
  echo "tv=$v"; grep "subtree" $D/stats_$v.txt | head -4
done
