python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q -k "not c4_full" 2>&1 | tail -3
timeout 600 python tools/subtree_stats.py 2>&1 | grep -v Warning | grep "C4\|subtree\]" | tail -4
bash tools/level_timing.sh 2>&1 | tail -2
