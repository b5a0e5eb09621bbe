python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 600 python tools/subtree_stats.py 2>&1 | grep -v Warning | grep "C4 A\|subtree" | tail -9 | head -5
