python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q -k "not c4_full" 2>&1 | tail -2
timeout 600 python tools/subtree_stats.py c4 2>&1 | grep -v Warning | tail -5
