python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q -k "not c4_full" 2>&1 | tail -3
bash tools/level_timing.sh 2>&1 | tail -34 | awk 'NR%3==1'
bash tools/level_timing.sh 2>&1 | tail -2
