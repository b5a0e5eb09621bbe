# round-2 call aw: compute-sanitizer on the final code (small end-to-end workload)
D=gpurun_out/r02aw; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for tool in memcheck synccheck racecheck; do
  timeout 900 compute-sanitizer --tool $tool python tools/sanitize_small.py > $D/$tool.log 2>&1; echo "$tool rc=$?"
  grep -E "SUMMARY" $D/$tool.log | tail -2
done
BF_TINY_V=2 timeout 900 compute-sanitizer --tool racecheck python tools/sanitize_small.py > $D/racecheck_tv2.log 2>&1; echo "racecheck tv2 rc=$?"
grep -E "SUMMARY" $D/racecheck_tv2.log | tail -2
grep -E "Race reported|Write Thread|Read Thread|at .*fit.cu" $D/racecheck.log | head -20
