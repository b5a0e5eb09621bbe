# round-2 call b: GPU suite, racecheck on the small end-to-end workload, C4 bench, subtree phase counters
D=gpurun_out/r02b; mkdir -p $D
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q -rf -x > $D/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $D/pytest_gpu.log
tail -n 6 $D/pytest_gpu.log
timeout 900 compute-sanitizer --tool racecheck --print-limit 20 python tools/sanitize_small.py > $D/racecheck.txt 2>&1; echo "rc=$?" >> $D/racecheck.txt
grep -E "RACECHECK SUMMARY|ERROR SUMMARY" $D/racecheck.txt | tail -2
timeout 900 compute-sanitizer --tool memcheck python tools/sanitize_small.py > $D/memcheck.txt 2>&1; echo "rc=$?" >> $D/memcheck.txt
grep -E "ERROR SUMMARY" $D/memcheck.txt | tail -1
timeout 1200 python bench.py --steps 3 --warmup 2 --no-cpu-baseline > $D/bench.log 2>&1; echo "bench rc=$?" >> $D/bench.log
grep "^{" $D/bench.log | tail -1 | cut -c1-400
BF_SUBTREE_STATS=1 timeout 600 python bench.py --ntree 200 --m-query 0 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-profile > $D/subtree_stats.txt 2>&1
grep "\[subtree" $D/subtree_stats.txt | tail -4
