# round-2 call c: racecheck with RMW-atomic queue, trees-in-flight sweep, GPU suite
D=gpurun_out/r02c; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 compute-sanitizer --tool racecheck --print-limit 10 python tools/sanitize_small.py > $D/racecheck.txt 2>&1; echo "rc=$?" >> $D/racecheck.txt
grep -E "RACECHECK SUMMARY|ERROR SUMMARY" $D/racecheck.txt | tail -2
for B in 20 37 0; do
  timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e --trees-in-flight $B > $D/bench_B$B.log 2>&1
  echo "B=$B"; grep "^{" $D/bench_B$B.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(d['value'], d['phases_ms'], {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:6]})"
done
timeout 2400 python -m pytest tests -m gpu -q -rf -x > $D/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $D/pytest_gpu.log
tail -n 3 $D/pytest_gpu.log
