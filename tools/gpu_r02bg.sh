# round-2 call bg: bf_release_workspace; allocator test alone and in the full GPU suite; smoke; default bench
D=gpurun_out/r02bg; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -k "library_memory" > $D/pytest_alloc.log 2>&1; echo "alloc test rc=$?"; tail -1 $D/pytest_alloc.log
timeout 2400 python -m pytest tests -x -q -m gpu > $D/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $D/pytest_gpu.log
tail -n 3 $D/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; echo "smoke rc=$?" >> $D/smoke.log; tail -2 $D/smoke.log
timeout 1500 python bench.py > $D/bench.log 2>&1; echo "bench rc=$?" >> $D/bench.log
grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], round(d['e2e']['value'],2), d['cpu_baseline']['value'], d['roofline']['frac'], d['gpu_launches'])"
