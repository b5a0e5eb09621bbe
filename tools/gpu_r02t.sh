# round-2 call t: partition ring 2 (restore), workflows on device, importance counters -- GPU suite + bench
D=gpurun_out/r02t; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q -rf > $D/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $D/pytest_gpu.log
tail -n 3 $D/pytest_gpu.log
timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $D/bench.log 2>&1
grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:8]}, d['importance_node_loads'], d['importance_rewalks'], d['predict_node_visits_per_walk'])"
