# round-2 call ad: mtry draw by shuffles, tiny-phase node values deferred to the flush; stats + bench
D=gpurun_out/r02ad; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  timeout 600 python tools/subtree_stats.py c4 > $D/stats.txt 2>&1
  grep "subtree" $D/stats.txt | head -4
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $D/bench.log 2>&1
  grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:8]})"
fi
