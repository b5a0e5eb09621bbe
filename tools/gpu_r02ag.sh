# round-2 call ag: subtree load phase with the next item's chunks in flight; packed pointer jumping for the G32 build
D=gpurun_out/r02ag; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_predict32.py -m gpu -q -rf -x -k "topology or config or c4 or predict32 or importance32 or tiny" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  timeout 600 python tools/subtree_stats.py c4 > $D/stats.txt 2>&1
  grep "subtree" $D/stats.txt | head -4
  timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('fit_ms=%.1f'%d['phases_ms']['fit'], {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:12]})"
fi
