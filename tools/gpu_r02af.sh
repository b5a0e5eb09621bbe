# round-2 call af: y_q persisting in L2 during the fit (access-policy window) -- parity + A/B
D=gpurun_out/r02af; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or c4" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for v in 0 1 0 1; do
    BF_YQ_PERSIST=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('persist=$v', 'fit_ms=%.1f'%d['phases_ms']['fit'], {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:5]})"
  done
fi
for v in 2 3; do
  BF_IMP32_ILP=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('ilp=$v', 'importance_ms=%.1f'%d['phases_ms']['importance'], {k: round(v['ms_per_step'],1) for k,v in d['kernels'].items() if 'imp' in k})"
done
