# round-2 call ae: OOB importance on the two-level groups (k_importance32), ILP 3 / 4
D=gpurun_out/r02ae; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_predict32.py tests/test_gpu_predict8.py tests/test_gpu_parity.py -m gpu -q -rf -x -k "importance or oob or c4 or config or predict32" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for v in "BF_PREDICT_V=2" "BF_IMP32_ILP=3" "BF_IMP32_ILP=4"; do
    env $v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('$v', 'importance_ms=%.1f'%d['phases_ms']['importance'], {k: round(v['ms_per_step'],1) for k,v in d['kernels'].items() if 'imp' in k or 'perm' in k or 'g32' in k or 'pack' in k})"
  done
fi
