# round-2 call bh: k_importance32 with the register budget of 6 CTAs per SM (BF_IMP32_ILP=36) vs default
D=gpurun_out/r02bh; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
BF_IMP32_ILP=36 timeout 900 python -m pytest tests/test_gpu_predict32.py tests/test_gpu_predict8.py -m gpu -q -rf -x -k "importance" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
for v in 36 3 36 3; do
  BF_IMP32_ILP=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('ilp=$v', {k: round(v['ms_per_step'],1) for k,v in d['kernels'].items() if 'imp' in k})"
done
