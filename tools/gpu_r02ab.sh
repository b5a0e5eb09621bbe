# round-2 call ab: tiny roots of up to 128 rows (lane-per-feature search); A/B vs 64
D=gpurun_out/r02ab; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for v in 64 128; do
    BF_TINY_MAX=$v timeout 600 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1
    echo "TT=$v"; grep "subtree" $D/stats_$v.txt | head -4
  done
  for v in 64 128 64 128; do
    BF_TINY_MAX=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $D/ab_$v.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$D/ab_$v.json').read().strip().splitlines()[-1])
print('TT=$v', 'fit_ms=%.1f'%d['phases_ms']['fit'], {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:4]})"
  done
fi
