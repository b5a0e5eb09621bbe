# round-2 call aj: tiny roots queued before the tiny phase taken largest first (LPT) -- parity, stats, A/B
D=gpurun_out/r02aj; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or tiny or c4" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for v in 0 1; do
    BF_TQ_LPT=$v timeout 600 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1
    echo "lpt=$v"; grep "subtree\]" $D/stats_$v.txt | head -2
  done
  for v in 0 1 0 1; do
    BF_TQ_LPT=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('lpt=$v', {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:2]})"
  done
fi
