# round-2 call aq: tiny roots of up to 128 rows with the per-root position table (BF_TINY_MAX=128, TV 3)
D=gpurun_out/r02aq; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
BF_TINY_MAX=128 timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or c4" > $D/pytest.log 2>&1; echo "pytest tt128 rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
for v in 128 64; do
  BF_TINY_MAX=$v timeout 300 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1; echo "tt=$v"; grep "subtree" $D/stats_$v.txt | head -4
done
for v in 128 64 128 64; do
  BF_TINY_MAX=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('tt=$v', {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:3]})"
done
