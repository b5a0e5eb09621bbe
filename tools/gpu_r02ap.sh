# round-2 call ap: position table built per tiny root by the warp that takes it (BF_TINY_V=3) vs ballot masks (2)
D=gpurun_out/r02ap; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
BF_TINY_V=3 timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or c4" > $D/pytest3.log 2>&1; echo "pytest tv3 rc=$?" >> $D/pytest3.log
tail -n 2 $D/pytest3.log
for v in 3 2; do
  BF_TINY_V=$v timeout 300 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1; echo "tv=$v"; grep "subtree" $D/stats_$v.txt | head -4
done
for v in 3 2 3 2; do
  BF_TINY_V=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('tv=$v', {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:2]})"
done
