# round-2 call an: ballot masks default (BF_TINY_V=2, one position per lane for roots of <= 32 rows); helper warps 2 / 4
D=gpurun_out/r02an; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or tiny or c4" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
for v in "BF_TINY_V=2" "BF_SUBTREE_HW=2" "BF_SUBTREE_HW=4"; do
  env $v timeout 300 python tools/subtree_stats.py c4 > $D/stats.txt 2>&1
  echo "$v"; grep "subtree" $D/stats.txt | head -4
done
for v in "BF_TINY_V=2" "BF_SUBTREE_HW=2" "BF_SUBTREE_HW=4" "BF_TINY_V=2" "BF_SUBTREE_HW=2"; do
  env $v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('$v', {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:2]})"
done
