# round-2 call ba: medium-level finalize by the warp that completes a node's last item (no barrier before it)
D=gpurun_out/r02ba; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1500 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or c4 or tiny" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
timeout 300 python tools/subtree_stats.py c4 > $D/stats.txt 2>&1; grep "subtree" $D/stats.txt | head -4
for r in 1 2; do
  timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print({k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:3]})"
done
