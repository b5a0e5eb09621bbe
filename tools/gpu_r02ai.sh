# round-2 call ai: split scan with 5 / 7 / 9 entries per thread (6 / 5 / 4 CTAs per SM)
D=gpurun_out/r02ai; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for v in 5 7; do
  BF_SCAN_TSV=$v timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config" > $D/pytest_$v.log 2>&1; echo "pytest tsv=$v rc=$?"
done
for v in 9 5 7 9 5; do
  BF_SCAN_TSV=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
  python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print('tsv=$v', {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:4]})"
done
timeout 600 python tools/subtree_stats.py c4 > $D/stats.txt 2>&1
grep "subtree" $D/stats.txt | head -4
