# usage (GPU box): bash tools/ab_subtree.sh <tag> — k_subtree time on a 200-tree C4 step, twice
mkdir -p gpurun_out/ab
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for r in 1 2; do
  timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ab/$1_$r.json 2>/dev/null
  python -c "
import json; d=json.loads(open('gpurun_out/ab/$1_$r.json').read().strip().splitlines()[-1])
print('$1 run $r', 'fit_ms=%.1f'%d['phases_ms']['fit'], 'subtree_ms=%.1f'%d['kernels']['k_subtree']['ms_per_step'])"
done
