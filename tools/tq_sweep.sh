# usage (GPU box): bash tools/tq_sweep.sh — k_subtree tiny-queue knobs on a 200-tree C4 step (fit share)
mkdir -p gpurun_out/tq
for cfg in "2048 0" "2048 1" "512 1" "256 1" "128 1" "256 0"; do
  set -- $cfg
  BF_TQ_SLEEP_MAX=$1 BF_TQ_BIGGER_FIRST=$2 timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/tq/s$1_b$2.json 2> gpurun_out/tq/s$1_b$2.err
  python -c "
import json,sys; d=json.loads(open('gpurun_out/tq/s$1_b$2.json').read().strip().splitlines()[-1])
print('sleep=$1 bigger=$2', 'fit_ms=%.1f'%d['phases_ms']['fit'], 'subtree_ms=%.1f'%d['kernels']['k_subtree']['ms_per_step'], 'trees/s=%.2f'%d['value'])"
done
timeout 300 python tools/subtree_stats.py c4 > gpurun_out/tq/stats.txt 2>&1; grep -i "subtree" gpurun_out/tq/stats.txt | head -20
