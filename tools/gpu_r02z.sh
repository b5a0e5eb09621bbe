# round-2 call z: lane-per-feature tiny-node search (BF_TINY_V=1) -- parity, A/B against the staged path, phase counters
D=gpurun_out/r02z; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_predict32.py tests/test_gpu_predict8.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for v in 0 1 0 1; do
    BF_TINY_V=$v timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > $D/ab_$v.json 2>/dev/null
    python -c "
import json; d=json.loads(open('$D/ab_$v.json').read().strip().splitlines()[-1])
print('TV=$v', 'fit_ms=%.1f'%d['phases_ms']['fit'], 'subtree_ms=%.1f'%d['kernels']['k_subtree']['ms_per_step'])"
  done
  for v in 0 1; do
    BF_TINY_V=$v timeout 600 python tools/subtree_stats.py c4 > $D/stats_$v.txt 2>&1
    echo "TV=$v"; grep "subtree" $D/stats_$v.txt | head -4
  done
fi
for v in "2 6 33554432" "3 4 33554432" "3 4 50331648" "3 6 50331648" "3 4 67108864"; do
  set -- $v
  PEXP_CASES=env BF_PREDICT_V=$1 BF_PREDICT32_SLOTS=$2 BF_PREDICT_BLOCK_BYTES=$3 timeout 600 python tools/predict_exp.py 200 10000000 2>&1 | grep -v "^trees" | sed "s/^/pv=$1 slots=$2 blk=$3 /" | head -3
done
