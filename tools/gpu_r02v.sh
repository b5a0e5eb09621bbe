# round-2 call u: importance re-walks started at the divergence point (PATH, 8 checks per batch) -- parity, A/B bench
D=gpurun_out/r02v; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_predict8.py tests/test_gpu_workflows.py -m gpu -q -rf -x -k "importance or oob or c4_bench or workflows or scaling" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for V in "" "BF_IMP_PATH=0"; do
    env $V timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $D/bench_${V:-default}.log 2>&1
    echo "== ${V:-default}"; grep "^{" $D/bench_${V:-default}.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], {k: round(v,1) for k,v in d['phases_ms'].items()}, round(d['kernels']['k_importance8']['ms_per_step'],1), d['importance_node_loads'], d['importance_rewalks'])"
  done
fi
