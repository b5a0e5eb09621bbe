# round-2 call j: L2 persisting window over the predict tree block (A/B), predict parity
D=gpurun_out/r02j; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_predict8.py tests/test_gpu_parity.py -m gpu -q -rf -x -k "predict or config or c4_bench or host" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 3 $D/pytest.log
for V in "" "BF_PREDICT_L2WIN=0"; do
  env $V timeout 900 python bench.py --ntree 200 --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $D/bench_${V:-default}.log 2>&1
  echo "== ${V:-default}"; grep "^{" $D/bench_${V:-default}.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), {k: round(v,1) for k,v in d['phases_ms'].items()}, d['predictions_per_s'])"
done
