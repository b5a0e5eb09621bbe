# round-2 call ac: importance / predict row tiles from a row-major float copy; tiny roots back to 64 rows (A 481)
D=gpurun_out/r02ac; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py tests/test_gpu_predict32.py tests/test_gpu_predict8.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for v in 0 1; do
    PEXP_CASES=env BF_PREDICT_XF=$v timeout 600 python tools/predict_exp.py 200 10000000 2>&1 | grep -v "^trees" | sed "s/^/xf=$v /" | head -3
  done
  timeout 900 python bench.py --steps 3 --warmup 2 --no-cpu-baseline --no-e2e > $D/bench.log 2>&1
  grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:14]})"
fi
