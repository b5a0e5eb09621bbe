# round-2 call h: split scan: warp-level running bests, one block merge per item (3 barriers per unit)
D=gpurun_out/r02l; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 3 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $D/bench.log 2>&1
  grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:7]})"
  BF_FIT_TIMING=1 timeout 900 python bench.py --m-query 0 --steps 1 --warmup 1 --no-cpu-baseline --no-e2e --no-profile > $D/fit_timing.txt 2>&1
  grep "fit timing" $D/fit_timing.txt | tail -2
fi
