# round-2 call f: warp-specialised split scan + shared-memory-root predict -- parity, then A/B against the old kernels
D=gpurun_out/r02g; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 3 $D/pytest.log
if grep -q "pytest rc=0" $D/pytest.log; then
  for V in "" "BF_SCAN_WS=0"; do
    env $V timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $D/bench_${V:-default}.log 2>&1
    echo "== ${V:-default}"; grep "^{" $D/bench_${V:-default}.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:7]})"
  done
fi
