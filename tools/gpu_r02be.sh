# round-2 call be: node-list work space kept across fits (no per-fit allocation of the multi-GB list buffers)
D=gpurun_out/r02be; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1500 python -m pytest tests/test_gpu_parity.py tests/test_gpu_predict32.py -m gpu -q -rf -x > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
timeout 1500 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $D/bench.log 2>&1; echo "bench rc=$?"
grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], round(d['e2e']['value'],2))"
