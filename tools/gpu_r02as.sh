# round-2 call as: step-time growth over consecutive C4 steps (r02ar: 7.9 -> 9.4 s); 32-byte list-init gathers
D=gpurun_out/r02as; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or c4" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
BF_FIT_TIMING=1 timeout 900 python bench.py --steps 8 --warmup 2 --no-e2e --no-cpu-baseline --no-profile > $D/bench_a.log 2> $D/bench_a.err
grep "^{" $D/bench_a.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('default', round(d['value'],2), [round(x) for x in d['step_ms']])"
grep "trees in flight\|total" $D/bench_a.err | head -30
PYTORCH_CUDA_ALLOC_CONF=expandable_segments:True timeout 900 python bench.py --steps 8 --warmup 2 --no-e2e --no-cpu-baseline --no-profile > $D/bench_b.log 2> $D/bench_b.err
grep "^{" $D/bench_b.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('expandable', round(d['value'],2), [round(x) for x in d['step_ms']])"
