# round-2 call y (final checkpoint of round 2): checkpoint of the restored code -- full GPU suite, smoke, bench with every leg,
# reference arm, launch list + ncu captures (with the details pages)
D=gpurun_out/r02av; mkdir -p $D
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q -rf > $D/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $D/pytest_gpu.log
tail -n 3 $D/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; echo "smoke rc=$?" >> $D/smoke.log; tail -2 $D/smoke.log
timeout 1500 python bench.py --steps 5 --warmup 3 > $D/bench.log 2>&1; echo "bench rc=$?" >> $D/bench.log
grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], d['e2e']['value'], d['cpu_baseline']['value'], d['roofline']['frac'], d['clocks'])"
timeout 900 python bench.py --impl reference --steps 1 --warmup 0 > $D/bench_ref.log 2>&1; echo "ref rc=$?" >> $D/bench_ref.log
grep "^{" $D/bench_ref.log | cut -c1-300
bash tools/gpu_profile_r02.sh r02av
