# round-2 call bd: C4 headline distribution over 10 steps (final code)
D=gpurun_out/r02bd; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1500 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > $D/bench.log 2>&1; echo "bench rc=$?"
grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], round(d['e2e']['value'],2), d['clocks'])"
