# round-2 call ay: C1 step-time variance (fit phases)
D=gpurun_out/r02ay; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
BF_FIT_TIMING=1 timeout 600 python bench.py --config C1 --steps 6 --warmup 3 --no-e2e --no-cpu-baseline --no-profile > $D/c1.log 2> $D/c1.err
grep "^{" $D/c1.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), [round(x,1) for x in d['step_ms']], d['phases_ms'])"
grep "total" $D/c1.err | tail -8
