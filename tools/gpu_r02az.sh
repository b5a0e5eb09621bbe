# round-2 call az: C1-C3 bench lines, twice each (r02ax's C1 steps alternated 24-78 ms)
D=gpurun_out/r02az; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for C in C1 C2 C3 C1 C2 C3; do
  timeout 1200 python bench.py --config $C --steps 5 --warmup 3 > $D/bench_$C.log 2>&1
  grep "^{" $D/bench_$C.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$C', round(d['value'],1), round(d.get('predictions_per_s') or 0), {k: round(v,1) for k,v in d['phases_ms'].items()}, [round(x,1) for x in d['step_ms']], round(d['e2e']['value'],1), round((d['cpu_baseline'] or {}).get('value') or 0, 2))"
  cp $D/bench_$C.log $D/bench_${C}_last.log
done
