# round-2 call at: list init with 16 trees per pass (32-byte weight gathers): kernel table; predict with 5 walks per thread
D=gpurun_out/r02at; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python bench.py --ntree 200 --m-query 1000000 --steps 3 --warmup 2 --no-e2e --no-cpu-baseline > $D/ab.json 2>/dev/null
python -c "
import json; d=json.loads(open('$D/ab.json').read().strip().splitlines()[-1])
print({k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:12]})"
for v in 4 5 4 5; do
  PEXP_CASES=env BF_PREDICT32_SLOTS=$v timeout 600 python tools/predict_exp.py 200 10000000 2>&1 | grep -v "^trees" | sed "s/^/slots=$v /" | head -2
done
