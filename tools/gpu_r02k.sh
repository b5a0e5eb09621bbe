# round-2 call k: importance kernel occupancy A/B (__launch_bounds__(IPT, 6) vs (IPT)) on the full C4 step
D=gpurun_out/r02k; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $D/bench_lb6.log 2>&1
echo "== lb6"; grep "^{" $D/bench_lb6.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:8]})"
sed -i 's/__launch_bounds__(IPT, 6) k_importance8/__launch_bounds__(IPT) k_importance8/' paper_conf_ipps_madougouvln16_b200/csrc/importance.cu
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python bench.py --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > $D/bench_lb0.log 2>&1
echo "== lb0"; grep "^{" $D/bench_lb0.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:8]})"
