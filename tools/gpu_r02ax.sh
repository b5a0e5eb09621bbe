# round-2 call ax: C1-C3 bench lines with the final code (oracle beside them) and their top kernels' ncu summaries
D=gpurun_out/r02ax; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for C in C1 C2 C3; do
  timeout 1200 python bench.py --config $C --steps 5 --warmup 3 > $D/bench_$C.log 2>&1; echo "$C rc=$?"
  grep "^{" $D/bench_$C.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],1), d.get('predictions_per_s'), {k: round(v,1) for k,v in d['phases_ms'].items()}, d['roofline']['kernel'], (d['cpu_baseline'] or {}).get('value'))"
  K=$(grep "^{" $D/bench_$C.log | python -c "import json,sys; print(json.loads(sys.stdin.read())['roofline']['kernel'])")
  timeout 600 ncu --set full --metrics l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,lts__t_bytes.sum --clock-control none --import-source on -k regex:$K -s 2 -c 1 -f -o $D/prof_${K}_$C python bench.py --config $C --steps 1 --warmup 1 --no-e2e --no-cpu-baseline --no-profile > $D/ncu_$C.log 2>&1
  python tools/ncu_summary.py full $D/prof_${K}_$C.ncu-rep $D/full_${K}_$C > /dev/null 2>&1; head -2 $D/full_${K}_$C.txt
  rm -f $D/prof_${K}_$C.ncu-rep
done
