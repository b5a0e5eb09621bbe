# round-2 call m: C1-C3 ncu captures (k_subtree and k_predict8, shared-memory pipe metrics) + partition barrier change A/B data
D=gpurun_out/r02m; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1800 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -x -k "topology or config or c4_bench or degenerate" > $D/pytest.log 2>&1; echo "pytest rc=$?" >> $D/pytest.log
tail -n 2 $D/pytest.log
timeout 900 python bench.py --steps 4 --warmup 2 --no-cpu-baseline --no-e2e > $D/bench.log 2>&1
grep "^{" $D/bench.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print(round(d['value'],2), [round(x) for x in d['step_ms']], {k: round(v,1) for k,v in d['phases_ms'].items()}, {k: round(v['ms_per_step'],1) for k,v in list(d['kernels'].items())[:7]})"
X="--metrics l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,lts__t_bytes.sum"
for C in C1 C2 C3; do
  for K in k_subtree k_predict8; do
    timeout 600 ncu --set full $X --clock-control none --import-source on -k regex:$K -s 0 -c 1 -f -o $D/prof_${K}_$C python bench.py --config $C --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-profile > $D/ncu_${K}_$C.log 2>&1
    python tools/ncu_summary.py full $D/prof_${K}_$C.ncu-rep $D/full_${K}_$C > /dev/null 2>&1; head -2 $D/full_${K}_$C.txt; grep "mem_shared.avg.pct" $D/full_${K}_$C.txt
    rm -f $D/prof_${K}_$C.ncu-rep
  done
done
