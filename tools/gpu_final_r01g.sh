# usage (GPU box): bash tools/gpu_final_r01g.sh — default bench, launch list and a k_subtree capture for r01g
mkdir -p gpurun_out/r01g
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 900 python bench.py > gpurun_out/r01g/bench.log 2>&1; echo "bench rc=$?"
tail -n 1 gpurun_out/r01g/bench.log | cut -c1-300
O=gpurun_out/r01g
B="bench.py --ntree 40 --m-query 10000000 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python $B > $O/launch_run.log 2>&1
echo "launch list rc=$?"
python tools/ncu_summary.py launches $O/launches.csv $O/launch_summary.txt | head -12
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_subtree -s 1 -c 1 -f -o $O/prof_k_subtree python $B > $O/ncu_k_subtree.log 2>&1
echo "k_subtree rc=$?"
python tools/ncu_summary.py full $O/prof_k_subtree.ncu-rep $O/full_k_subtree > /dev/null 2>&1
head -5 $O/full_k_subtree.txt
gzip -f $O/launches.csv
