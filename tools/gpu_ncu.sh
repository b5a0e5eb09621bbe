# ncu captures of the top kernels on a reduced C4 step (numbers under ncu are never bench values)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
B="bench.py --ntree 16 --m-query 200000 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python $B > gpurun_out/ncu_launch.log 2>&1; echo "launch list rc=$?"
for K in k_subtree k_partition k_split_scan; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s 2 -c 1 -f -o gpurun_out/prof_$K python $B > gpurun_out/ncu_$K.log 2>&1; echo "$K rc=$?"
done
ls -la gpurun_out
