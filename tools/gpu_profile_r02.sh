# usage (on the GPU box, via gpurun): bash tools/gpu_profile_r02.sh <tag>
# C4 launch list of a 74-tree step (two batches of 37 trees, as bench.py fits them) with the 10M-row query batch,
# one `ncu --set full` capture of each top kernel (+ shared-memory pipe and L2 byte counters), summarised into
# gpurun_out/<tag>/; numbers taken under ncu are never bench values.
R=${1:-r02e}
O=gpurun_out/$R
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
X="--metrics l1tex__data_pipe_lsu_wavefronts_mem_shared.avg.pct_of_peak_sustained_elapsed,l1tex__data_pipe_lsu_wavefronts_mem_shared.sum,lts__t_bytes.sum"
B="bench.py --ntree 74 --m-query 10000000 --steps 1 --warmup 0 --no-e2e --no-cpu-baseline --no-profile"
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python $B > $O/launch_run.log 2>&1
echo "launch list rc=$?"
python tools/ncu_summary.py launches $O/launches.csv $O/launch_summary.txt | head -16
for spec in "k_subtree 0" "k_partition_tree 4" "k_split_scan_tree 4" "k_predict32 3" "k_importance32 1"; do
  set -- $spec
  timeout 900 ncu --set full $X --clock-control none --import-source on -k regex:$1 -s $2 -c 1 -f -o $O/prof_$1 python $B > $O/ncu_$1.log 2>&1
  echo "$1 rc=$?"
  python tools/ncu_summary.py full $O/prof_$1.ncu-rep $O/full_$1 > /dev/null 2>&1
  ncu -i $O/prof_$1.ncu-rep --page details --print-details all > $O/details_$1.txt 2>&1
  head -3 $O/full_$1.txt
done
ls $O/*.ncu-rep | grep -v k_subtree | xargs rm -f
du -sh $O
