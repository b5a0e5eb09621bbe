# usage (on the GPU box, via gpurun): bash tools/gpu_profile_round.sh <round tag>
# Launch list of a reduced bench step + one `ncu --set full` capture of each
# top kernel, summarised into gpurun_out/<tag>/ (numbers under ncu are never
# bench values).  Copy the .txt/.json summaries into profiles/<tag>/.
R=${1:-r01}
O=gpurun_out/$R
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
B="bench.py --ntree 40 --m-query 10000000 --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
timeout 1800 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches.csv python $B > $O/launch_run.log 2>&1
echo "launch list rc=$?"
python tools/ncu_summary.py launches $O/launches.csv $O/launch_summary.txt | head -25
# kernel, launches to skip (a representative launch of the second batch / a mid level)
for spec in "k_subtree 1" "k_partition_tree 40" "k_split_scan_tree 40" "k_predict8 3" "k_importance8 1" "k_perm_fill 1" "k_list_scatter 1"; do
  set -- $spec
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$1 -s $2 -c 1 -f -o $O/prof_$1 python $B > $O/ncu_$1.log 2>&1
  echo "$1 rc=$?"
  python tools/ncu_summary.py full $O/prof_$1.ncu-rep $O/full_$1 > /dev/null 2>&1
  head -3 $O/full_$1.txt
done
# keep only the subtree report (source view); the rest are summarised
ls $O/*.ncu-rep | grep -v k_subtree | xargs rm -f
du -sh $O
