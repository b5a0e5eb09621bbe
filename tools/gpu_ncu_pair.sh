# usage: bash tools/gpu_ncu_pair.sh "<bench args>" kernel1 skip1 [kernel2 skip2 ...]
# one `ncu --set full` capture per kernel, summarised into gpurun_out/full_<kernel>.{txt,json}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
BA="$1"; shift
while [ $# -ge 2 ]; do
  K=$1; S=$2; shift 2
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:$K -s $S -c 1 -f -o gpurun_out/prof_$K python bench.py $BA > gpurun_out/ncu_$K.log 2>&1; echo "ncu $K rc=$?"
  python tools/ncu_summary.py full gpurun_out/prof_$K.ncu-rep gpurun_out/full_$K > /dev/null 2>&1
  head -40 gpurun_out/full_$K.txt
done
