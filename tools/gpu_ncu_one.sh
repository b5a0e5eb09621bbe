# usage: bash tools/gpu_ncu_one.sh <kernel regex> <skip> "<bench args>"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:$1 -s $2 -c 1 -f -o gpurun_out/prof_$1 python bench.py $3 > gpurun_out/ncu_$1.log 2>&1; echo "ncu rc=$?"
tail -n 3 gpurun_out/ncu_$1.log
