# usage: bash tools/gpu_run.sh "<pytest -k expr or SKIP>" "<bench args or SKIP>" [extra cmd]
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
if [ "$1" != "SKIP" ]; then
  timeout 1500 python -m pytest tests -m gpu -x -q -k "$1" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/pytest_gpu.log
  tail -n 4 gpurun_out/pytest_gpu.log
fi
if [ "$2" != "SKIP" ]; then
  timeout 1200 python bench.py $2 > gpurun_out/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/bench.log
  tail -c 3000 gpurun_out/bench.log
fi
if [ -n "$3" ]; then eval "$3"; fi
