set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo smoke rc=$? >> gpurun_out/smoke.log
timeout 900 python -m pytest tests -m gpu -x -q -k "not c4_full" > gpurun_out/pytest_gpu.log 2>&1; echo rc=$? >> gpurun_out/pytest_gpu.log
timeout 600 python bench.py --ntree 32 --m-query 1000000 --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/bench_small.log 2>&1; echo rc=$? >> gpurun_out/bench_small.log
for f in gpurun_out/smoke.log gpurun_out/pytest_gpu.log gpurun_out/bench_small.log; do tail -n 5 $f; done
