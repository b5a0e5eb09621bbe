# round-2 first GPU call: full -m gpu suite, smoke, then a short C4 bench
mkdir -p gpurun_out/r02a
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv,noheader
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q -rf > gpurun_out/r02a/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> gpurun_out/r02a/pytest_gpu.log
tail -n 15 gpurun_out/r02a/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02a/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/r02a/smoke.log
tail -2 gpurun_out/r02a/smoke.log
timeout 1200 python bench.py --steps 3 --warmup 3 > gpurun_out/r02a/bench.log 2>&1; echo "bench rc=$?" >> gpurun_out/r02a/bench.log
tail -c 1500 gpurun_out/r02a/bench.log
