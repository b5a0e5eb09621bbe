# round-2 call bf: allocator test alone (fresh process) and the full GPU suite with the list work space
D=gpurun_out/r02bf; mkdir -p $D
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python -m pytest tests/test_gpu_parity.py -m gpu -q -rf -k "library_memory" > $D/pytest_alloc.log 2>&1; echo "alloc test rc=$?"; tail -1 $D/pytest_alloc.log
timeout 2400 python -m pytest tests -x -q -m gpu > $D/pytest_gpu.log 2>&1; echo "pytest rc=$?" >> $D/pytest_gpu.log
tail -n 3 $D/pytest_gpu.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $D/smoke.log 2>&1; echo "smoke rc=$?" >> $D/smoke.log; tail -2 $D/smoke.log
