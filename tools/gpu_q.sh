python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 600 python tools/tune.py C2 reps=3 "server_workers=6" 2>&1 | cut -c1-230
timeout 900 python -m pytest tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
