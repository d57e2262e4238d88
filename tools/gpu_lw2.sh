python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
timeout 600 python tools/tune.py C2 reps=2 "server_workers=6" "server=1,cluster_size=4" "server=1,cluster_size=16" "server=1,cluster_size=16,client_warps=441" 2>&1 | cut -c1-250
timeout 300 python tools/tune.py C3 reps=1 "server_workers=7,server_recv=1,n_tx=4194304" 2>&1 | cut -c1-150
