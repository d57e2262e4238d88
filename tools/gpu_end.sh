# parity + round-end evidence for the current code
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 1500 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
TAG=r01e bash tools/gpu_profile.sh
timeout 300 python tools/phases.py C4 n_tx=16777216 publish=1 server_workers=6 server_combine=8 ro_streak=32 ro_adaptive=1 log_mode=0 client_warps=294 | cut -c1-900
timeout 300 python tools/phases.py C3 n_tx=4194304 publish=1 server_workers=7 server_recv=1 server_combine=8 ro_streak=8 ro_adaptive=1 log_mode=0 client_warps=294 | cut -c1-900
