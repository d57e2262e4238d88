# parity + round-end evidence for the current code
set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null || exit 1
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/pytest_gpu.log 2>&1; tail -2 gpurun_out/pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; tail -1 gpurun_out/smoke.log
TAG=${TAG:-r01g} bash tools/gpu_profile.sh
for W in C3 C4; do timeout 600 python bench.py --config $W --no-cpu-baseline > gpurun_out/bench_${W}_${TAG:-r01g}.json 2>/dev/null; tail -1 gpurun_out/bench_${W}_${TAG:-r01g}.json | cut -c1-300; done
timeout 300 python tools/phases.py C3 n_tx=4194304 publish=1 server_workers=7 server_recv=1 server_combine=8 ro_streak=8 ro_adaptive=1 log_mode=0 client_warps=294 > gpurun_out/phases_c3.json; cat gpurun_out/phases_c3.json
timeout 300 python tools/phases.py C2 n_tx=16777216 publish=1 server_workers=6 server_combine=8 ro_streak=8 ro_adaptive=1 log_mode=0 client_warps=294 > gpurun_out/phases_c2.json; cat gpurun_out/phases_c2.json
