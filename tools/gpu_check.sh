# build, GPU parity tests, C2 probe and bench (one gpurun call)
set -x
python -c "import __graft_entry__ as g; g.build()" || exit 1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
timeout 300 python tools/probe.py C2 n_tx=16777216 client_warps=294 publish=1 server_workers=6 server_combine=4 ro_streak=8 reps=3 | cut -c1-400
timeout 300 python bench.py --no-cpu-baseline | tail -1
