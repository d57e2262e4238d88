python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
for cs in 2 4 8 16; do timeout 300 python tools/probe.py C2 n_tx=16777216 log_mode=0 client_warps=294 publish=1 server_workers=6 ro_streak=8 server_combine=4 server=1 cluster_size=$cs reps=1; done
timeout 300 python tools/probe.py C2 n_tx=16777216 log_mode=0 client_warps=294 publish=1 server_workers=6 ro_streak=8 server_combine=4 reps=1
