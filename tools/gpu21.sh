python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for cw in 294 1176; do timeout 300 python tools/probe.py C4 n_tx=16777216 log_mode=0 client_warps=$cw publish=1 server_workers=6 ro_streak=8 reps=1; done
timeout 300 python tools/probe.py C3 n_tx=4194304 log_mode=0 client_warps=294 publish=1 server_workers=6 ro_streak=8 server_combine=4 reps=1
timeout 300 python tools/probe.py C2 n_tx=16777216 log_mode=0 client_warps=294 publish=1 server_workers=6 ro_streak=8 server_combine=4 reps=1
