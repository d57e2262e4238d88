python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for cb in 1 2 4; do timeout 120 python tools/probe.py C2 n_tx=8388608 client_warps=294 publish=1 server_workers=8 ro_streak=8 server_combine=$cb reps=1; done
for cw in 512 1024; do timeout 120 python tools/probe.py C2 n_tx=8388608 client_warps=$cw publish=1 server_workers=8 ro_streak=8 server_combine=4 reps=1; done
timeout 120 python tools/probe.py C2 n_tx=8388608 client_warps=512 publish=1 server_workers=4 ro_streak=8 server_combine=4 reps=1
timeout 120 python tools/probe.py C2 n_tx=8388608 client_warps=512 publish=0 server_workers=8 ro_streak=8 server_combine=4 reps=1
