python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for st in 0 8; do for sw in 4 8; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=128 publish=1 server_workers=$sw ro_streak=$st reps=1; done; done
for cw in 64 256 512; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=$cw publish=1 server_workers=8 ro_streak=8 reps=1; done
timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=128 publish=0 server_workers=8 ro_streak=8 reps=1
timeout 120 python tools/probe.py C3 n_tx=1048576 client_warps=64 publish=1 server_workers=8 ro_streak=16 reps=1
timeout 120 python tools/probe.py C3 n_tx=1048576 client_warps=256 publish=1 server_workers=8 ro_streak=16 reps=1
