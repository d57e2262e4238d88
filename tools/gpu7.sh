python -c "import __graft_entry__ as g; g.build()"
for sw in 2 4 8; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=64 publish=1 server_workers=$sw reps=1; done
for cw in 32 96 128; do timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=$cw publish=1 server_workers=4 reps=1; done
timeout 120 python tools/probe.py C2 n_tx=4194304 client_warps=64 publish=0 server_workers=4 reps=1
timeout 300 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
